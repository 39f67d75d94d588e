# round 2: attn_tc4 timeline (trace build) + cta vs cluster-scope release on the P arrivals
set -x
FPS_LIB=paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_atrace.so timeout 120 python tools/attn4_trace.py 4608 4608 24
timeout 300 python -m pytest tests/test_gpu_attention.py -x -q -k "pair" 2>&1 | tail -2
for s in "1331 4608 24 128 1" "4608 4608 24 128 1"; do
  timeout 120 python tools/attn_probe.py $s 0; timeout 120 python tools/attn_probe.py $s 4096
  FPS_LIB=paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_a4rel.so timeout 120 python tools/attn_probe.py $s 4096
done
