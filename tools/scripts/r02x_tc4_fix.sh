# round 2: attn_tc4 after ordering the scale arrive + sleeping MMA / correction waits
set -x
L=paper_conf_eurosys_jianglyfdlzllyl26_b200
FPS_LIB=$L/libflashps_atrace.so timeout 120 python tools/attn4_trace.py 4608 4608 24 | tail -32
timeout 300 python -m pytest tests/test_gpu_attention.py -x -q -k "pair" 2>&1 | tail -2
for s in "1331 4608 24 128 1" "4608 4608 24 128 1"; do
  timeout 120 python tools/attn_probe.py $s 0; timeout 120 python tools/attn_probe.py $s 4096
  FPS_LIB=$L/libflashps_a4spin.so timeout 120 python tools/attn_probe.py $s 4096
  FPS_LIB=$L/libflashps_a4poly2.so timeout 120 python tools/attn_probe.py $s 4096
done
