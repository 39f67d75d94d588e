# round 2: attn_tc4 with the MMA issue split over two warps (S / PV)
set -x
L=paper_conf_eurosys_jianglyfdlzllyl26_b200
FPS_LIB=$L/libflashps_watch.so timeout 300 python -m pytest tests/test_gpu_attention.py -x -q -k "pair" 2>&1 | tail -2
FPS_LIB=$L/libflashps_watch.so timeout 300 python -m pytest tests/test_gpu_block.py -x -q -k "split_kv" 2>&1 | tail -2
FPS_LIB=$L/libflashps_atrace.so timeout 120 python tools/attn4_trace.py 4608 4608 24 | tail -34
for s in "1331 4608 24 128 1" "4608 4608 24 128 1" "600 4096 24 128 8"; do
  timeout 120 python tools/attn_probe.py $s 0; timeout 120 python tools/attn_probe.py $s 4096
  FPS_LIB=$L/libflashps_a4nosplit.so timeout 120 python tools/attn_probe.py $s 4096
done
