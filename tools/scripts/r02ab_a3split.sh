# round 2: attn_tc3 with the MMA issue split over three warps (S / PV_A / PV_B): parity, A/B
set -x
L=paper_conf_eurosys_jianglyfdlzllyl26_b200
FPS_LIB=$L/libflashps_a3splitw.so timeout 300 python -m pytest tests/test_gpu_attention.py -x -q 2>&1 | tail -2
FPS_LIB=$L/libflashps_a3splitw.so timeout 600 python -m pytest tests/test_gpu_block.py -x -q 2>&1 | tail -2
for s in "1331 4608 24 128 1" "4608 4608 24 128 1" "600 4096 24 128 8" "4916 4096 10 64 1" "1228 1024 20 64 1"; do
  timeout 120 python tools/attn_probe.py $s 0; FPS_LIB=$L/libflashps_a3split.so timeout 120 python tools/attn_probe.py $s 0
  timeout 120 python tools/attn_probe.py $s 0; FPS_LIB=$L/libflashps_a3split.so timeout 120 python tools/attn_probe.py $s 0
done
