# attn_tc3 with P released in quarters (pq4 build) vs halves (default): parity, then timing
set -x
FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_pq4.so timeout 600 python -m pytest tests/test_gpu_attention.py -q -x 2>&1 | tail -1
for v in "" _pq4 "" _pq4; do
  for args in "1331 4608 24 128 1 0" "4608 4608 24 128 1 0" "1229 4096 10 64 4 65536"; do
    FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps$v.so timeout 120 python tools/attn_probe.py $args | tail -1 | sed "s/^/lib$v /"
  done
done
