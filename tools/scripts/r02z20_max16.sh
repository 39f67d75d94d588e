# row max with 16 FMNMX3 chains (default build) vs 4 chains (c4 build), attn_tc3 d=128 and attn_tc5 d=64
set -x
timeout 600 python -m pytest tests/test_gpu_attention.py -q -x 2>&1 | tail -2
for v in "" _c4 "" _c4; do
  for args in "1331 4608 24 128 1" "4608 4608 24 128 1" "1229 4096 10 64 4" "4096 4096 10 64 4"; do
    FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps$v.so timeout 120 python tools/attn_probe.py $args 0 | tail -1 | sed "s/^/lib$v /"
  done
done
