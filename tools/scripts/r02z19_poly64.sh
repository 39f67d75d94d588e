# attn_tc5 at d = 64: share of exponentials on the FMA pipe (every N-th group of 8: 2 = 1/2, 3 = 1/3, 4 = 1/4 default, 8 = 1/8)
set -x
for v in "" _p2 _p3 _p8; do
  for args in "1229 4096 10 64 4" "4096 4096 10 64 4" "307 1024 20 64 4"; do
    FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps$v.so timeout 120 python tools/attn_probe.py $args 0 | tail -1 | sed "s/^/lib$v /"
  done
done
