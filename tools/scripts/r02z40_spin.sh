# MMA warp spinning vs sleeping in try_wait (FPS_ATTN_MMA_SPIN) on the final attention kernels
set -x
for v in "" _spin "" _spin; do
  for args in "1331 4608 24 128 1 0" "4608 4608 24 128 1 0" "1229 4096 10 64 4 0" "4096 4096 10 64 4 0"; do
    FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps$v.so timeout 120 python tools/attn_probe.py $args | tail -1 | sed "s/^/lib$v /"
  done
done
