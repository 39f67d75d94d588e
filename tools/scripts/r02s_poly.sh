# round 2: attention exponentials on the FMA pipe -- share 1/N per build (N = 2, 3, 4 default, 8)
set -x
for lib in libflashps.so libflashps_p2.so libflashps_p3.so libflashps_p8.so; do
  for s in "1331 4608 24 128 1" "4608 4608 24 128 1" "1229 4096 10 64 4" "307 1024 20 64 4"; do
    FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/$lib python tools/attn_probe.py $s | sed "s/^/$lib /"
  done
done
