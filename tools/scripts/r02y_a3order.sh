# round 2: attn_tc3 with the scale arrive ordered ahead of the exponentials (A/B)
set -x
L=paper_conf_eurosys_jianglyfdlzllyl26_b200
for s in "1331 4608 24 128 1" "4608 4608 24 128 1" "4916 4096 10 64 1" "600 4096 24 128 8"; do
  timeout 120 python tools/attn_probe.py $s 0; FPS_LIB=$L/libflashps_a3order.so timeout 120 python tools/attn_probe.py $s 0
  timeout 120 python tools/attn_probe.py $s 0; FPS_LIB=$L/libflashps_a3order.so timeout 120 python tools/attn_probe.py $s 0
done
