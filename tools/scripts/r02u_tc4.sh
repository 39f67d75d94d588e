# round 2: CTA-pair attention (attn_tc4) -- first parity under the hang-watch build, then A/B
set -x
W=paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_watch.so
FPS_LIB=$W timeout 300 python -m pytest tests/test_gpu_attention.py -x -q -k "pair" 2>&1 | tail -15
FPS_LIB=$W timeout 300 python -m pytest tests/test_gpu_block.py -x -q -k "split_kv" 2>&1 | tail -5
for s in "1331 4608 24 128 1" "4608 4608 24 128 1" "600 4096 24 128 8" "200 4608 24 128 1"; do
  for f in 0 4096; do timeout 120 python tools/attn_probe.py $s $f; done
done
