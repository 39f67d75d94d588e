# attn_tc5 (d = 64, three rotating S buffers): parity, then tc5 vs tc3 (flag bit 16) at SDXL shapes
set -x
timeout 600 python -m pytest tests/test_gpu_attention.py -q -x 2>&1 | tail -2
for args in "1229 4096 10 64 4" "4096 4096 10 64 4" "307 1024 20 64 4" "1024 1024 20 64 4" "4916 4096 10 64 1"; do
  timeout 120 python tools/attn_probe.py $args 0
  timeout 120 python tools/attn_probe.py $args 65536
done
