# register-tile mma.sync attention for <= 128 keys at d = 64 (SDXL cross-attention): parity, timing, C2 lines
set -x
timeout 900 python -m pytest tests/test_gpu_attention.py tests/test_gpu_sdxl.py tests/test_gpu_block.py -q -x 2>&1 | tail -2
for args in "1229 77 10 64 4" "307 77 20 64 4" "4096 77 10 64 4" "1024 77 20 64 4"; do
  timeout 120 python tools/attn_probe.py $args 0
  timeout 120 python tools/attn_probe.py $args 131072
done
for c in C2A C2B; do
timeout 1200 python bench.py --config $c --no-extras --no-cpu > gpurun_out/r02z27_$c.json 2> gpurun_out/r02z27_$c.err
python -c "import json;d=json.load(open('gpurun_out/r02z27_$c.json'));print('$c', d['config']['cache_mode'], round(d['ms_per_step'],3), d['plan']['cached_blocks'])"
done
