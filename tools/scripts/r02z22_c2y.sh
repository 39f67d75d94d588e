# configs[1] with Y caching as the default cache mode (bench C2A / C2B, two-level step)
set -x
timeout 900 python -m pytest tests/test_gpu_sdxl.py -q -x 2>&1 | tail -2
timeout 1200 python bench.py --config C2A --no-cpu > gpurun_out/r02z22_c2a.json 2> gpurun_out/r02z22_c2a.err
timeout 1200 python bench.py --config C2B --no-cpu > gpurun_out/r02z22_c2b.json 2> gpurun_out/r02z22_c2b.err
for c in c2a c2b; do python -c "import json;d=json.load(open('gpurun_out/r02z22_$c.json'));print('$c', d['config']['cache_mode'], round(d['ms_per_step'],3), d['plan']['cached_blocks'], d['roofline']['frac'], {k:round(v,3) for k,v in d['extras'].items() if 'ms' in k or 'frac' in k})"; done
timeout 1200 python tools/c2_step.py 10 3 y > gpurun_out/r02z22_c2_two_level_y.json 2> gpurun_out/r02z22_c2_two_level_y.err
timeout 1200 python tools/c2_step.py 10 3 kv > gpurun_out/r02z22_c2_two_level_kv.json 2> gpurun_out/r02z22_c2_two_level_kv.err
for m in y kv; do python -c "import json;d=json.load(open('gpurun_out/r02z22_c2_two_level_$m.json'));print('two-level $m', round(d['ms_per_step'],3), round(d['dense_ms_per_step'],3), round(d['time_fraction_of_dense'],3))"; done
