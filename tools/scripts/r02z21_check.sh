# engine tests incl. the wide high-priority gather, then C2A / C2B bench lines with attn_tc5
set -x
timeout 1200 python -m pytest tests/test_gpu_engine.py -q -x 2>&1 | tail -2
timeout 1200 python bench.py --config C2A --no-cpu > gpurun_out/r02z21_c2a.json 2> gpurun_out/r02z21_c2a.err
timeout 1200 python bench.py --config C2B --no-cpu > gpurun_out/r02z21_c2b.json 2> gpurun_out/r02z21_c2b.err
for c in c2a c2b; do python -c "import json;d=json.load(open('gpurun_out/r02z21_$c.json'));print('$c', round(d['ms_per_step'],3), d['plan']['cached_blocks'], {k:round(v,3) for k,v in d['extras'].items() if 'ms' in k or 'frac' in k}, {k:(round(v['ms_per_step'],3), v.get('tflops') and round(v['tflops'])) for k,v in d['kernels'].items() if v['ms_per_step']>0.05})"; done
