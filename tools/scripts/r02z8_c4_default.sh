# C4 with its new default H2D (TMA row gather, 8 reserved SMs, high-priority load stream), full
# bench line with extras (the whole-entry DMA arm in the same run); C3 default unchanged
set -x
timeout 600 python -m pytest tests/test_gpu_rows.py tests/test_gpu_engine.py -q -x -k "prefetch or delayed or method" 2>&1 | tail -2
timeout 2400 python bench.py --config C4 --steps 6 --no-cpu > gpurun_out/r02z8_c4.json 2> gpurun_out/r02z8_c4.err; tail -2 gpurun_out/r02z8_c4.err
python -c "import json;d=json.load(open('gpurun_out/r02z8_c4.json'));print('C4', round(d['ms_per_step'],1), d['value'], d['config'].get('h2d_method'), d['plan']['cached_blocks'], d['e2e'], {k:v for k,v in d['extras'].items() if 'ms' in k or 'frac' in k})"
