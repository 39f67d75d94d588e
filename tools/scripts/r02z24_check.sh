# two-source LN (Y-mode parallel block) bit-identity + parity, Y-mode C3 line, C4 default line with extras
set -x
timeout 900 python -m pytest tests/test_gpu_block.py tests/test_gpu_engine.py -q -x 2>&1 | tail -2
timeout 1500 python bench.py --mode y --no-cpu > gpurun_out/r02z24_c3y.json 2> gpurun_out/r02z24_c3y.err
python -c "import json;d=json.load(open('gpurun_out/r02z24_c3y.json'));print('c3y', round(d['ms_per_step'],3), d['extras']['time_fraction_of_dense'], d['extras']['dense_ms_per_step'], d['e2e']['ms_per_step'])"
timeout 2400 python bench.py --config C4 --steps 6 --no-cpu > gpurun_out/r02z24_c4.json 2> gpurun_out/r02z24_c4.err
python -c "import json;d=json.load(open('gpurun_out/r02z24_c4.json'));print('c4', d['config']['cache_mode'], round(d['ms_per_step'],1), {k:round(v,2) for k,v in d['extras'].items() if 'ms' in k or 'frac' in k})"
