# attn_tc3 grid reordered (heads fastest): attention parity, then C3 with the TMA row gather on
# 6 / 8 reserved SMs (high-priority load stream) against the whole-entry DMA default
set -x
timeout 900 python -m pytest tests/test_gpu_attention.py -q -x 2>&1 | tail -2
run() { # tag args...
tag=$1; shift
timeout 1500 python bench.py "$@" --steps 8 --warmup 3 --no-extras --no-cpu > gpurun_out/r02z9_$tag.json 2> gpurun_out/r02z9_$tag.err
python -c "import json;d=json.load(open('gpurun_out/r02z9_$tag.json'));print('$tag', round(d['ms_per_step'],2), d['plan']['cached_blocks'], round(d['plan']['predicted_ms_per_step'],1), round(d['plan']['fit'].get('load_gbs'),1), d['plan']['refinement'].get('measured_ms'), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})"
}
run C3_m2 
run C3_m3_8 --copy-method 3 --copy-ctas 8
run C3_m3_6 --copy-method 3 --copy-ctas 6
run C3y_m3_8 --mode y --copy-method 3 --copy-ctas 8
run C3y_m2 --mode y
timeout 2400 python bench.py --config C4 --steps 6 --no-cpu > gpurun_out/r02z9_c4.json 2> gpurun_out/r02z9_c4.err
python -c "import json;d=json.load(open('gpurun_out/r02z9_c4.json'));print('C4', round(d['ms_per_step'],1), d['plan']['cached_blocks'], {k:round(v,2) for k,v in d['extras'].items() if 'ms' in k or 'frac' in k})"
