# GEMM tile choice with reserved SMs (pair kernel only for >= 2 full pair waves): C3 gather vs DMA
set -x
run() { # tag args...
tag=$1; shift
timeout 1500 python bench.py "$@" --steps 8 --warmup 3 --no-extras --no-cpu > gpurun_out/r02z10_$tag.json 2> gpurun_out/r02z10_$tag.err
python -c "import json;d=json.load(open('gpurun_out/r02z10_$tag.json'));print('$tag', round(d['ms_per_step'],2), d['plan']['cached_blocks'], round(d['plan']['predicted_ms_per_step'],1), round(d['plan']['fit'].get('load_gbs'),1), d['plan']['refinement'].get('measured_ms'), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})"
}
run C3_m2
run C3_m3_8 --copy-method 3 --copy-ctas 8
run C3_m3_6 --copy-method 3 --copy-ctas 6
run C3_m3_4 --copy-method 3 --copy-ctas 4
run C4 --config C4 --steps 6
