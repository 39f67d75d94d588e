# grouped (double-stream) GEMMs at one pair wave: 1-SM 256 tile vs pair kernel on ties; Y-mode C3
set -x
for t in 0 1 2 0 1 2; do
FPS_GROUPED_TIE=$t timeout 900 python bench.py --mode y --steps 10 --warmup 3 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02z13_t$t.json 2> gpurun_out/r02z13_t$t.err
python -c "import json;d=json.load(open('gpurun_out/r02z13_t$t.json'));print('tie $t', round(d['ms_per_step'],3), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})"
done
timeout 600 python -m pytest tests/test_gpu_double.py -q -x 2>&1 | tail -1
FPS_GROUPED_TIE=2 timeout 600 python -m pytest tests/test_gpu_double.py -q -x 2>&1 | tail -1
