# row-norm: one CTA per row (default) vs a grid striding over the rows (FPS_LN_GRID CTAs)
set -x
timeout 600 python -m pytest tests/test_gpu_block.py -q -x -k "flux or parallel or grouped" 2>&1 | tail -1
for g in 0 1184 2368 592 0 1184 2368; do
FPS_LN_GRID=$g timeout 900 python bench.py --mode y --steps 10 --warmup 3 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02z31_g$g.json 2> gpurun_out/r02z31_g$g.err
python -c "import json;d=json.load(open('gpurun_out/r02z31_g$g.json'));print('lngrid $g', round(d['ms_per_step'],3), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})"
done
