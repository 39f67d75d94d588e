# Y-mode parallel block: W1(M) + K|V(U) in one grouped launch (per-problem N) -- parity, then A/B
set -x
timeout 1500 python -m pytest tests/test_gpu_block.py tests/test_gpu_engine.py tests/test_gpu_gemm.py -q -x 2>&1 | tail -2
for g in 1 0 1 0; do
FPS_Y_GROUPED=$g timeout 900 python bench.py --mode y --steps 10 --warmup 3 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02z14_g$g.json 2> gpurun_out/r02z14_g$g.err
python -c "import json;d=json.load(open('gpurun_out/r02z14_g$g.json'));print('ygroup $g', round(d['ms_per_step'],3), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})"
done
