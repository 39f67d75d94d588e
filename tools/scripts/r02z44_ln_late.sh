# row-norm loading the modulation vectors after the statistics (48 vs 64 registers): Y-mode C3
set -x
for v in "" _late "" _late "" _late; do
FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps$v.so timeout 900 python bench.py --mode y --steps 10 --warmup 3 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02z44$v.json 2> gpurun_out/r02z44$v.err
python -c "import json;d=json.load(open('gpurun_out/r02z44$v.json'));print('lib$v', round(d['ms_per_step'],3), {k:round(v['ms_per_step'],2) for k,v in d['kernels'].items() if v['ms_per_step']>1})"
done
