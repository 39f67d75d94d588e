# C4 (Y-mode default) on 2 ranks sharing the one GPU: functional check of --gpus 2 with the shared arena
set -x
FPS_BENCH_TIMEOUT=900 timeout 1200 python bench.py --config C4 --gpus 2 --steps 4 --no-extras --no-cpu > gpurun_out/r02z41_c4_2ranks.json 2> gpurun_out/r02z41_c4_2ranks.err; tail -3 gpurun_out/r02z41_c4_2ranks.err
python -c "import json;d=json.load(open('gpurun_out/r02z41_c4_2ranks.json'));print('c4 2 ranks', d['ms_per_step'], d['value'], d['n_gpus'], d['config'].get('cache_mode'), d['config'].get('cache_tier'))"
