# Round-2 evidence on the final code (second session): ncu launch list of the default command
# first (the bench lines read its per-class summary), GPU suite, smoke, bench lines of every
# config, the two-level SDXL step, 2 ranks (functional), reference arm
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv
FPS_PROFILE_RANGE=1 timeout 1500 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r02g_launches.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu > gpurun_out/r02g_ncu_bench.json 2> gpurun_out/r02g_ncu_bench.err
python tools/ncu_classes.py gpurun_out/r02g_launches.csv C3 2 > /dev/null; mkdir -p gpurun_out/ncu_r02g; cp profiles/ncu/C3_classes.json profiles/ncu/C3_traffic.json gpurun_out/ncu_r02g/
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -4
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 1500 python bench.py > gpurun_out/r02g_c3.json 2> gpurun_out/r02g_c3.err; tail -1 gpurun_out/r02g_c3.err
timeout 1500 python bench.py --mode y --no-cpu > gpurun_out/r02g_c3_y.json 2> gpurun_out/r02g_c3_y.err
timeout 1500 python bench.py --tier hbm --no-extras --no-cpu > gpurun_out/r02g_c3_hbm.json 2> gpurun_out/r02g_c3_hbm.err
timeout 2400 python bench.py --config C4 --steps 6 --no-cpu > gpurun_out/r02g_c4.json 2> gpurun_out/r02g_c4.err
timeout 2400 python bench.py --config C4 --mode kv --steps 6 --no-extras --no-cpu > gpurun_out/r02g_c4_kv.json 2> gpurun_out/r02g_c4_kv.err
timeout 1500 python bench.py --config C2A --no-cpu > gpurun_out/r02g_c2a.json 2> gpurun_out/r02g_c2a.err
timeout 1500 python bench.py --config C2B --no-cpu > gpurun_out/r02g_c2b.json 2> gpurun_out/r02g_c2b.err
timeout 1500 python tools/c2_step.py 10 3 y > gpurun_out/r02g_c2_two_level.json 2> gpurun_out/r02g_c2_two_level.err
FPS_BENCH_TIMEOUT=600 timeout 900 python bench.py --gpus 2 --no-extras --no-cpu > gpurun_out/r02g_c3_2ranks.json 2> gpurun_out/r02g_c3_2ranks.err; tail -2 gpurun_out/r02g_c3_2ranks.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r02g_ref.json 2> gpurun_out/r02g_ref.err
for f in gpurun_out/r02g_*.json; do python -c "
import json
try:
  d=json.load(open('$f'))
  print('$f', d.get('ms_per_step'), d.get('value'), d.get('n_gpus'), (d.get('config') or {}).get('cache_mode'), (d.get('plan') or {}).get('cached_blocks'), (d.get('extras') or {}).get('time_fraction_of_dense'), (d.get('roofline') or {}).get('frac'))
except Exception as e: print('$f', 'ERR', e)
"; done
