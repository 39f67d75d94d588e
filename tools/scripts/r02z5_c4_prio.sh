# C4: TMA row gather (method 3) with a high-priority load stream vs whole-entry DMA
set -x
for v in "2 0" "3 0" "3 -5"; do set -- $v
timeout 1500 python bench.py --config C4 --copy-method $1 --load-priority $2 --steps 6 --warmup 3 --no-extras --no-cpu > gpurun_out/r02z5_C4_m$1_p$2.json 2> gpurun_out/r02z5_C4_m$1_p$2.err
python -c "import json;d=json.load(open('gpurun_out/r02z5_C4_m$1_p$2.json'));print('C4 m$1 p$2', round(d['ms_per_step'],1), d['plan']['cached_blocks'], d['plan']['predicted_ms_per_step'], d['plan']['fit'].get('load_gbs'), d['plan']['refinement'], {k:round(v['ms_per_step'],1) for k,v in d['kernels'].items()})"
done
