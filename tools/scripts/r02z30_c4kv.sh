# C4 KV-mode line again with the step-roofline link-peak fix (max of probe and arena fit)
set -x
timeout 2400 python bench.py --config C4 --mode kv --steps 6 --no-extras --no-cpu > gpurun_out/r02z30_c4_kv.json 2> gpurun_out/r02z30_c4_kv.err
python -c "import json;d=json.load(open('gpurun_out/r02z30_c4_kv.json'));print('c4kv', round(d['ms_per_step'],1), d['step_roofline'])"
