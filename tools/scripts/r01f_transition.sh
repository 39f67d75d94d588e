# KV-mode transition block (R28): engine parity tests, then C3 default bench with it on / off
timeout 900 python -m pytest tests/test_gpu_engine.py tests/test_gpu_double.py tests/test_gpu_sdxl.py -x -q > gpurun_out/r01f_tr_tests.log 2>&1; echo tests=$?
tail -3 gpurun_out/r01f_tr_tests.log
for t in 1 0 1 0; do
timeout 400 python bench.py --no-cpu --no-extras --kv-transition $t > gpurun_out/r01f_tr$t.json 2> gpurun_out/r01f_tr$t.err; echo tr$t=$?
python -c "import json;d=json.loads(open('gpurun_out/r01f_tr$t.json').read().strip().splitlines()[-1]);print('tr$t', d['ms_per_step'], d['e2e']['ms_per_step'], d['plan'])"
done
