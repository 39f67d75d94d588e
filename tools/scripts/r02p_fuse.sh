# round 2: a2 fused into the first cached block (x_full_rows) -- parity suites that cover it
set -x
timeout 2400 python -m pytest tests/test_gpu_block.py tests/test_gpu_double.py tests/test_gpu_engine.py tests/test_gpu_fullscale.py tests/test_gpu_sdxl.py -m gpu -q -x 2>&1 | tail -8
python -c "import __graft_entry__ as g; g.smoke()"
timeout 900 python bench.py --steps 10 --warmup 3 --no-extras --no-cpu > gpurun_out/r02p_c3.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/r02p_c3.json'));print(d['ms_per_step'], d['plan'], d['gpu_launches'])"
