# round 2: TMA bulk row gather (copy method 3) -- targeted GPU tests, then C3 A/B vs whole-entry DMA
set -x
timeout 600 python -m pytest tests/test_gpu_rows.py tests/test_gpu_engine.py -q -x -k "prefetch or copy_methods or delayed or cross_step" 2>&1 | tail -15
for cm in 3 2 3; do
  timeout 600 python bench.py --steps 10 --warmup 3 --copy-method $cm --no-extras --no-cpu > gpurun_out/r02a_c3_m$cm.json 2> gpurun_out/r02a_c3_m$cm.err
  python -c "import json;d=json.load(open('gpurun_out/r02a_c3_m$cm.json'));print($cm, d['ms_per_step'], d['plan']['cached_blocks'], d['plan']['predicted_ms_per_step'], d['plan']['fit'], d['kernels']['cache_prefetch'], d['clocks'])"
done
