# round 2: TMA row gather (method 3) vs whole-entry DMA (method 2) per config, bench lines
set -x
timeout 600 python -m pytest tests/test_gpu_rows.py tests/test_gpu_engine.py -q -x -k "prefetch or copy_methods or delayed or cross_step" 2>&1 | tail -3
for cfg in C3 C4 C2A C2B; do
  for cm in 3 2; do
    timeout 900 python bench.py --config $cfg --steps 10 --warmup 3 --copy-method $cm --no-extras --no-cpu > gpurun_out/r02f_${cfg}_m$cm.json 2> gpurun_out/r02f_${cfg}_m$cm.err
    python -c "import json;d=json.load(open('gpurun_out/r02f_${cfg}_m$cm.json'));print('$cfg', $cm, round(d['ms_per_step'],2), d['plan']['cached_blocks'], round(d['plan']['predicted_ms_per_step'],2), round(d['plan']['fit']['load_gbs'] or 0,1), round(d['kernels']['cache_prefetch']['ms_per_step'],2), d['clocks']['sm_mhz'])"
  done
done
