# y_split norm in one launch (rows M compact + token rows, rows U token rows): parity, C2A / C2B lines
set -x
timeout 1500 python -m pytest tests/test_gpu_block.py tests/test_gpu_sdxl.py tests/test_gpu_engine.py -q -x 2>&1 | tail -2
for c in C2A C2B; do
timeout 1200 python bench.py --config $c --no-extras --no-cpu > gpurun_out/r02z26_$c.json 2> gpurun_out/r02z26_$c.err
python -c "import json;d=json.load(open('gpurun_out/r02z26_$c.json'));print('$c', d['config']['cache_mode'], round(d['ms_per_step'],3), d['plan']['cached_blocks'])"
done
