# y_split (sequential / SDXL block, Y-mode): Q over rows M + K|V over all rows in one grouped launch
set -x
timeout 1500 python -m pytest tests/test_gpu_block.py tests/test_gpu_sdxl.py tests/test_gpu_engine.py -q -x 2>&1 | tail -2
for c in C2A C2B C2A C2B; do
timeout 1200 python bench.py --config $c --no-extras --no-cpu > gpurun_out/r02z35_$c.json 2> gpurun_out/r02z35_$c.err
python -c "import json;d=json.load(open('gpurun_out/r02z35_$c.json'));print('$c', round(d['ms_per_step'],3), d['plan']['cached_blocks'], d['roofline']['frac'])"
FPS_KERNEL_FLAGS=32768 timeout 1200 python bench.py --config $c --no-extras --no-cpu > gpurun_out/r02z35_${c}_two.json 2> gpurun_out/r02z35_${c}_two.err
python -c "import json;d=json.load(open('gpurun_out/r02z35_${c}_two.json'));print('$c two-launch', round(d['ms_per_step'],3), d['plan']['cached_blocks'], d['roofline']['frac'])"
done
