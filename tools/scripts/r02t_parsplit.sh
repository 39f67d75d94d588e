# round 2: Y-mode parallel block with the K|V split -- parity, then Y-mode C3 A/B (split on / off)
set -x
timeout 1200 python -m pytest tests/test_gpu_block.py tests/test_gpu_fullscale.py tests/test_gpu_engine.py -m gpu -q -x -k "parallel or single_stream or full_buffer or run_batch or flow or c4" 2>&1 | tail -3
for fl in 0 2048 0 2048; do
FPS_KERNEL_FLAGS=$fl timeout 900 python bench.py --mode y --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02t_y_$fl.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/r02t_y_$fl.json'));print($fl, d['ms_per_step'], d['plan']['cached_blocks'], d['clocks']['sm_mhz'])"
done
