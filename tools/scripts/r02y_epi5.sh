# round 2: GEMM epilogue (transposed stores, cooperative residual loads) vs the committed one:
# parity, block probes at Flux / SDXL scale, C3 / C2A bench lines
set -x
timeout 1500 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_block.py tests/test_gpu_double.py tests/test_gpu_sdxl.py tests/test_gpu_fullscale.py -m gpu -q -x 2>&1 | tail -3
B=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_base.so
for lib in "" $B; do
  echo "== lib ${lib:-new}"
  FPS_LIB=$lib python tools/block_probe.py C3 0 par 2>&1 | tail -4
  FPS_LIB=$lib python tools/block_probe.py C3 0 flux 2>&1 | tail -4
  FPS_LIB=$lib python tools/block_probe.py C2A 0 sdxl 2>&1 | tail -4
done
for lib in "" $B; do
  FPS_LIB=$lib timeout 900 python bench.py --steps 10 --warmup 3 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02y_c3_${lib:+base}.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/r02y_c3_${lib:+base}.json'));print('C3 ${lib:+base}', d['ms_per_step'], d['plan']['cached_blocks'], d['roofline']['achieved'])"
  FPS_LIB=$lib timeout 900 python bench.py --config C2A --tier hbm --steps 10 --warmup 3 --no-extras --no-cpu --plan-refine 0 > gpurun_out/r02y_c2a_${lib:+base}.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/r02y_c2a_${lib:+base}.json'));print('C2A hbm ${lib:+base}', d['ms_per_step'], d['plan']['cached_blocks'], d['roofline']['achieved'])"
done
