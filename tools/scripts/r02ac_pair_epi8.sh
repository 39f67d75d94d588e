# round 2: 8 epilogue warps in the CTA-pair GEMM too -- parity + A/B + C3 step
set -x
timeout 1200 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_block.py tests/test_gpu_double.py tests/test_gpu_sdxl.py tests/test_gpu_fullscale.py -x -q 2>&1 | tail -3
for s in "1331 3072 15360" "1331 21504 3072" "1331 9216 3072" "4608 9216 3072" "4608 3072 12288" "4608 3072 3072"; do
  for f in 0 2048; do python tools/gemm_probe.py $s $f 1 bias; done
done
timeout 900 python bench.py --no-cpu --no-extras > gpurun_out/r02ac_c3.json 2> gpurun_out/r02ac_c3.err
FPS_KERNEL_FLAGS=2048 timeout 900 python bench.py --no-cpu --no-extras > gpurun_out/r02ac_c3_e4.json 2> gpurun_out/r02ac_c3_e4.err
timeout 900 python bench.py --no-cpu --no-extras > gpurun_out/r02ac_c3b.json 2> gpurun_out/r02ac_c3b.err
python - <<'P'
import json
for f in ['r02ac_c3','r02ac_c3_e4','r02ac_c3b']:
    d=json.load(open(f'gpurun_out/{f}.json')); print(f, d['ms_per_step'], d['value'], d['roofline']['frac'], d['plan']['cached_blocks'] if 'plan' in d else None)
P
