# round 2: 8-warp GEMM epilogue (1-SM kernel) -- parity + A/B against the 4-warp epilogue
set -x
python -m pytest tests/test_gpu_gemm.py tests/test_gpu_sdxl.py tests/test_gpu_block.py tests/test_gpu_double.py -x -q 2>&1 | tail -5
for s in "4916 640 640" "4916 1920 640" "4916 5120 640" "4916 640 2560" "1228 1280 1280" "1228 3840 1280" "1228 10240 1280" "1228 1280 5120" "1331 3072 3072" "4608 3072 3072"; do
  for f in 0 2048; do echo "$s f=$f"; python tools/gemm_probe.py $s $f 1 bias; done
done
python bench.py --config C2A --no-cpu --no-extras 2>/dev/null | tail -1 > gpurun_out/r02t_c2a.json; FPS_KERNEL_FLAGS=2048 python bench.py --config C2A --no-cpu --no-extras 2>/dev/null | tail -1 > gpurun_out/r02t_c2a_e4.json
python bench.py --config C2B --no-cpu --no-extras 2>/dev/null | tail -1 > gpurun_out/r02t_c2b.json
python - <<'P'
import json
for f in ['r02t_c2a','r02t_c2a_e4','r02t_c2b']:
    d=json.load(open(f'gpurun_out/{f}.json')); print(f, d['ms_per_step'], d['roofline']['frac'], d['roofline']['avg_launch_ms'])
P
