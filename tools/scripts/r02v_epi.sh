# round 2: transposed-store GEMM epilogue -- GEMM parity, per-CTA timeline, times at SDXL / Flux shapes
set -x
timeout 900 python -m pytest tests/test_gpu_gemm.py -m gpu -q -x 2>&1 | tail -3
L=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_gtrace.so
for s in "4916 640 640" "4916 5120 640" "1331 3072 3072"; do FPS_LIB=$L python tools/gemm_trace.py $s 4; done
for s in "4916 640 640" "4916 1920 640" "4916 5120 640" "4916 640 2560" "1331 21504 3072" "1331 3072 15360" "4608 9216 3072" "1331 3072 3072"; do python tools/gemm_probe.py $s 0 4; done
