for K in 64 128 256 640 1280; do python tools/gemm_probe.py 4916 640 $K 4; done
for K in 64 640; do python tools/gemm_probe.py 512 256 $K 4; done
python tools/gemm_probe.py 4916 640 640 8
