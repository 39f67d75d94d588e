# round 2: SDXL-scale GEMMs (K = 640 / 2560, N = 640 / 1920 / 5120, M = 4916) -- times + one ncu --set full
set -x
for s in "4916 640 640" "4916 1920 640" "4916 5120 640" "4916 640 2560"; do
  for f in 0 4 8; do python tools/gemm_probe.py $s $f 4; done
done
ncu --set full --clock-control none --import-source on -k regex:gemm_tc -s 3 -c 1 -o gpurun_out/r02r_gemm_o python tools/gemm_probe.py 4916 640 640 0 4 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:gemm_tc -s 3 -c 1 -o gpurun_out/r02r_gemm_qkv python tools/gemm_probe.py 4916 1920 640 0 4 > /dev/null 2>&1
