# round 2: ncu --set full (with source) of the SDXL-scale GEMMs whose epilogue dominates (K = 640)
set -x
N="ncu --set full --clock-control none --import-source on -s 3 -c 1"
$N -k regex:gemm_tc -o gpurun_out/r02s_gemm_640 python tools/gemm_probe.py 4916 640 640 0 1 bias > gpurun_out/r02s_g1.log 2>&1
$N -k regex:gemm_tc -o gpurun_out/r02s_gemm_5120 python tools/gemm_probe.py 4916 5120 640 0 1 bias > gpurun_out/r02s_g2.log 2>&1
for s in "4916 640 640" "4916 1920 640" "4916 5120 640" "4916 640 2560" "1228 1280 1280" "1228 10240 1280" "1228 1280 5120"; do
  for f in 0 4; do echo "$s f=$f"; python tools/gemm_probe.py $s $f 1 bias; done
done
ls -la gpurun_out/
