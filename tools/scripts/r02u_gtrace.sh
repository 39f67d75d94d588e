# round 2: per-CTA timeline of small (SDXL-scale) and Flux-scale 1-SM GEMMs
set -x
L=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_gtrace.so
for s in "4916 640 640" "4916 1920 640" "4916 5120 640" "4916 640 2560" "1331 3072 3072" "4608 9216 3072"; do
  FPS_LIB=$L python tools/gemm_trace.py $s 4
done
