set -x
L=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_gtrace.so
for s in "4916 640 640" "1331 3072 3072"; do FPS_LIB=$L python tools/gemm_trace.py $s 4; done
