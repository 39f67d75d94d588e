for lib in libflashps.so libflashps_epi.so; do
  export FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/$lib
  echo "== $lib"
  python tools/gemm_probe.py 4916 640 640 0 1 bias
  python tools/gemm_probe.py 4916 1920 640 0 1 bias
  python tools/gemm_probe.py 1331 3072 3072 0 1 bias
  python tools/gemm_probe.py 1331 9216 3072 0 1 bias
  python tools/block_probe.py C2A
  python tools/block_probe.py C2B
  python tools/block_probe.py C3
done 2>&1 | grep -E "==|TF|ms/block"
