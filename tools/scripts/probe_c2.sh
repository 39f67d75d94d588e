set -x
for v in "" _p0 _p3 _p2 _p1; do
  lib=paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps$v.so
  echo "== $v"
  FPS_LIB=$PWD/$lib python tools/attn_probe.py 1229 4096 10 64 4
  FPS_LIB=$PWD/$lib python tools/attn_probe.py 4096 4096 10 64 4
  FPS_LIB=$PWD/$lib python tools/attn_probe.py 307 1024 20 64 4
done
python tools/attn_probe.py 1331 4608 24 128 1
for f in 0 4 8; do
python tools/gemm_probe.py 4916 1920 640 $f
python tools/gemm_probe.py 4916 640 640 $f
python tools/gemm_probe.py 4916 5120 640 $f
python tools/gemm_probe.py 4916 640 2560 $f
python tools/gemm_probe.py 16384 1920 640 $f
python tools/gemm_probe.py 1228 3840 1280 $f
python tools/gemm_probe.py 1228 1280 1280 $f
python tools/gemm_probe.py 1228 10240 1280 $f
python tools/gemm_probe.py 1228 1280 5120 $f
done
