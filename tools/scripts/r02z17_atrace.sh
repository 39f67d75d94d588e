# attn_tc3 clock64 timeline (one CTA): masked C3, dense C3, SDXL d=64
set -x
FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_atrace.so python tools/attn_trace.py 1331 4608 24 128
FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_atrace.so python tools/attn_trace.py 4608 4608 24 128
FPS_LIB=$PWD/paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_atrace.so python tools/attn_trace.py 4096 4096 10 64
