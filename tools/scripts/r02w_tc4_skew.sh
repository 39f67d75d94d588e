# round 2: attn_tc4 per-warp skew (trace build)
set -x
FPS_LIB=paper_conf_eurosys_jianglyfdlzllyl26_b200/libflashps_atrace.so timeout 120 python tools/attn4_trace.py 4608 4608 24 | tail -40
