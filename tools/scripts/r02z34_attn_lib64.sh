# d = 64 attention at the C2A shapes: torch SDPA (cuDNN / flash / efficient) vs ours (attn_tc5, attn_tc3)
set -x
timeout 300 python tools/attn_library_ref.py sdxl
for f in 0 65536; do for n in 1229 4096; do timeout 120 python tools/attn_probe.py $n 4096 10 64 4 $f; done; done
