"""clock64 timeline of one attn_tc4 CTA (leader of pair 1, head 3; developer build
`make VARIANT=atrace EXTRA=-DFPS_ATTN_TRACE`): per key tile kt -- softmax warps of lane quarter 0
(h = 0 / 1): S ready, S loaded, row max exchanged, exponentials done, P stores waited, fence,
arrived; correction warp: scale seen, arrived; MMA warp: V ready, P(keys 0-63) seen,
P(64-127) seen, next S issued.  Cycles
relative to the h = 0 softmax's S-ready stamp of the same kt.

  FPS_LIB=.../libflashps_atrace.so python tools/attn4_trace.py n L heads
"""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
from paper_conf_eurosys_jianglyfdlzllyl26_b200 import _lib

n, L, heads = (int(v) for v in sys.argv[1:4])
d = 128
H = heads * d
q = torch.randn(n, H, device="cuda").to(torch.bfloat16)
kv = torch.randn(L, 2 * H, device="cuda").to(torch.bfloat16)
F.fps_set_disable_tc(4096)
for _ in range(3):
    F.masked_attention(q, kv, [n], [L], heads)
torch.cuda.synchronize()
lib = C.CDLL(_lib.LIB_PATH)
buf = (C.c_longlong * (4 * 64 * 8))()
assert lib.fps_debug_attn4_trace(buf) == 0
t = np.frombuffer(buf, dtype=np.int64).reshape(4, 64, 8).astype(np.float64)
nk = (L + 127) // 128
print("rows: h0 / h1 softmax [S ready, S loaded, max exchanged, exps done, stores waited, "
      "fence+syncwarp, arrived]; corr [scale seen, arrived]; mma [V ready, P1 seen, P2 seen, S+2 issued]")
steps = []
for kt in range(min(nk, 64)):
    b = t[0, kt, 0]
    step = t[0, kt + 1, 0] - b if kt + 1 < min(nk, 64) else float("nan")
    steps.append(step)
    f = lambda row, k: " ".join(f"{int(t[row, kt, j] - b):5d}" for j in k)
    print(f"{kt:2d} | {f(0, range(7))} | {f(1, range(7))} | {f(3, range(2))} | {f(2, range(4))} | {step:6.0f}")
print("median step (cycles):", np.nanmedian(steps[2:-2]))
# per-warp skew (both CTAs of the pair): median over the steady key tiles of each warp's stamps
# relative to softmax warp 4's "max exchanged" stamp of the same kt on the same SM
wb = (C.c_longlong * (2 * 16 * 64 * 2))()
assert lib.fps_debug_attn4_warps(wb) == 0
w = np.frombuffer(wb, dtype=np.int64).reshape(2, 16, 64, 2).astype(np.float64)
ks = list(range(4, min(nk, 64) - 2))
names = {1: "mma [P1 seen, P2 seen]", 2: "mma (PV warp) [P1 seen, P2 seen]", 12: "corr [stat seen, arrived]"}
for rank in range(2):
    print(f"rank {rank}: warp: median offsets [slot0, slot1] vs warp 4 slot0")
    for wi in [1, 2] + list(range(4, 16)):
        if not w[rank, wi, ks[0], 0]:
            continue
        d0 = np.median([w[rank, wi, k, 0] - w[rank, 4, k, 0] for k in ks])
        d1 = np.median([w[rank, wi, k, 1] - w[rank, 4, k, 0] for k in ks])
        print(f"  warp {wi:2d} {names.get(wi, names.get(12) if wi >= 12 else 'softmax [exchanged, P arrived]')}: {d0:7.0f} {d1:7.0f}")
