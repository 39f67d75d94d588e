"""clock64 timeline of one attention CTA (developer build `make VARIANT=atrace
EXTRA=-DFPS_ATTN_TRACE`): per key tile kt and query tile t -- S ready (softmax saw bar_s), S in
registers, max done, first half of P stored, second half stored (softmax warp of rows 0-31),
PV on the first / second half issued (MMA warp).  Prints medians over the steady key tiles.

  FPS_LIB=.../libflashps_atrace.so python tools/attn_trace.py n L heads d
"""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
from paper_conf_eurosys_jianglyfdlzllyl26_b200 import _lib

n, L, heads, d = (int(v) for v in sys.argv[1:5])
H = heads * d
q = torch.randn(n, H, device="cuda").to(torch.bfloat16)
kv = torch.randn(L, 2 * H, device="cuda").to(torch.bfloat16)
for _ in range(3):
    F.masked_attention(q, kv, [n], [L], heads)
torch.cuda.synchronize()
lib = C.CDLL(_lib.LIB_PATH)
buf = (C.c_longlong * (2 * 64 * 8))()
assert lib.fps_debug_attn_trace(buf) == 0
t = np.frombuffer(buf, dtype=np.int64).reshape(2, 64, 8).astype(np.float64)
nk = (L + 127) // 128
names = ["S ready", "S loaded", "max", "P half 1", "P half 2", "PV1 issued", "PV2 issued"]
for tile in range(2):
    a = t[tile, 2:min(nk, 64) - 1]
    print(f"tile {tile}: per key-tile step {np.median(np.diff(a[:, 0])):.0f} cycles")
    for s in range(1, 7):
        print(f"  S ready -> {names[s]:<11} {np.median(a[:, s] - a[:, 0]):7.0f} cycles")
