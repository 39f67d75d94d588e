"""Time the merged-key attention alone (device time, host work hoisted out of the loop):
python tools/attn_probe.py n_active L heads d n_req [kernel flags: 16 one-tile, 32 two-tile
smem-P, 48 two-tile P-in-TMEM]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F

n, L, heads, d, R = (int(v) for v in sys.argv[1:6])
if len(sys.argv) > 6:
    F.fps_set_disable_tc(int(sys.argv[6]))
H = heads * d
q = torch.randn(R * n, H, device="cuda").to(torch.bfloat16)
kv = torch.randn(R * L, 2 * H, device="cuda").to(torch.bfloat16)
o = torch.empty_like(q)
cu_q = np.arange(R + 1, dtype=np.int32) * n
cu_k = np.arange(R + 1, dtype=np.int32) * L
d_cu_q, d_cu_k = torch.as_tensor(cu_q).cuda(), torch.as_tensor(cu_k).cuda()
s = F.stream_ptr()


def call():
    F.fps_masked_attention(F.FPS_BF16, q.data_ptr(), kv.data_ptr(), o.data_ptr(), heads, d,
                           d_cu_q.data_ptr(), d_cu_k.data_ptr(), cu_q.ctypes.data,
                           cu_k.ctypes.data, R, s)


for _ in range(3):
    call()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
e0.record()
for _ in range(20):
    call()
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 20
print(f"attn n={n} L={L} h={heads} d={d} R={R} flags={sys.argv[6] if len(sys.argv) > 6 else 0}: "
      f"{ms:.4f} ms {4 * R * n * L * H / ms / 1e9:.0f} TF/s")
