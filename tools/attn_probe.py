"""Time the merged-key attention alone: python tools/attn_probe.py n_active L heads d n_req"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F

n, L, heads, d, R = (int(v) for v in sys.argv[1:6])
if len(sys.argv) > 6:
    F.fps_set_disable_tc(int(sys.argv[6]))                # 16 one-tile, 32 two-tile kernel
H = heads * d
q = torch.randn(R * n, H, device="cuda").to(torch.bfloat16)
kv = torch.randn(R * L, 2 * H, device="cuda").to(torch.bfloat16)
o = torch.empty_like(q)
for _ in range(3):
    F.masked_attention(q, kv, [n] * R, [L] * R, heads, out=o)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
e0.record()
for _ in range(10):
    F.masked_attention(q, kv, [n] * R, [L] * R, heads, out=o)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 10
print(f"attn n={n} L={L} h={heads} d={d} R={R}: {ms:.4f} ms {4 * R * n * L * H / ms / 1e9:.0f} TF/s")
