"""Time one fps_linear shape: python tools/gemm_probe.py M N K [force: 0 auto, 4 1-SM, 8 pair]."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F

M, N, K = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
force = int(sys.argv[4]) if len(sys.argv) > 4 else 0
nw = int(sys.argv[5]) if len(sys.argv) > 5 else 1         # >1: cycle weights (cold in L2)
use_bias = len(sys.argv) > 6 and sys.argv[6] == "bias"
a = torch.randn(M, K, device="cuda").to(torch.bfloat16)
ws = [(torch.randn(N, K, device="cuda") / K ** 0.5).to(torch.bfloat16) for _ in range(nw)]
out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
bias = torch.randn(N, device="cuda").to(torch.bfloat16) if use_bias else None
F.fps_set_disable_tc(force)
for i in range(3):
    F.linear(a, ws[i % nw], bias=bias, out=out)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
e0.record()
for i in range(16):
    F.linear(a, ws[i % nw], bias=bias, out=out)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 16
# the same 16 launches replayed from a CUDA graph: device time without host launch overhead
g = torch.cuda.CUDAGraph()
s = torch.cuda.Stream()
with torch.cuda.stream(s):
    with torch.cuda.graph(g, stream=s):
        for i in range(16):
            F.linear(a, ws[i % nw], bias=bias, out=out)
g.replay()
torch.cuda.synchronize()
e0.record()
for _ in range(4):
    g.replay()
e1.record()
torch.cuda.synchronize()
gms = e0.elapsed_time(e1) / 64
print(f"{M}x{N}x{K} force={force} weights={nw}: {ms:.4f} ms {2 * M * N * K / ms / 1e9:.0f} TF/s | "
      f"graph {gms:.4f} ms {2 * M * N * K / gms / 1e9:.0f} TF/s")
