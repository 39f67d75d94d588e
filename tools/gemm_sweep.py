"""Time fps_linear over the block GEMM shapes for each kernel choice (CUDA events, weights cycled
so they are cold in L2 as in the stack).  python tools/gemm_sweep.py [shape-set]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F

SHAPES = []
for M in (1331, 922, 717, 1741, 2560, 4608):                     # C3 active rows at m = .2 .1 .05 .3 .5, dense
    for N, K in ((9216, 3072), (3072, 3072), (12288, 3072), (3072, 12288)):
        SHAPES.append((M, N, K))
for M, C in ((4 * 1012, 640), (4 * 371, 1280)):                 # C2 levels, batch 4 (mean ratio .3)
    for N, K in ((3 * C, C), (C, C), (4 * C, C), (C, 4 * C)):
        SHAPES.append((M, N, K))
FORCES = {"auto": 0, "1sm": 4, "pair": 8, "swap": 12}
nw = 4
for (M, N, K) in SHAPES:
    a = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    ws = [(torch.randn(N, K, device="cuda") / K ** 0.5).to(torch.bfloat16) for _ in range(nw)]
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    res = {}
    for name, f in FORCES.items():
        F.fps_set_disable_tc(f)
        for i in range(4):
            F.linear(a, ws[i % nw], out=out)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        for i in range(20):
            F.linear(a, ws[i % nw], out=out)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 20
        res[name] = (ms * 1e3, 2 * M * N * K / ms / 1e9)
    F.fps_set_disable_tc(0)
    print(f"{M:6d}x{N:6d}x{K:6d} " + " ".join(f"{k}={v[0]:7.1f}us/{v[1]:5.0f}TF" for k, v in res.items()),
          flush=True)
