"""Time one masked block (KV-mode) at a bench workload's shapes with per-kernel-class device
times: python tools/block_probe.py CONFIG [kernel flags] [block kind]"""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench
import synth
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F

cfg = sys.argv[1]
flags = int(sys.argv[2]) if len(sys.argv) > 2 else 0
kind = sys.argv[3] if len(sys.argv) > 3 else ("sdxl" if cfg.startswith("C2") else "seq")
w = dict(bench.WORKLOADS[cfg], block=kind, layers=4)
dev = torch.device("cuda", 0)
layers, mod, cache = bench.build_engine_inputs(F, w, "kv", dev, 2, 0, 1)
pool = bench.make_requests(w, w["batch"], bench.SEED)
H, L = w["H"], w["L_img"] + w["L_txt"]
ns = [p["n_active"] for p in pool]
cu_k = np.arange(len(ns) + 1) * L
q_row = torch.as_tensor(np.concatenate([np.flatnonzero(p["mask_np"]) + cu_k[i]
                                        for i, p in enumerate(pool)]).astype(np.int32), device=dev)
Lc = bench.SDXL_CTX[0] if kind == "sdxl" else 0
ctx_kv = torch.randn(len(ns) * Lc, 2 * H, device=dev).to(torch.bfloat16) if Lc else None
b = F.VarlenBatch(ns, [L] * len(ns), q_row=q_row, ctx_kv=ctx_kv, n_ctx=[Lc] * len(ns),
                  act_ids=[np.flatnonzero(p["mask_np"]) for p in pool], L_img=w["L_img"],
                  mod_stride=12 * H if kind == "flux" else 0)
x = torch.randn(sum(ns), H, device=dev).to(torch.bfloat16)
kv = torch.randn(len(ns) * L, 2 * H, device=dev).to(torch.bfloat16)
ws = F.workspace(H, w["F"], F.FPS_BF16, sum(ns), 0, dev)
y = torch.empty_like(x)
F.fps_set_disable_tc(flags)
for _ in range(3):
    for l in layers:
        F.masked_block_forward(l, b, x, kv, y_act=y, ws=ws)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    for l in layers:
        F.masked_block_forward(l, b, x, kv, y_act=y, ws=ws)
e1.record()
torch.cuda.synchronize()
per_block = e0.elapsed_time(e1) / (5 * len(layers))
# the same blocks replayed from a CUDA graph (no host launch cost): if this is much faster, the
# eager number above is host-bound
g = torch.cuda.CUDAGraph()
gs = torch.cuda.Stream()
with torch.cuda.stream(gs):
    with torch.cuda.graph(g, stream=gs):
        for l in layers:
            F.masked_block_forward(l, b, x, kv, y_act=y, ws=ws, stream=gs)
g.replay()
torch.cuda.synchronize()
e0.record()
for _ in range(5):
    g.replay()
e1.record()
torch.cuda.synchronize()
graph_block = e0.elapsed_time(e1) / (5 * len(layers))
F.fps_profile_enable(1)
for l in layers:
    F.masked_block_forward(l, b, x, kv, y_act=y, ws=ws)
torch.cuda.synchronize()
ms, fl, cnt = np.zeros(7), np.zeros(7), np.zeros(7, dtype=np.int64)
P = C.POINTER(C.c_double)
F.fps_profile_read(ms.ctypes.data_as(P), fl.ctypes.data_as(P), None, cnt.ctypes.data_as(C.POINTER(C.c_int64)))
F.fps_profile_enable(0)
names = ["gemm", "attn", "ln", "rows"]
print(f"{cfg} {kind} flags={flags} rows={sum(ns)}: {per_block:.4f} ms/block (graph {graph_block:.4f}) | " +
      " ".join(f"{names[k]} {ms[k] / len(layers):.4f}ms" + (f" {fl[k] / ms[k] / 1e9:.0f}TF/s" if fl[k] else "")
               for k in range(4)))
