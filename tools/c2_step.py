"""configs[1] as ONE SDXL request step covering both UNet levels (PAPER.md L79 / L92: SDXL's
transformer blocks sit at several UNet resolutions; L390: SDXL 2.2x at m = 0.2; reading R19:
10 blocks at 64 x 64 / 640 channels -- 4 on the way down, 6 on the way up -- and 60 at
32 x 32 / 1280 channels, in UNet order A(4) -> B(60) -> A(6)).

Each request has ONE editing mask in pixel space (1024 x 1024, blob-shaped, ratios 10/30/50/30 %,
batch 4); fps_mask_to_tokens pools it to each level's token grid (f = 16 for 64 x 64, 32 for
32 x 32; reading R8), so every level runs with its own mask.  A step runs the three level stacks
in UNet order through fps_run_batch on the same compute and load streams (each with its own
template cache in pinned host DRAM, whole-entry DMA, the level's own calibrated planner).  The
convolutions / resamplers between the levels are out of scope: each level keeps
its own hidden state.  Reports ms per step, images/s (50 steps), the dense step on the same
kernels, and per-level times.

  python tools/c2_step.py [steps=10] [warmup=3] [mode=y|kv] > profiles/r02/c2_two_level_step.json

(mode: the cache mode, default y -- the paper's Y caching, Fig. 5-Bottom, which bench.py uses for
the SDXL-scale levels)
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import bench
import synth


def main():
    K = int(sys.argv[1]) if len(sys.argv) > 1 else 10
    W = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    mode = sys.argv[3] if len(sys.argv) > 3 else "y"
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    F.require_gpu()
    dev = torch.device("cuda", 0)
    S_IMG, B = 50, 4
    ratios = [0.1, 0.3, 0.5, 0.3]
    g = synth.rng(1001)
    # one pixel mask per request (1024 x 1024 image), pooled per level on the GPU
    pix = torch.as_tensor(np.stack([synth.mask_blobs(g, 1024, 1024, m).reshape(1024, 1024)
                                    for m in ratios])).to(dev)
    tokA = F.mask_to_tokens(pix, 16)                        # [4, 4096]
    tokB = F.mask_to_tokens(pix, 32)                        # [4, 1024]
    levels = [("A_down", "C2A", 4, tokA), ("B", "C2B", 60, tokB), ("A_up", "C2A", 6, tokA)]
    gen = torch.Generator(device=dev).manual_seed(7)
    ctx = [torch.randn(*bench.SDXL_CTX, generator=gen, device=dev).to(torch.bfloat16) for _ in range(B)]
    stream, ls = torch.cuda.current_stream(), torch.cuda.Stream(device=dev)
    built = []
    for name, cfg, nl, tok in levels:
        w = dict(bench.WORKLOADS[cfg], block="sdxl", layers=nl, steps=max(S_IMG, W + K + 2))
        layers, mod, cache = bench.build_engine_inputs(F, w, mode, dev, 2 * (nl + 1), 0, 2)
        cm, fit = bench.calibrate(F, w, mode, layers, cache, [dict()] * B, dev)
        L = w["L_img"]
        reqs = [dict(template_id=i, step=0, n_steps=w["steps"], mask=tok[i].contiguous(),
                     x=torch.randn(L, w["H"], generator=gen, device=dev).to(torch.bfloat16),
                     ctx=ctx[i]) for i in range(B)]
        built.append(dict(name=name, w=w, layers=layers, cache=cache, cm=cm, fit=fit, reqs=reqs,
                          ratio_tok=[float(tok[i].float().mean()) for i in range(B)]))

    def engines(policy):
        es = []
        for b in built:
            w = b["w"]
            es.append(F.Engine(b["layers"], w["heads"], F.MODE_CODE[mode], F.FPS_BF16, w["L_img"], 0, B,
                               w["steps"], synth.delta_table(w["steps"]), b["cache"], mod_table=None,
                               plan_policy=policy, cost_model=b["cm"].as_engine_model(),
                               L_ctx=bench.SDXL_CTX[0], cross_step=True))
        return es

    def run(es):
        for b in built:
            for r in b["reqs"]:
                r["step"] = 0
        for _ in range(W):
            for e, b in zip(es, built):
                e.run_batch(b["reqs"], 1, stream=stream, load_stream=ls)
        torch.cuda.synchronize()
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(len(es) + 1)]
        per = [0.0] * len(es)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        marks = []
        for _ in range(K):
            for i, (e, b) in enumerate(zip(es, built)):
                a = torch.cuda.Event(enable_timing=True)
                a.record(stream)
                e.run_batch(b["reqs"], 1, stream=stream, load_stream=ls)
                z = torch.cuda.Event(enable_timing=True)
                z.record(stream)
                marks.append((i, a, z))
        e1.record(stream)
        torch.cuda.synchronize()
        for i, a, z in marks:
            per[i] += a.elapsed_time(z) / K
        return e0.elapsed_time(e1) / K, per, [list(e.last_plan()[0]) for e in es]

    out = {"workload": "configs[1] SDXL-scale: one request step over both UNet levels, A(4) -> "
                       "B(60) -> A(6) blocks, batch 4, pixel masks 10/30/50/30 % pooled per level",
           "cache_mode": mode,
           "images_per_step": B, "denoise_steps": S_IMG, "steps": K, "warmup": W}
    ms, per, plans = run(engines(0))
    dms, dper, _ = run(engines(2))
    out.update(ms_per_step=ms, images_per_s=B / (ms * 1e-3 * S_IMG), dense_ms_per_step=dms,
               time_fraction_of_dense=ms / dms, speedup_vs_dense=dms / ms,
               levels=[{"level": b["name"], "blocks": len(b["layers"]), "ms_per_step": per[i],
                        "dense_ms_per_step": dper[i], "cached_blocks": int(sum(plans[i])),
                        "token_mask_ratio": b["ratio_tok"], "fit": b["fit"]}
                       for i, b in enumerate(built)])
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
