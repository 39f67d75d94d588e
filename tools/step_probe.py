"""Step-time probe at a bench workload: for several H2D methods and plans (k cached blocks),
the step with loads and the same step with loads skipped (fps_engine_set_skip_loads), so the
exposed load time and the compute-side cost of a method (e.g. reserved SMs) separate.

  python tools/step_probe.py [C3] [methods=3,2] [ks=38,40,42,44] [steps=8]
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch

import bench
import synth


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
    methods = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "3,2").split(",")]
    ks = [int(x) for x in (sys.argv[3] if len(sys.argv) > 3 else "38,40,42,44").split(",")]
    K = int(sys.argv[4]) if len(sys.argv) > 4 else 8
    mode = os.environ.get("PROBE_MODE", "kv")
    bench.COPY_CTAS = int(os.environ.get("PROBE_CTAS", 0))
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    F.require_gpu()
    if os.environ.get("FPS_KERNEL_FLAGS"):
        F.fps_set_disable_tc(int(os.environ["FPS_KERNEL_FLAGS"]))
    dev = torch.device("cuda", 0)
    w = dict(bench.WORKLOADS[cfg], block="sdxl" if cfg.startswith("C2") else "flux")
    w["steps"] = max(w["steps"], 3 + K)
    L = w["L_img"] + w["L_txt"]
    pool = bench.make_requests(w, w["batch"], bench.SEED)
    g = torch.Generator(device=dev).manual_seed(bench.SEED)
    layers, mod, cache = bench.build_engine_inputs(F, w, mode, dev, 2 * (w["layers"] + 1), 0,
                                                   methods[0])
    L_ctx = bench.SDXL_CTX[0] if w["block"] == "sdxl" else 0
    reqs = []
    for i, p in enumerate(pool):
        reqs.append(dict(template_id=i, step=0, n_steps=w["steps"], mask=torch.as_tensor(p["mask_np"]).to(dev),
                         x=torch.randn(L, w["H"], generator=g, device=dev).to(torch.bfloat16)))
        if L_ctx:
            reqs[-1]["ctx"] = torch.randn(*bench.SDXL_CTX, generator=g, device=dev).to(torch.bfloat16)
    # PROBE_LOAD_PRIO: priority of the load stream (lower = higher; torch range [-3, 0] or so)
    prio = int(os.environ.get("PROBE_LOAD_PRIO", 0))
    stream, ls = torch.cuda.current_stream(), torch.cuda.Stream(device=dev, priority=prio)
    deltas = synth.delta_table(w["steps"])
    out = []
    for me in methods:
        c = cache if me == methods[0] else bench.make_cache(F, w, mode, 2 * (w["layers"] + 1), 0, me)
        cm, fit = bench.calibrate(F, w, mode, layers, c, [dict()] * w["batch"], dev)
        for k in [None] + ks:
            N = w["layers"]
            plan = None if k is None else [0] * (N - k) + [1] * k
            eng = F.Engine(layers, w["heads"], F.MODE_CODE[mode], F.FPS_BF16, w["L_img"], w["L_txt"],
                           len(reqs), w["steps"], deltas, c, mod_table=mod, slots=0,
                           plan_policy=0 if k is None else 3, plan=plan,
                           cost_model=cm.as_engine_model(), L_ctx=L_ctx,
                           mod_width=12 * w["H"] if w["block"] == "flux" else 0, cross_step=True)
            row = {"method": me, "k": k}
            for skip in (0, 1):
                F.fps_engine_set_skip_loads(eng.h, skip)
                ms, _ = bench.run_engine_timed(F, eng, reqs, K, 3, stream, ls, 0, 1)
                row["noload_ms" if skip else "ms"] = ms
            used, pred = eng.last_plan()
            row["cached"], row["pred_ms"] = sum(used), pred
            print(json.dumps(row), flush=True)
            out.append(row)
            eng.close()
        print(json.dumps({"method": me, "fit": fit}), flush=True)


if __name__ == "__main__":
    main()
