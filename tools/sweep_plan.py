"""Measure the engine step for explicit KV-mode suffix plans (k cached blocks) on the bench
workload, to check the planner's choice against the measured optimum.
   python tools/sweep_plan.py [--config C3] [--mode kv] [--tier host] K0 K1 [K2 ...]"""
import argparse, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import bench, synth
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3"); ap.add_argument("--mode", default="kv")
ap.add_argument("--tier", default="host"); ap.add_argument("--steps", type=int, default=8)
ap.add_argument("--cross-step", type=int, default=1)
ap.add_argument("--block", default="flux")
ap.add_argument("--kv-transition", type=int, default=1)
ap.add_argument("ks", type=int, nargs="+")
a = ap.parse_args()
w = bench.WORKLOADS[a.config]
dev = torch.device("cuda", 0)
loc = {"host": 0, "hbm": 1}[a.tier]
w = dict(w, block=a.block)
layers, mod, cache = bench.build_engine_inputs(F, w, a.mode, dev, 2 * (w["layers"] + 1), loc,
                                               2 if loc == 1 else 1)
pool = bench.make_requests(w, w["batch"], bench.SEED)
L = w["L_img"] + w["L_txt"]
g = torch.Generator(device=dev).manual_seed(bench.SEED)
reqs = [dict(template_id=i, step=0, n_steps=w["steps"], mask=torch.as_tensor(p["mask_np"]).to(dev),
             x=torch.randn(L, w["H"], generator=g, device=dev).to(torch.bfloat16))
        for i, p in enumerate(pool)]
L_ctx = bench.SDXL_CTX[0] if a.block == "sdxl" else 0
for r in reqs:
    if L_ctx:
        r["ctx"] = torch.randn(*bench.SDXL_CTX, generator=g, device=dev).to(torch.bfloat16)
ls = torch.cuda.Stream()
N = w["layers"]
for k in a.ks:
    plan = [0] * (N - k) + [1] * k
    eng = F.Engine(layers, w["heads"], F.MODE_CODE[a.mode], F.FPS_BF16, w["L_img"], w["L_txt"],
                   len(reqs), w["steps"], synth.delta_table(w["steps"]), cache, mod_table=mod,
                   slots=0, plan_policy=3, plan=plan, cross_step=bool(a.cross_step),
                   mod_width=12 * w["H"] if a.block == "flux" else 0, L_ctx=L_ctx)
    F.fps_engine_set_kv_transition(eng.h, a.kv_transition)
    ms, _ = bench.run_engine_timed(F, eng, reqs, a.steps, 3, torch.cuda.current_stream(), ls, 0, 1)
    print(f"k={k:2d} cached: {ms:.2f} ms/step", flush=True)
    del eng
