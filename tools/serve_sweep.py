"""configs[4]-style serving sweep, simulated: Poisson arrivals of Flux-scale editing requests
(mask ratios ~ Beta(2, 8.5)) routed to 1/2/4/8 GPU workers by Alg. 2 (mask-aware)
or by request-count baselines, each worker running step-level continuous batching (max batch 8,
L326).  Step latencies come from the Alg. 1 planner over the linear latency models the bench
fitted on a B200 (`plan.fit` of a bench JSON line): a prediction from measured models, not a
multi-GPU measurement (gpurun exposes one GPU).

  python tools/serve_sweep.py profiles/r01e2_bench_c3.json > profiles/r01e2_serving_sim.json
  python tools/serve_sweep.py --mixed C3.json C2A.json C2B.json > profiles/r02/serving_sim_mixed.json
    (configs[4]'s mixed traffic: half the requests SDXL -- two UNet levels, 50 steps -- and half
    Flux, 28 steps; every worker holds both stacks and steps both sub-batches in turn)
Also the NEXT-3 comparisons: router policies at token vs request granularity (§6.5) and the
worker's batching policy -- static / strawman / disaggregated continuous (§6.4).
"""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth
from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched


def _model(b, n_layers, H, F, L_img):
    fit = b["plan"]["fit"]
    mode = b["config"]["cache_mode"]
    comp = (fit["comp_ms_per_tflop"] / 1e12, max(fit["comp_b_ms"], 1e-3))
    load = (1.0 / (fit["load_gbs"] * 1e6), max(fit["load_e_ms"], 1e-3))
    whole = "whole" in b["config"].get("h2d_method", "")
    # the bench fits per batch of `batch_per_gpu` requests; the models are linear in FLOPs / bytes
    return sched.CostModel(n_layers, H, F, mode, comp=comp, load=load,
                           full_entry_rows=L_img if whole else None,
                           kind="sdxl" if b["config"].get("block") == "sdxl" else "seq",
                           Lc=77 if b["config"].get("block") == "sdxl" else 0)


def mixed(files):
    """configs[4]: Poisson arrivals of mixed SDXL / Flux editing requests, 1/2/4/8 workers."""
    b3, b2a, b2b = (json.load(open(f)) for f in files)
    flux = _model(b3, 57, 3072, 12288, 4096)
    sdxl = sched.SdxlCost([_model(b2a, 10, 640, 2560, 4096), _model(b2b, 60, 1280, 5120, 1024)],
                          [4096, 1024])
    cost = sched.MixedCost({"flux": flux, "sdxl": sdxl})
    g = synth.rng(2025)
    n_req = 400
    ratios = synth.sample_mask_ratios(g, n_req)
    kinds = g.random(n_req) < 0.5
    typical = ([sched.Request(i, synth.n_masked_for(0.19, 4096) + 512, 4608, model="flux") for i in range(4)]
               + [sched.Request(4 + i, 0, 4096, model="sdxl", ratio=0.19) for i in range(4)])
    mean_steps = 0.5 * (28 + 50)
    cap = 8 / (cost.step_latency(typical) * mean_steps / 1e3)
    out = {"source_bench": files, "one_gpu_capacity_images_per_s": cap,
           "mix": "50 % Flux (57 blocks, 28 steps) / 50 % SDXL (10 blocks at 64x64/640 + 60 at "
                  "32x32/1280, 50 steps), mask ratios ~ Beta(2, 8.5) clipped [0.05, 0.6] (L90)",
           "runs": []}

    def pool(rate):
        t = np.cumsum(g.exponential(1e3 / rate, n_req))
        reqs = []
        for i in range(n_req):
            m = float(ratios[i])
            if kinds[i]:
                n = synth.n_masked_for(m, 4096)
                reqs.append(sched.Request(i, n + 512, 4608, arrival=float(t[i]), steps=28, tokens=n,
                                          model="flux", ratio=m))
            else:
                n = synth.n_masked_for(m, 4096)
                reqs.append(sched.Request(i, n, 4096, arrival=float(t[i]), steps=50, tokens=n,
                                          model="sdxl", ratio=m))
        return reqs

    for n_gpu in (1, 2, 4, 8):
        for load_frac in (0.5, 0.8, 0.95):
            reqs = pool(load_frac * cap * n_gpu)
            for pol in ("mask_aware", "least_requests", "least_tokens", "round_robin"):
                res = sched.simulate_serving(reqs, n_gpu, 8, cost.step_latency, pol)
                st = sched.latency_stats(res)
                st.update(n_gpus=n_gpu, load=load_frac, policy=pol,
                          images_per_s=n_req / (st["makespan_ms"] / 1e3))
                out["runs"].append(st)
    print(json.dumps(out, indent=1))


def main():
    if sys.argv[1] == "--mixed":
        return mixed(sys.argv[2:5])
    b = json.load(open(sys.argv[1]))
    fit = b["plan"]["fit"]
    mode = b["config"]["cache_mode"]
    comp = (fit["comp_ms_per_tflop"] / 1e12, max(fit["comp_b_ms"], 1e-3))
    load = (1.0 / (fit["load_gbs"] * 1e6), max(fit["load_e_ms"], 1e-3))
    L_img, L_txt, steps = 4096, 512, 28
    whole = "whole" in b["config"].get("h2d_method", "")
    cm = sched.CostModel(57, 3072, 12288, mode, comp=comp, load=load,
                         full_entry_rows=L_img if whole else None)
    g = synth.rng(2024)
    n_req = 400
    ratios = synth.sample_mask_ratios(g, n_req)
    n_active = [synth.n_masked_for(float(m), L_img) + L_txt for m in ratios]
    # capacity of one worker: closed-loop step time of a full batch of 8 typical requests
    typical = [sched.Request(i, int(np.median(n_active)), L_img + L_txt) for i in range(8)]
    cap_img_s = 8 / (cm.step_latency(typical) * steps / 1e3)
    out = {"source_bench": sys.argv[1], "mode": mode, "fit": fit,
           "one_gpu_capacity_images_per_s": cap_img_s, "runs": []}
    tokens = [synth.n_masked_for(float(m), L_img) for m in ratios]

    def pool(rate):
        t = np.cumsum(g.exponential(1e3 / rate, n_req))
        return [sched.Request(i, n_active[i], L_img + L_txt, arrival=float(t[i]), steps=steps,
                              tokens=tokens[i]) for i in range(n_req)]

    for n_gpu in (1, 2, 4, 8):
        for load_frac in (0.5, 0.8, 0.95):
            reqs = pool(load_frac * cap_img_s * n_gpu)              # requests per second
            for pol in ("mask_aware", "least_requests", "least_tokens", "round_robin"):
                res = sched.simulate_serving(reqs, n_gpu, 8, cm.step_latency, pol)
                st = sched.latency_stats(res)
                st.update(n_gpus=n_gpu, load=load_frac, policy=pol,
                          images_per_s=n_req / (st["makespan_ms"] / 1e3))
                out["runs"].append(st)
    # NEXT-3, §6.4 (Fig. 16-Left): one worker (max batch 8) with static batching, the strawman
    # continuous batching whose pre/post-processing interrupts the denoising process (0.36 s per
    # interruption, L398 -- the paper's CPU-side cost, taken as given), and FlashPS's
    # disaggregated continuous batching; P95 latency at several loads
    out["batching"] = []
    for load_frac in (0.3, 0.5, 0.7):
        reqs = pool(load_frac * cap_img_s)
        for bat in ("continuous", "strawman", "static"):
            res = sched.simulate_serving(reqs, 1, 8, cm.step_latency, "mask_aware", bat,
                                         interrupt_ms=360.0)
            st = sched.latency_stats(res)
            st.update(n_gpus=1, load=load_frac, batching=bat, interrupt_ms=360.0)
            out["batching"].append(st)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
