"""A serving run on the real engine (configs[4]'s one-GPU point; PAPER.md L237 step-level
continuous batching, L326 max batch 8, L90 mask ratios): Poisson arrivals of Flux-scale editing
requests (mask ratios ~ Beta(2, 8.5) clipped to [0.05, 0.6], 28 steps each) join the running
batch at step boundaries and leave after their last step; every step is one fps_run_batch call
over the live requests (KV cache streamed from pinned host, cross-step prefetch, admission
reuse while the batch is unchanged).  Latency = finish - arrival, wall clock, with the device
synchronised at every step boundary (as a serving loop that reports completions must).

The same arrival trace goes through the serving simulator (sched.simulate_serving) with the
latency models this run fitted, so the measured P50 / P95 check the DES's prediction.

  python tools/serve_real.py [load fractions=0.5,0.8] [n_requests=60] > profiles/r02/serving_real_1gpu.json
"""
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import bench
import synth


def main():
    loads = [float(v) for v in (sys.argv[1] if len(sys.argv) > 1 else "0.5,0.8").split(",")]
    n_req = int(sys.argv[2]) if len(sys.argv) > 2 else 60
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    F.require_gpu()
    dev = torch.device("cuda", 0)
    S, MAXB = 28, 8
    w = dict(bench.WORKLOADS["C3"], block="flux", steps=S, batch=MAXB)
    L = w["L_img"] + w["L_txt"]
    layers, mod, cache = bench.build_engine_inputs(F, w, "kv", dev, 2 * 58, 0, 2)
    cm, fit = bench.calibrate(F, w, "kv", layers, cache, [dict()] * 4, dev)
    stream, ls = torch.cuda.current_stream(), torch.cuda.Stream(device=dev)
    eng = F.Engine(layers, w["heads"], F.FPS_MODE_KV, F.FPS_BF16, w["L_img"], w["L_txt"], MAXB, S,
                   synth.delta_table(S), cache, mod_table=mod, plan_policy=0,
                   cost_model=cm.as_engine_model(), mod_width=12 * w["H"], cross_step=True,
                   layer_comp=cm.layer_comp)
    g = synth.rng(4242)
    ratios = synth.sample_mask_ratios(g, n_req)
    masks = [synth.token_mask(synth.mask_blobs(g, 64, 64, float(m)), w["L_txt"]) for m in ratios]
    n_active = [int(mk.sum()) for mk in masks]
    # one-GPU capacity from the model: a full batch of typical requests
    typical = [sched.Request(i, int(np.median(n_active)), L) for i in range(MAXB)]
    cap = MAXB / (cm.step_latency(typical) * S / 1e3)
    gen = torch.Generator(device=dev).manual_seed(5)
    out = {"workload": f"Flux-scale (57 blocks), KV cache from pinned host, {n_req} requests, "
                       f"mask ratios ~ Beta(2, 8.5) clipped [0.05, 0.6], {S} steps, max batch {MAXB}",
           "model_capacity_images_per_s": cap, "fit": fit, "runs": []}
    for lf in loads:
        rate = lf * cap
        arrivals = np.cumsum(g.exponential(1.0 / rate, n_req))
        reqs = [dict(template_id=i % 8, step=0, n_steps=S, mask=torch.as_tensor(masks[i]).to(dev),
                     x=torch.randn(L, w["H"], generator=gen, device=dev).to(torch.bfloat16))
                for i in range(n_req)]
        torch.cuda.synchronize()
        pending, live, finish, steps_run, batch_sizes = list(range(n_req)), [], {}, 0, []
        t0 = time.perf_counter()
        while pending or live:
            now = time.perf_counter() - t0
            while pending and arrivals[pending[0]] <= now and len(live) < MAXB:
                live.append(pending.pop(0))          # joins at this step boundary
            if not live:
                time.sleep(max(0.0, arrivals[pending[0]] - now))
                continue
            batch = [reqs[i] for i in live]
            eng.run_batch(batch, 1, stream=stream, load_stream=ls)
            torch.cuda.synchronize()
            steps_run += 1
            batch_sizes.append(len(live))
            t = time.perf_counter() - t0
            for i in list(live):
                if reqs[i]["step"] >= S:
                    finish[i] = t
                    live.remove(i)                   # leaves at this step boundary
        lat = sorted(finish[i] - arrivals[i] for i in range(n_req))
        pick = lambda q: lat[min(len(lat) - 1, int(np.ceil(q * len(lat))) - 1)]
        makespan = max(finish.values()) - arrivals[0]
        # the serving simulator on the same arrival trace and the models fitted here
        sim_reqs = [sched.Request(i, n_active[i], L, arrival=float(arrivals[i]) * 1e3, steps=S)
                    for i in range(n_req)]
        sim = sched.latency_stats(sched.simulate_serving(sim_reqs, 1, MAXB, cm.step_latency,
                                                         "mask_aware"))
        out["runs"].append({
            "load": lf, "rate_req_per_s": rate, "steps_run": steps_run,
            "mean_batch": statistics.mean(batch_sizes),
            "measured": {"p50_s": pick(0.5), "p95_s": pick(0.95), "mean_s": statistics.mean(lat),
                         "images_per_s": n_req / makespan},
            "simulated": {"p50_s": sim["p50_ms"] / 1e3, "p95_s": sim["p95_ms"] / 1e3,
                          "mean_s": sim["mean_ms"] / 1e3,
                          "images_per_s": n_req / (sim["makespan_ms"] / 1e3)}})
        print(json.dumps(out["runs"][-1]), file=sys.stderr, flush=True)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
