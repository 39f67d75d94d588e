"""§6.6 system overheads measured on the real engine (NEXT-3; routing
decision 0.6 ms, per-step batch assembly 1.2 ms, latent serialisation 1.1 ms + communication
1.3 ms on the paper's H800 system).

  * route decision: Alg. 2 (sched.route) for one new request over 8 workers with 7 running
    requests each -- CalcCost = the library planner over the latency models, per candidate;
  * batch assembly: the admission path of fps_run_batch when the batch changes at a step
    boundary (mask index, host-side varlen metadata, the one host sync, plan) -- a step with a
    changed batch minus a step that reuses the admission, batch of 8 Flux-scale requests;
  * serialisation + communication of a finished request's latent: device -> pinned host copy,
    pickle, and a pipe to a post-processing process (the disaggregated design of §4.3), for the
    Flux VAE latent (4096 x 64 bf16) and for the block-stack hidden state (4608 x 3072 bf16).

  python tools/overheads.py > profiles/r02/overheads.json
"""
import json
import multiprocessing as mp
import os
import pickle
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import bench
import synth


def _sink(conn):
    while True:
        msg = conn.recv_bytes()
        if msg == b"stop":
            break
        pickle.loads(msg)
        conn.send_bytes(b"ok")


def main():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    F.require_gpu()
    dev = torch.device("cuda", 0)
    out = {}
    # ---- route decision -------------------------------------------------------------------
    cm = sched.CostModel(57, 3072, 12288, "kv", comp=(7.2e-13, 0.095), load=(1 / 5.5e7, 0.003),
                         full_entry_rows=4096, layer_comp=[(7.3e-13, 0.097)] * 19 + [(7.1e-13, 0.092)] * 38)
    g = synth.rng(1)
    ratios = synth.sample_mask_ratios(g, 64)
    n_act = [synth.n_masked_for(float(m), 4096) + 512 for m in ratios]
    workers = [[sched.Request(w * 8 + i, n_act[w * 8 + i], 4608) for i in range(7)] for w in range(8)]
    times = []
    for k in range(200):
        r = sched.Request(1000 + k, n_act[k % 64], 4608)
        t0 = time.perf_counter()
        sched.route(r, workers, cm.step_latency, 8)
        times.append((time.perf_counter() - t0) * 1e3)
    out["route_decision_ms"] = {"median": statistics.median(times), "p95": sorted(times)[189],
                                "what": "Alg. 2 over 8 workers x 7 running requests (8 planner calls)",
                                "paper_ms": 0.6}
    # ---- batch assembly (admission) -----------------------------------------------------------
    w = dict(bench.WORKLOADS["C3"], block="flux", steps=28)
    layers, mod, cache = bench.build_engine_inputs(F, w, "kv", dev, 2 * 58, 0, 2)
    L = w["L_img"] + w["L_txt"]
    pool = bench.make_requests(dict(w, ratios=list(np.linspace(0.05, 0.6, 8))), 8, bench.SEED)
    gen = torch.Generator(device=dev).manual_seed(3)
    reqs = [dict(template_id=i, step=0, n_steps=28, mask=torch.as_tensor(p["mask_np"]).to(dev),
                 x=torch.randn(L, w["H"], generator=gen, device=dev).to(torch.bfloat16))
            for i, p in enumerate(pool)]
    eng = F.Engine(layers, 24, F.FPS_MODE_KV, F.FPS_BF16, 4096, 512, 8, 28,
                   synth.delta_table(28), cache, mod_table=mod, plan_policy=1, mod_width=12 * 3072,
                   cross_step=True)
    s, ls = torch.cuda.current_stream(), torch.cuda.Stream()
    res = {}
    for reuse in (1, 0):
        F.fps_engine_set_admission_reuse(eng.h, reuse)
        for r in reqs:
            r["step"] = 0
        eng.run_batch(reqs, 2, load_stream=ls)
        torch.cuda.synchronize()
        dev_ms, host_ms = [], []
        for _ in range(6):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            t0 = time.perf_counter()
            eng.run_batch(reqs, 1, load_stream=ls)
            host_ms.append((time.perf_counter() - t0) * 1e3)
            e1.record(s)
            torch.cuda.synchronize()
            dev_ms.append(e0.elapsed_time(e1))
        res[reuse] = (statistics.median(dev_ms), statistics.median(host_ms))
    out["batch_assembly_ms"] = {
        "step_with_admission_ms": res[0][0], "step_reusing_admission_ms": res[1][0],
        "per_changed_step_ms": res[0][0] - res[1][0],
        "host_ms_of_call_admission": res[0][1], "host_ms_of_call_reuse": res[1][1],
        "what": "fps_run_batch step of 8 Flux-scale requests (57 blocks, all cached) that re-admits "
                "its batch (a request joined or left) minus one that reuses the admission",
        "paper_ms": 1.2}
    eng.close()
    cache.close()
    # ---- latent serialisation + communication --------------------------------------------------
    ctx = mp.get_context("spawn")
    a, b = ctx.Pipe()
    p = ctx.Process(target=_sink, args=(b,))
    p.start()
    ser = {}
    for name, shape in (("flux_vae_latent_4096x64", (4096, 64)), ("stack_hidden_4608x3072", (4608, 3072))):
        x = torch.randn(*shape, device=dev).to(torch.bfloat16)
        host = torch.empty(shape, dtype=torch.bfloat16).pin_memory()
        d2h, sl, comm = [], [], []
        for _ in range(20):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            host.copy_(x)                              # synchronous D2H
            t1 = time.perf_counter()
            blob = pickle.dumps(host.view(torch.int16).numpy(), protocol=5)
            t2 = time.perf_counter()
            a.send_bytes(blob)
            a.recv_bytes()
            t3 = time.perf_counter()
            d2h.append((t1 - t0) * 1e3)
            sl.append((t2 - t1) * 1e3)
            comm.append((t3 - t2) * 1e3)
        ser[name] = {"bytes": int(np.prod(shape) * 2), "d2h_ms": statistics.median(d2h),
                     "serialise_ms": statistics.median(sl),
                     "communicate_ms_incl_deserialise": statistics.median(comm)}
    a.send_bytes(b"stop")
    p.join()
    out["latent_serialisation"] = dict(ser, paper_ms={"serialise": 1.1, "communicate": 1.3})
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
