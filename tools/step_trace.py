"""Launch timeline of the bench's step (fps_profile_trace: CUDA events around every library
launch, on its own stream).  Prints, per stream, busy time and idle gaps per step, and the
compute stream's idle time right after a wait for a cache load -- where the step is load-bound.
Events around every launch perturb PDL overlap a little; use for structure, not for the number.

  python tools/step_trace.py [C3] [method=3] [k=-1 (planner)] [steps=4] [mode=kv]
"""
import ctypes as C
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import bench
import synth

NAMES = ["gemm", "attn", "ln", "rows", "prefetch", "euler", "index"]


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
    me = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    k = int(sys.argv[3]) if len(sys.argv) > 3 else -1
    K = int(sys.argv[4]) if len(sys.argv) > 4 else 4
    mode = sys.argv[5] if len(sys.argv) > 5 else "kv"
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    F.require_gpu()
    dev = torch.device("cuda", 0)
    w = dict(bench.WORKLOADS[cfg], block="sdxl" if cfg.startswith("C2") else "flux")
    w["steps"] = max(w["steps"], 3 + 2 * K)
    L = w["L_img"] + w["L_txt"]
    pool = bench.make_requests(w, w["batch"], bench.SEED)
    g = torch.Generator(device=dev).manual_seed(bench.SEED)
    layers, mod, cache = bench.build_engine_inputs(F, w, mode, dev, 2 * (w["layers"] + 1), 0, me)
    L_ctx = bench.SDXL_CTX[0] if w["block"] == "sdxl" else 0
    reqs = []
    for i, p in enumerate(pool):
        reqs.append(dict(template_id=i, step=0, n_steps=w["steps"], mask=torch.as_tensor(p["mask_np"]).to(dev),
                         x=torch.randn(L, w["H"], generator=g, device=dev).to(torch.bfloat16)))
        if L_ctx:
            reqs[-1]["ctx"] = torch.randn(*bench.SDXL_CTX, generator=g, device=dev).to(torch.bfloat16)
    stream, ls = torch.cuda.current_stream(), torch.cuda.Stream(device=dev)
    cm, fit = bench.calibrate(F, w, mode, layers, cache, [dict()] * w["batch"], dev)
    N = w["layers"]
    plan = None if k < 0 else [0] * (N - k) + [1] * k
    eng = F.Engine(layers, w["heads"], F.MODE_CODE[mode], F.FPS_BF16, w["L_img"], w["L_txt"],
                   len(reqs), w["steps"], synth.delta_table(w["steps"]), cache, mod_table=mod,
                   slots=0, plan_policy=0 if plan is None else 3, plan=plan,
                   cost_model=cm.as_engine_model(), L_ctx=L_ctx,
                   mod_width=12 * w["H"] if w["block"] == "flux" else 0, cross_step=True)
    ms, _ = bench.run_engine_timed(F, eng, reqs, K, 3, stream, ls, 0, 1)
    F.fps_profile_enable(1)
    ms_p, _ = bench.run_engine_timed(F, eng, reqs, K, 3, stream, ls, 0, 1)
    n = 200000
    st, en = np.zeros(n), np.zeros(n)
    kd, sid = np.zeros(n, np.int32), np.zeros(n, np.int64)
    P = C.POINTER(C.c_double)
    cnt = F.fps_profile_trace(st.ctypes.data_as(P), en.ctypes.data_as(P),
                              kd.ctypes.data_as(C.POINTER(C.c_int32)),
                              sid.ctypes.data_as(C.POINTER(C.c_int64)), n)
    F.fps_profile_enable(0)
    st, en, kd, sid = st[:cnt], en[:cnt], kd[:cnt], sid[:cnt]
    plan_used, pred = eng.last_plan()
    comp = sid[kd == 0][0]
    # the timed steps are the last K of the W + K profiled ones: cut at euler launches
    eul = np.flatnonzero((kd == 5) & (sid == comp))
    t_begin = en[eul[-K - 1]]
    t_end = en[eul[-1]]
    out = {"cfg": cfg, "method": me, "cached": int(sum(plan_used)), "pred_ms": pred,
           "ms_per_step": ms, "ms_per_step_profiled": ms_p,
           "window_ms_per_step": (t_end - t_begin) / K}
    for name, sel in (("compute", sid == comp), ("load", sid != comp)):
        sel = sel & (st >= t_begin) & (en <= t_end + 1e-6)
        s_, e_ = st[sel], en[sel]
        o = np.argsort(s_)
        s_, e_ = s_[o], e_[o]
        busy = (e_ - s_).sum()
        # union of intervals (kernels on one stream do not overlap except via PDL)
        u, cur_s, cur_e = 0.0, None, None
        for a, b in zip(s_, e_):
            if cur_e is None or a > cur_e:
                if cur_e is not None:
                    u += cur_e - cur_s
                cur_s, cur_e = a, b
            else:
                cur_e = max(cur_e, b)
        if cur_e is not None:
            u += cur_e - cur_s
        gaps = np.maximum(s_[1:] - np.maximum.accumulate(e_)[:-1], 0)
        out[name] = {"busy_ms_per_step": busy / K, "union_ms_per_step": u / K,
                     "idle_ms_per_step": ((t_end - t_begin) - u) / K,
                     "gaps_over_20us_per_step": float((gaps > 0.02).sum()) / K,
                     "largest_gaps_ms": sorted(gaps.tolist())[-8:]}
        per = {}
        for kk in range(7):
            m = kd[sel] == kk
            if m.any():
                per[NAMES[kk]] = float((e_[m[o]] - s_[m[o]]).sum() / K) if False else float(
                    (en[sel][m] - st[sel][m]).sum() / K)
        out[name]["per_class_ms_per_step"] = per
    print(json.dumps(out, indent=1))
    dump = os.environ.get("TRACE_OUT")
    if dump:
        np.savez_compressed(dump, st=st, en=en, kd=kd, sid=sid, comp=comp, t0=t_begin, t1=t_end)


if __name__ == "__main__":
    main()
