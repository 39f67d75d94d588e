#!/usr/bin/env python
"""FlashPS hot-path benchmark on B200.

A step = one denoising step of the whole hot path for one batch of synthetic requests: mask-aware
stack of N blocks (a4-a8) with the Alg. 1 plan, layer-ahead cache prefetch from pinned host DRAM
(a3), replenish (a9) and the sampler update, through fps_run_batch.  Default workload: configs[2]
(Flux-scale DiT stack -- Flux's 19 double-stream + 38 single-stream blocks -- 4096 image + 512
text tokens, H 3072, 24x128 heads, bf16, 20% mask, cached K/V streamed from pinned host per
layer).

  python bench.py [--gpus N --steps K --warmup W --config C3|C4|C2A|C2B --mode kv|y]
  python bench.py --impl reference ...     (the CPU oracle on the same workload)
Multi-GPU: one process per GPU under torchrun; requests are routed to GPUs by Alg. 2 (no data
path collective); value = images/s of all GPUs; timing = max over ranks of device time.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import synth

WORKLOADS = {
    # name: dims, mask ratios (per request), batch, layers, steps
    "C3": dict(H=3072, heads=24, F=12288, L_img=4096, L_txt=512, grid=(64, 64), ratios=[0.2],
               batch=1, layers=57, steps=28, desc="Flux-scale DiT stack, 20% mask, batch 1"),
    "C4": dict(H=3072, heads=24, F=12288, L_img=4096, L_txt=512, grid=(64, 64),
               ratios=list(np.linspace(0.05, 0.60, 16)), batch=16, layers=57, steps=28,
               desc="continuous batch of 16 heterogeneous masks (5-60%), Flux-scale",
               # cache mode: Y (the paper's default; configs[3] does not name one): 473.6
               # ms/step with whole-entry DMA vs 486.7 with the row gather and 522.1 for KV-mode
               # (profiles/r02/c4_mode/).  KV-mode here streams exactly the unmasked rows with the
               # TMA row gather on 8 reserved SMs: whole entries move 1.48x the unmasked bytes
               # (mean m 0.33) -- 524 vs 614 ms/step (profiles/r02/c4_h2d/); at C3 (1.25x) the
               # reserved SMs cost more than the bytes saved
               mode="y", kv_copy_method=3, kv_copy_ctas=8),
    "C2B": dict(H=1280, heads=20, F=5120, L_img=1024, L_txt=0, grid=(32, 32),
                ratios=[0.1, 0.3, 0.5, 0.3], batch=4, layers=60, steps=50,
                desc="SDXL-scale 32x32 level (1280 ch), masks 10/30/50%, batch 4",
               # cache mode: Y (Fig. 5-Bottom, the paper's default; configs[1] does not name
               # one): 12.31 vs 14.49 ms/step for KV in the same run (profiles/r02/c2_y/)
               mode="y"),
    "C2A": dict(H=640, heads=10, F=2560, L_img=4096, L_txt=0, grid=(64, 64),
                ratios=[0.1, 0.3, 0.5, 0.3], batch=4, layers=10, steps=50,
                desc="SDXL-scale 64x64 level (640 ch), masks 10/30/50%, batch 4",
                mode="y"),      # 3.66 vs 4.46 ms/step for KV in the same run
}
SEED = 1003
TIER_NAMES = {"host": "pinned host DRAM", "hbm": "device HBM (NEXT-1)",
              "host_hugepage": "pinned host DRAM on 2 MiB pages",
              "host_shared": "pinned host DRAM, one arena shared by all ranks (memfd)"}
H2D_NAMES = ["SM row gather", "DMA of the unmasked row runs", "DMA of whole entries",
             "TMA bulk row gather (exact rows, reserved SMs)"]
SDXL_CTX = (77, 2048)          # SDXL prompt encoding: 77 tokens x 2048 channels (R24)
FLUX_DOUBLE = 19               # Flux: 19 double-stream blocks, then 38 single-stream (R19, R25)


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def ncu_summary(config, what):
    """The committed ncu summary of the bench's own command for this config (profiles/ncu/):
    what = "classes" (per-class kernel time of one step from the launch list) or "traffic"
    (DRAM bytes per launch of each class over one step's launch mix).  None if absent."""
    p = os.path.join(ROOT, "profiles", "ncu", f"{config}_{what}.json")
    return json.load(open(p)) if os.path.exists(p) else None


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d["hbm_gbs"], d["bf16_tflops"], d.get("bf16_tflops_sustained", d["bf16_tflops"]), "measured"
    return 6650.0, 1590.0, 1400.0, "fallback"


# ---------------------------------------------------------------------------------------
class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index):
        self.index, self.samples, self.proc = index, [], None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.samples.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4)
                          if len(s) > i + 2 and s[i + 2].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(self.samples)}


# ---------------------------------------------------------------------------------------
def make_requests(w, n_requests, seed):
    """Masks shaped like the paper's workloads: blob masks at the config's ratios (L144)."""
    g = synth.rng(seed)
    gh, gw = w["grid"]
    ratios = w["ratios"]
    reqs = []
    for i in range(n_requests):
        m = float(ratios[i % len(ratios)])
        mask = synth.token_mask(synth.mask_blobs(g, gh, gw, m), w["L_txt"])
        reqs.append(dict(ratio=m, mask_np=mask, n_active=int(mask.sum())))
    return reqs


def route_job(pool, w, world, rank, cm):
    """Alg. 2 over the job's request pool (L263-L287): every rank routes the same pool with the
    same cost model (rank 0's fit), so all ranks agree on the assignment without any data-path
    communication; each keeps its share.  Max batch per GPU = the config's batch (C4: 16 of a
    16 x N pool of heterogeneous masks; C3: one request per GPU).
    Returns (this rank's pool indices, the assignment of every rank, held requests)."""
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    L = w["L_img"] + w["L_txt"]
    return sched.shard_requests([p["n_active"] for p in pool], L, world, rank, cm, w["batch"])


COPY_CTAS = 0
LOAD_PRIORITY = 0     # CUDA priority of the cache-load streams (--load-priority)
# Timing the calibration blocks under concurrent loads was tried: the noisier fit (R^2 0.84)
# over-weights the intercept, the planner caches too many blocks and the step gets slower
# (49.9 vs 43.0 ms on C3), so the models are fitted on isolated timings (as the paper does).
LOADED_CALIBRATION = False


SHM_PATH = None      # location 3: the shared arena file every rank maps


def make_cache(F, w, mode, n_entries, location=0, copy_method=0):
    return F.Cache(F.MODE_CODE[mode], F.FPS_BF16, w["H"], w["L_img"], w["layers"], w["steps"],
                   n_templates=64, n_entries=n_entries, copy_method=copy_method, location=location,
                   copy_ctas=COPY_CTAS if location != 1 else 0,
                   shm_path=SHM_PATH if location == 3 else None)


def weight_bytes(w):
    """bf16 bytes of the stack's block weights (what every step streams from HBM)."""
    H, Fd, N, blk = w["H"], w["F"], w["layers"], w.get("block", "seq")
    seq = 3 * H * H + 3 * H + H * H + H + Fd * H + Fd + H * Fd + H
    par = (3 * H + Fd) * H + 3 * H + Fd + H * (H + Fd) + H
    D = SDXL_CTX[1]
    sdxl = 3 * H * H + H * H + H + 2 * Fd * H + 2 * Fd + H * Fd + H + H * H + 2 * H * D + H * H + H + 6 * H
    if blk == "flux":
        n = FLUX_DOUBLE * 2 * seq + (N - FLUX_DOUBLE) * par
    else:
        n = N * {"seq": seq, "par": par, "sdxl": sdxl}[blk]
    return 2 * n


def build_engine_inputs(F, w, mode, device, n_entries, location=0, copy_method=0):
    """Random-init block weights (N(0, 1/fan_in), bf16) and adaLN table on the GPU; pinned cache
    arena (contents do not affect timing; entries alias modulo n_entries)."""
    gen = torch.Generator(device=device).manual_seed(SEED)
    H, Fd, N = w["H"], w["F"], w["layers"]

    def rnd(*shape, scale=1.0):
        return (torch.randn(*shape, generator=gen, device=device) * scale).to(torch.bfloat16)

    layers = []
    D = SDXL_CTX[1]
    flux = w.get("block") == "flux"
    for li in range(N):
        kind = (("double" if li < FLUX_DOUBLE else "par") if flux else w.get("block", "seq"))
        par, sdxl = kind == "par", kind == "sdxl"
        if kind == "double":  # Flux double-stream block: a sequential set per stream (R25)
            t = {}
            for pre, bpre in (("w_", "b_"), ("t_", "tb_")):
                t.update({pre + "qkv": rnd(3 * H, H, scale=H ** -0.5), bpre + "qkv": rnd(3 * H, scale=0.02),
                          pre + "o": rnd(H, H, scale=H ** -0.5), bpre + "o": rnd(H, scale=0.02),
                          pre + "up": rnd(Fd, H, scale=H ** -0.5), bpre + "up": rnd(Fd, scale=0.02),
                          pre + "down": rnd(H, Fd, scale=Fd ** -0.5), bpre + "down": rnd(H, scale=0.02)})
        elif sdxl:     # SDXL UNet transformer block (R24): self-attn, cross-attn, GEGLU
            t = {"w_qkv": rnd(3 * H, H, scale=H ** -0.5),
                 "w_o": rnd(H, H, scale=H ** -0.5), "b_o": rnd(H, scale=0.02),
                 "w_up": rnd(2 * Fd, H, scale=H ** -0.5), "b_up": rnd(2 * Fd, scale=0.02),
                 "w_down": rnd(H, Fd, scale=Fd ** -0.5), "b_down": rnd(H, scale=0.02),
                 "w_q2": rnd(H, H, scale=H ** -0.5), "w_kv2": rnd(2 * H, D, scale=D ** -0.5),
                 "w_o2": rnd(H, H, scale=H ** -0.5), "b_o2": rnd(H, scale=0.02)}
            for i in (1, 2, 3):
                t[f"ln{i}_w"] = (1.0 + rnd(H, scale=0.02).float()).to(torch.bfloat16)
                t[f"ln{i}_b"] = rnd(H, scale=0.02)
            wp, bp = torch.empty_like(t["w_up"]), torch.empty_like(t["b_up"])
            F.fps_geglu_pack(F.FPS_BF16, t["w_up"].data_ptr(), t["b_up"].data_ptr(), Fd, H,
                             wp.data_ptr(), bp.data_ptr(), F.stream_ptr())
            t["w_up"], t["b_up"] = wp, bp
        elif par:    # parallel (Flux single-stream) block: W1 [3H+F, H], W2 [H, H+F] (R23)
            t = {"w_qkv": rnd(3 * H + Fd, H, scale=H ** -0.5), "b_qkv": rnd(3 * H + Fd, scale=0.02),
                 "w_down": rnd(H, H + Fd, scale=(H + Fd) ** -0.5), "b_down": rnd(H, scale=0.02)}
        else:
            t = {"w_qkv": rnd(3 * H, H, scale=H ** -0.5), "b_qkv": rnd(3 * H, scale=0.02),
                 "w_o": rnd(H, H, scale=H ** -0.5), "b_o": rnd(H, scale=0.02),
                 "w_up": rnd(Fd, H, scale=H ** -0.5), "b_up": rnd(Fd, scale=0.02),
                 "w_down": rnd(H, Fd, scale=Fd ** -0.5), "b_down": rnd(H, scale=0.02)}
        layers.append(F.BlockWeights.__new__(F.BlockWeights))
        bw = layers[-1]
        bw.t, bw.H, bw.F, bw.heads, bw.dtype = t, H, Fd, w["heads"], F.FPS_BF16
        bw.kind = F._KIND[kind]
        bw.D_ctx = D if sdxl else 0
        ptrs = lambda keys: [t[k].data_ptr() if k in t else None for k in keys]
        bw.c = F.fps_block_weights(H, w["heads"], H // w["heads"], Fd, F.FPS_BF16,
                                   *ptrs(F._SEQ_KEYS), bw.kind, bw.D_ctx, *ptrs(F._SDXL_KEYS),
                                   *ptrs(("t_qkv", "tb_qkv", "t_o", "tb_o", "t_up", "tb_up",
                                          "t_down", "tb_down")))
    ns = 2 if flux else 1              # double-stream blocks: image 6H then text 6H per row
    mod = torch.zeros(N, w["steps"], ns, 6, H, device=device)
    mod += 0.02 * torch.randn(N, w["steps"], ns, 6, H, generator=gen, device=device)
    mod[:, :, :, 2] += 1.0
    mod[:, :, :, 5] += 1.0
    mod = mod.reshape(N, w["steps"], ns * 6 * H).to(torch.bfloat16)
    if w.get("block") == "sdxl":
        mod = None                    # SDXL blocks are not adaLN-modulated (R24)
    cache = make_cache(F, w, mode, n_entries, location, copy_method)
    return layers, mod, cache


def calibrate(F, w, mode, layers, cache, reqs, device):
    """Fit the §4.4 linear latency models on this GPU (L255-L257): block time vs FLOPs per block
    kind (Flux's stack: the double-stream and the single-stream blocks separately), and
    per-layer cache-load time vs bytes.  Returns (CostModel, fit info)."""
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    link = host_link_gbs(w, mode, device)
    if w.get("block") == "flux":
        fits = [_calibrate_one(F, w, mode, layers, cache, reqs, device, first=f)
                for f in (0, FLUX_DOUBLE)]
        cm, info = fits[0]
        cm_p, info_p = fits[1]
        N = w["layers"]
        cm.layer_comp = [cm.comp] * FLUX_DOUBLE + [cm_p.comp] * (N - FLUX_DOUBLE)
        # the stack-wide (a, b): FLOP-weighted mix, for the callers that take one model
        fd = FLUX_DOUBLE / N
        cm.comp = (fd * cm.comp[0] + (1 - fd) * cm_p.comp[0], fd * cm.comp[1] + (1 - fd) * cm_p.comp[1])
        info = dict(info, comp_double=(info["comp_ms_per_tflop"], info["comp_b_ms"], info["comp_r2"]),
                    comp_single=(info_p["comp_ms_per_tflop"], info_p["comp_b_ms"], info_p["comp_r2"]),
                    comp_ms_per_tflop=cm.comp[0] * 1e12, comp_b_ms=cm.comp[1], link_gbs=link)
        return cm, info
    cm, info = _calibrate_one(F, w, mode, layers, cache, reqs, device)
    info["link_gbs"] = link
    return cm, info


def host_link_gbs(w, mode, device, reps=8):
    """The host link's copy-engine rate: pinned host -> HBM cudaMemcpyAsync of one cache entry
    (L_img rows of the mode's width), back to back (the step roofline's link peak)."""
    nb = max(w["L_img"] * (2 if mode == "kv" else 1) * w["H"] * 2, 64 << 20)
    h = torch.empty(nb, dtype=torch.uint8).pin_memory()
    d = torch.empty(nb, dtype=torch.uint8, device=device)
    d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    best = 0.0
    for _ in range(3):                     # best of 3 (the link is shared with nothing here)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            d.copy_(h, non_blocking=True)
        e1.record()
        torch.cuda.synchronize()
        best = max(best, reps * nb / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    return best


def _calibrate_one(F, w, mode, layers, cache, reqs, device, first=0):
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    H, Fd, L = w["H"], w["F"], w["L_img"] + w["L_txt"]
    B = len(reqs)
    s = torch.cuda.current_stream()
    xs, ys, bx, by = [], [], [], []
    kv = torch.zeros(B * L, 2 * H, dtype=torch.bfloat16, device=device)
    # compute is timed while cache loads stream on the load stream, as they do inside a step:
    # the row gather shares the SMs, so block latency under load is what the planner needs
    Wl = (2 if mode == "kv" else 1) * H
    ld_dst = torch.empty(B * L, Wl, dtype=torch.bfloat16, device=device)
    ld_rows = torch.arange(w["L_img"], device=device, dtype=torch.int32)
    h_ld_rows = np.arange(w["L_img"], dtype=np.int32)
    ld_items = [F.fps_prefetch_item(i, 0, 0, w["L_img"], ld_rows.data_ptr(), h_ld_rows.ctypes.data,
                                    ld_dst[i * L].data_ptr(), Wl * 2) for i in range(B)]
    ld_stream = torch.cuda.Stream(device=device, priority=LOAD_PRIORITY)
    kind = w.get("block", "seq")
    kind = "double" if kind == "flux" else kind         # FLOPs per row: double == seq == par
    Lc = SDXL_CTX[0] if kind == "sdxl" else 0
    ctx_kv = (torch.randn(B * Lc, 2 * H, device=device).to(torch.bfloat16) if Lc else None)
    for m in (0.05, 0.2, 0.4, 0.7, 1.0):
        n_img = synth.n_masked_for(m, w["L_img"])
        n = n_img + w["L_txt"]
        q_row = torch.cat([torch.arange(n, device=device, dtype=torch.int32) + i * L for i in range(B)])
        ids = np.concatenate([np.arange(n_img), np.arange(w["L_img"], L)])
        b = F.VarlenBatch([n] * B, [L] * B, q_row=q_row, mode=F.FPS_MODE_KV,
                          ctx_kv=ctx_kv, n_ctx=[Lc] * B, act_ids=[ids] * B, L_img=w["L_img"])
        x = torch.randn(B * n, H, device=device).to(torch.bfloat16)
        ws = F.workspace(H, Fd, F.FPS_BF16, B * n, 0, device)
        y = torch.empty_like(x)
        # consecutive blocks with their own weights, as in the stack (weights stream from HBM,
        # 226 MB per Flux block > L2), after enough work for the clocks to settle at the
        # power-capped level the step runs at
        nl = min(8, len(layers) - first)
        def fn():
            for i in range(first, first + nl):
                F.masked_block_forward(layers[i], b, x, kv, y_act=y, ws=ws)
        # (a 1.5 s clock-settling burst before the fits made the predicted step match the
        # measured one within 1% but moved the plan to 45-46 cached blocks, measured slower than
        # the 41-44 this fit picks: tools/sweep_plan.py, C3 k = 41..44 within noise at ~32.5 ms)
        settle = float(os.environ.get("FPS_CALIB_SETTLE", 0.5))
        t_end = time.perf_counter() + settle
        while time.perf_counter() < t_end:
            fn()
            torch.cuda.synchronize()
        fn()
        torch.cuda.synchronize()
        if LOADED_CALIBRATION:
            for _ in range(12):                            # > 5 blocks' worth of loads in flight
                cache.prefetch(ld_items, ld_stream)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(3):
            fn()
        e1.record(s)
        torch.cuda.synchronize()
        xs.append(B * sched.block_flops("kv", n, L, H, Fd, kind, Lc))
        ys.append(e0.elapsed_time(e1) / (3 * nl))
    a, bb, r2c = sched.fit_linear(xs, ys)
    # loads: rows of one layer for the batch at several unmasked counts
    W = (2 if mode == "kv" else 1) * H
    dst = torch.empty(B * L, W, dtype=torch.bfloat16, device=device)
    ls = torch.cuda.Stream(device=device, priority=LOAD_PRIORITY)
    whole = cache.desc.copy_method == 2
    for k, m in enumerate((0.05, 0.3, 0.6, 0.9)):
        u = w["L_img"] - synth.n_masked_for(m, w["L_img"])
        # unmasked rows with the run structure of a blob mask: the masked rows form chunks of
        # ~28 consecutive tokens spread over the grid (one per image row the blob crosses)
        nm = w["L_img"] - u
        keep = np.ones(w["L_img"], bool)
        n_chunks = max(1, nm // 28)
        starts = np.linspace(0, w["L_img"] - 28, n_chunks).astype(int)
        for c0 in starts:
            keep[c0:c0 + 28] = False
        drop = np.flatnonzero(keep)[:max(0, keep.sum() - u)]   # exact count u
        keep[drop] = False
        h_rows = np.flatnonzero(keep).astype(np.int32)
        u = len(h_rows)
        rows = torch.as_tensor(h_rows, device=device)
        items = [F.fps_prefetch_item(i, 0, 0, u, rows.data_ptr(), h_rows.ctypes.data,
                                     dst[i * L].data_ptr(), W * 2) for i in range(B)]
        if whole:                 # whole-entry DMA: bytes do not depend on u; vary the count
            items = items * (k + 1)
            u = w["L_img"] * (k + 1)
        for _ in range(2):
            cache.prefetch(items, ls)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(ls)
        for _ in range(4):
            cache.prefetch(items, ls)
        e1.record(ls)
        torch.cuda.synchronize()
        bx.append(B * u * W * 2)
        by.append(e0.elapsed_time(e1) / 4)
    c, e, r2l = sched.fit_linear(bx, by)
    # a whole-entry DMA (copy_method 2) moves the same bytes whatever the mask: its load time is
    # flat in the row count, the fitted slope ~0 (or slightly negative by noise) -> clamp at 0
    cm = sched.CostModel(w["layers"], H, Fd, mode, comp=(max(a, 1e-16), max(bb, 1e-4)),
                         load=(max(c, 0.0), max(e, 1e-4)),
                         full_entry_rows=w["L_img"] if whole else None, kind=kind, Lc=Lc)
    info = {"comp_ms_per_tflop": a * 1e12, "comp_b_ms": bb, "comp_r2": r2c,
            "load_gbs": 1.0 / (c * 1e6) if c > 0 else None, "load_e_ms": e, "load_r2": r2l}
    return cm, info


def run_engine_timed(F, eng, reqs_dev, K, W, stream, load_stream, rank, world, ranged=False):
    """W warm-up steps, then exactly K timed steps bracketed by barrier + synchronize.
    ranged: bracket the K steps with cudaProfilerStart / Stop when FPS_PROFILE_RANGE is set
    (ncu --profile-from-start off then records exactly the timed region's launches)."""
    import torch.distributed as dist
    for r in reqs_dev:
        r["step"], r["status"] = 0, 0
    if W:
        eng.run_batch(reqs_dev, W, stream=stream, load_stream=load_stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    l0 = F.fps_launch_count()
    prof_range = ranged and os.environ.get("FPS_PROFILE_RANGE")
    if prof_range:
        torch.cuda.profiler.start()
    e0.record(stream)
    eng.run_batch(reqs_dev, K, stream=stream, load_stream=load_stream)
    e1.record(stream)
    torch.cuda.synchronize()
    if prof_range:
        torch.cuda.profiler.stop()
    launches = F.fps_launch_count() - l0
    ms = e0.elapsed_time(e1)
    if world > 1:
        ms = dist_max(ms)
        dist.barrier()
    return ms / K, launches


DIST_DEVICE = None   # device of the all-reduce tensors: the GPU (NCCL) or the CPU (gloo)


def dist_max(v):
    """Max over ranks of a host float (device-timed values are reduced, never wall clock)."""
    import torch.distributed as dist
    t = torch.tensor([float(v)], dtype=torch.float64, device=DIST_DEVICE)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def oracle_block_sample(w, mode, ratio, seed=7, kind=None):
    """CPU oracle: one mask-aware block for one request of the workload (fp64 numpy, all host
    cores).  Returns (seconds, the block's algorithmic FLOPs)."""
    from paper_conf_eurosys_jianglyfdlzllyl26_b200.sched import block_flops
    from oracle import block as OB
    from oracle.index import build_mask_index
    g = synth.rng(seed)
    H, Fd, L_img, L_txt = w["H"], w["F"], w["L_img"], w["L_txt"]
    L = L_img + L_txt
    if kind is None:
        kind = w.get("block", "seq")
        kind = "double" if kind == "flux" else kind
    wt = synth.block_weights(g, H, Fd, "bf16", kind, D_ctx=SDXL_CTX[1])
    ctx = synth.context(g, *SDXL_CTX, "bf16") if kind == "sdxl" else None
    mask = synth.token_mask(synth.mask_blobs(g, *w["grid"], ratio), L_txt)
    M, U = build_mask_index(mask)
    x = synth.latent(g, L, H, "bf16")
    K, V = synth.latent(g, L, H, "bf16"), synth.latent(g, L, H, "bf16")
    mod = synth.mod_table(g, 1, 1, H, "bf16", streams=2 if kind == "double" else 1)[0, 0]
    t0 = time.perf_counter()
    if mode == "kv":
        OB.masked_block_kv(x[M], M, U, K[U], V[U], wt, mod, w["heads"], L, ctx, L_txt)
    else:
        OB.masked_block_y(x[M], M, U, x[U], wt, mod, w["heads"], L, ctx, L_txt)
    t = time.perf_counter() - t0
    Lc = SDXL_CTX[0] if kind == "sdxl" else 0
    return t, block_flops(mode, len(M), L, H, Fd, "sdxl" if kind == "sdxl" else "seq", Lc)


def cpu_threads():
    try:
        from threadpoolctl import threadpool_info
        n = [i.get("num_threads") for i in threadpool_info() if i.get("user_api") == "blas"]
        if n:
            return int(n[0])
    except Exception:
        pass
    return os.cpu_count()


# ---------------------------------------------------------------------------------------
def resolve_defaults(args):
    """Per-config defaults of the cache mode and the H2D path (flags the user gave win).
    Mode: KV for C3 (configs[2] names cached KV), Y -- the paper's default (L157) -- for the
    configs that name none (C2A / C2B / C4; measured faster there, profiles/r02/c2_y, c4_mode).
    H2D: whole-entry DMA (measured on B200, C3, profiles/r01f5_*: 34.6 ms/step vs 36.2 with one
    DMA per unmasked row run and 48.5 with the SM row gather; HBM tier 21.2), except KV-mode at
    C4 on the host tier: the TMA row gather on 8 SMs (WORKLOADS["C4"]).  Load-stream priority:
    highest with the row gather, else the compute stream's."""
    wl = WORKLOADS[args.config]
    if args.mode is None:
        args.mode = wl.get("mode", "kv")
    if args.copy_method is None:
        args.copy_method = 2
        if args.mode == "kv" and args.tier != "hbm" and "kv_copy_method" in wl:
            args.copy_method = wl["kv_copy_method"]
            if args.copy_ctas == 0:
                args.copy_ctas = wl.get("kv_copy_ctas", 0)
    if args.load_priority is None:
        args.load_priority = -5 if args.copy_method == 3 else 0
    return args


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C3", choices=list(WORKLOADS))
    ap.add_argument("--mode", default=None, choices=["kv", "y"],
                    help="cache mode: K|V of the unmasked rows (KV-mode, L161) or the block "
                         "outputs Y (Y-mode, the paper's default, L157). Default: kv for C3 / C4 "
                         "(configs[2] names cached KV), y for the SDXL-scale levels C2A / C2B")
    ap.add_argument("--block", default=None, choices=["seq", "par", "sdxl", "flux"],
                    help="block kind: sequential attention -> MLP, the parallel (Flux "
                         "single-stream) block with fused input / output projections, or the SDXL "
                         "block with cross-attention and GEGLU, or Flux's stack of 19 double-stream "
                         "then 38 single-stream blocks (NEXT-2); default: sdxl for the "
                         "SDXL-scale configs (C2A/C2B), flux for the Flux-scale ones (C3/C4)")
    ap.add_argument("--tier", default=None, choices=["host", "hbm", "host_hugepage", "host_shared"],
                    help="template cache in pinned host DRAM (configs[2]), HBM (NEXT-1), on 2 MiB "
                         "pages, or one pinned arena shared by all ranks of the box (default "
                         "host at 1 GPU, host_shared with more ranks)")
    ap.add_argument("--sampler", default="euler", choices=["euler", "flow"],
                    help="update after the stack: the synthetic Euler step (R21) or the "
                         "flow-matching Euler step with inpainting blend (R29)")
    ap.add_argument("--copy-ctas", type=int, default=0, help="CTAs of the SM row gather (0 = lib default)")
    ap.add_argument("--copy-method", type=int, default=None, choices=[0, 1, 2, 3],
                    help="H2D method: 0 SM zero-copy row gather, 1 one DMA per unmasked row run, "
                         "2 whole-entry DMA, 3 TMA bulk row gather on reserved SMs")
    ap.add_argument("--load-priority", type=int, default=None,
                    help="CUDA priority of the cache-load stream (lower = higher; 0 = the compute "
                         "stream's). Default: highest (-5) with the TMA row gather (method 3), whose "
                         "CTAs then take the reserved SMs ahead of queued compute CTAs (C4: 525 "
                         "vs 548 ms/step), else 0")
    ap.add_argument("--cross-step", type=int, default=1, choices=[0, 1],
                    help="cross-step prefetch (R26): the next step's loads start as soon as their "
                         "slots are consumed (1, default), or the per-step pipeline of Fig. 9 (0)")
    ap.add_argument("--admission-reuse", type=int, default=1, choices=[0, 1],
                    help="fps_run_batch reuses the previous call's admission when the batch is "
                         "unchanged (1, default) or re-admits every call (0)")
    ap.add_argument("--kv-transition", type=int, default=1, choices=[0, 1],
                    help="KV-mode: run the last dense block before the cached suffix as a masked "
                         "block over the fresh full input (R28; 0 = dense, for A/B)")
    ap.add_argument("--plan-refine", type=int, default=1, choices=[0, 1],
                    help="refine Alg. 1's plan by measuring it and its +-2-block neighbours "
                         "(1, default) or time the planner's plan as is (0)")
    ap.add_argument("--no-extras", action="store_true", help="skip dense / Y-mode / profile legs")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        # one process per GPU: start the N ranks ourselves (the driver's own launch sets
        # WORLD_SIZE and lands in the branch below)
        import socket
        with socket.socket() as so:
            so.bind(("127.0.0.1", 0))
            port = so.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
               f"--nproc-per-node={args.gpus}", "--master-addr", "127.0.0.1",
               "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
        log(f"launching {args.gpus} ranks: {' '.join(cmd)}")
        sys.exit(subprocess.call(cmd))
    if int(os.environ.get("WORLD_SIZE", 1)) != args.gpus:
        log(f"--gpus {args.gpus} but WORLD_SIZE={os.environ.get('WORLD_SIZE', 1)}: refusing to "
            f"report a {os.environ.get('WORLD_SIZE', 1)}-rank run as {args.gpus} GPUs")
        sys.exit(2)
    import faulthandler                   # a stuck run dumps every thread's stack and exits
    import signal
    faulthandler.dump_traceback_later(int(os.environ.get("FPS_BENCH_TIMEOUT", 900)), exit=True)
    faulthandler.register(signal.SIGUSR1, all_threads=True)   # `timeout -s USR1`: dump stacks
    global LOAD_PRIORITY
    cm_given = args.copy_method is not None
    resolve_defaults(args)
    LOAD_PRIORITY = args.load_priority

    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if args.tier is None:
        args.tier = "host_shared" if world > 1 else "host"
    if args.block is None:       # the evaluated models' own block structure (R24, R25)
        args.block = "sdxl" if args.config.startswith("C2") else "flux"
    w = dict(WORKLOADS[args.config], block=args.block)
    K, W = args.steps, max(args.warmup, 0)
    # images/s counts the schedule's denoising steps (S_IMG); a run longer than one schedule
    # (W + K > S_IMG) just gives the requests, cache and modulation table more steps
    S_IMG = w["steps"]
    w["steps"] = max(S_IMG, W + K)
    L = w["L_img"] + w["L_txt"]
    metric_unit = "images/s"
    base_cfg = {"workload": args.config, "desc": w["desc"], "H": w["H"], "heads": w["heads"],
                "head_dim": w["H"] // w["heads"], "mlp": w["F"], "tokens": L,
                "image_tokens": w["L_img"], "text_tokens": w["L_txt"], "blocks": w["layers"],
                "denoise_steps": S_IMG, "cache_mode": args.mode,
                "batch_per_gpu": w["batch"], "block": args.block,
                "l2": f"inputs > L2 ({weight_bytes(w) / 1e9:.1f} GB of weights streamed per step)",
                "sampler": {"euler": "synthetic Euler (R21)",
                            "flow": "flow-matching Euler + inpainting blend (R29)"}[args.sampler]}

    metric_name = ("masked-block stack images/s (Flux-scale, 20% mask) [ms/step alongside]"
                   if args.config == "C3" else f"masked-block stack images/s ({args.config})")
    base_cfg["cache_tier"] = TIER_NAMES[args.tier]
    base_cfg["h2d_method"] = H2D_NAMES[args.copy_method]
    if args.copy_method == 3:
        base_cfg["h2d_reserved_sms"] = args.copy_ctas or 4
    if args.load_priority:
        base_cfg["load_stream_priority"] = args.load_priority
    base_cfg["parallelism"] = f"request-parallel x{world} (Alg. 2 routing)"
    base_cfg["cross_step_prefetch"] = bool(args.cross_step)
    base_cfg["kv_transition_block"] = bool(args.kv_transition) and args.mode == "kv"

    if args.impl == "reference":
        if rank != 0:
            return
        # the same config keys as our arm's line (one GPU: the whole pool is this rank's)
        ref_pool = make_requests(w, w["batch"], SEED)
        base_cfg.update(mask_ratios=sorted({p["ratio"] for p in ref_pool}),
                        mean_active_rows=statistics.mean(p["n_active"] for p in ref_pool))
        # the oracle as it stands, one block of one request per step; extrapolated to the step
        times = []
        for i in range(W + K):
            t, _ = oracle_block_sample(w, args.mode, float(w["ratios"][0]), seed=11 + i)
            if i >= W:
                times.append(t)
        block_s = statistics.mean(times)
        step_ms = block_s * 1e3 * w["layers"] * w["batch"]
        ips = w["batch"] / (step_ms * 1e-3 * S_IMG)
        cpu = {"value": ips, "unit": metric_unit, "cores": cpu_threads(), "kind": "oracle",
               "sample": f"1 mask-aware block x 1 request per step (fp64 numpy), extrapolated x"
                         f"{w['layers']} blocks x{w['batch']} requests x{S_IMG} steps"}
        print(json.dumps({"impl": "reference", "metric": metric_name,
                          "value": ips, "unit": metric_unit, "n_gpus": world, "steps": K,
                          "warmup": W, "ms_per_step": step_ms, "higher_is_better": True,
                          "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                          "data": "synthetic", "config": base_cfg, "cpu_baseline": cpu,
                          "e2e": {"value": ips, "unit": metric_unit, "h2d_bytes_per_step": 0,
                                  "d2h_bytes_per_step": 0}}), flush=True)
        return

    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    F.require_gpu()
    # one process per GPU; only on a box with fewer GPUs than ranks (a functional check of the
    # multi-rank path on one GPU) do ranks share devices, with gloo for the two host reductions
    n_dev = torch.cuda.device_count()
    torch.cuda.set_device(local % n_dev)
    device = torch.device("cuda", local % n_dev)
    if os.environ.get("FPS_KERNEL_FLAGS"):            # experiments: force kernel variants
        F.fps_set_disable_tc(int(os.environ["FPS_KERNEL_FLAGS"]))
    if world > 1:
        import torch.distributed as dist
        global DIST_DEVICE
        if n_dev >= world:
            dist.init_process_group("nccl", device_id=device)
            DIST_DEVICE = device
        else:
            dist.init_process_group("gloo")
            DIST_DEVICE = torch.device("cpu")
            log(f"[rank {rank}] {world} ranks on {n_dev} GPU(s): shared devices, gloo reductions")
            # processes time-sharing one GPU: launch without programmatic dependent launch (two
            # such runs hung a rank's step -- device work never completed -- out of eight)
            F.fps_set_disable_tc(int(os.environ.get("FPS_KERNEL_FLAGS", 0)) | 64)

    # requests of the whole job, routed to GPUs by Alg. 2 (identical on every rank: no comms)
    pool = make_requests(w, w["batch"] * world, SEED)
    t0 = time.perf_counter()
    n_entries = 2 * (w["layers"] + 1)
    location = {"host": 0, "hbm": 1, "host_hugepage": 2, "host_shared": 3}[args.tier]
    global COPY_CTAS, SHM_PATH
    COPY_CTAS = args.copy_ctas
    shm_fd = None
    if location == 3:
        # one pinned arena for every rank of the box: rank 0 makes a memfd, the others map it
        # through /proc (setup only; host control, not the data path)
        if rank == 0:
            shm_fd = os.memfd_create("flashps_arena")
            SHM_PATH = f"/proc/{os.getpid()}/fd/{shm_fd}"
        if world > 1:
            import torch.distributed as dist
            obj = [SHM_PATH]
            dist.broadcast_object_list(obj, src=0)
            SHM_PATH = obj[0]
    layers, mod, cache = build_engine_inputs(F, w, args.mode, device, n_entries, location,
                                             args.copy_method)
    wbytes = sum(t.numel() * t.element_size() for l in layers for t in l.t.values())
    assert abs(wbytes - weight_bytes(w)) < 1e6, (wbytes, weight_bytes(w))
    torch.cuda.synchronize()
    log(f"[rank {rank}] inputs ready in {time.perf_counter() - t0:.1f}s")
    my_pool = pool[:w["batch"]]
    log(f"[rank {rank}] calibrating")
    if world > 1 and n_dev < world:
        # ranks sharing a device (the functional check of the multi-rank path on one GPU):
        # calibrate one rank at a time so the fits do not time each other's kernels
        import torch.distributed as dist
        for r in range(world):
            if r == rank:
                cm, fit = calibrate(F, w, args.mode, layers, cache, [dict()] * w["batch"], device)
            dist.barrier()
    else:
        cm, fit = calibrate(F, w, args.mode, layers, cache, [dict()] * w["batch"], device)
    log(f"[rank {rank}] fit {fit}")
    if world > 1:
        # every rank routes the same pool with Alg. 2; the cost models must be identical for the
        # assignments to agree, so all ranks use rank 0's fit (setup only, not on the data path)
        import torch.distributed as dist
        obj = [(cm.comp, cm.load, cm.layer_comp, fit)]
        dist.broadcast_object_list(obj, src=0)
        cm.comp, cm.load, cm.layer_comp, fit = obj[0]
    my_ids, assign, held = route_job(pool, w, world, rank, cm)
    mine = [pool[i] for i in my_ids]
    g = torch.Generator(device=device).manual_seed(SEED + rank)
    reqs_dev = []
    L_ctx = SDXL_CTX[0] if args.block == "sdxl" else 0
    MODW = 12 * w["H"] if args.block == "flux" else 0
    for i, p in enumerate(mine):
        reqs_dev.append(dict(template_id=i, step=0, n_steps=w["steps"],
                             mask=torch.as_tensor(p["mask_np"]).to(device),
                             x=torch.randn(L, w["H"], generator=g, device=device).to(torch.bfloat16)))
        if L_ctx:
            reqs_dev[-1]["ctx"] = torch.randn(*SDXL_CTX, generator=g, device=device).to(torch.bfloat16)
        if args.sampler == "flow":     # the request's template latent and noise (R29)
            reqs_dev[-1]["z"] = torch.randn(w["L_img"], w["H"], generator=g, device=device).to(torch.bfloat16)
            reqs_dev[-1]["noise"] = torch.randn(w["L_img"], w["H"], generator=g, device=device).to(torch.bfloat16)
    stream = torch.cuda.current_stream()
    load_stream = torch.cuda.Stream(device=device, priority=LOAD_PRIORITY)
    deltas = synth.delta_table(w["steps"])

    sigmas = None
    if args.sampler == "flow":
        from oracle.sampler import FLUX_SHIFT      # a constant, not the oracle's arithmetic
        t = 1.0 - np.arange(w["steps"]) / w["steps"]
        sigmas = list(FLUX_SHIFT * t / (1.0 + (FLUX_SHIFT - 1.0) * t)) + [0.0]

    def engine(policy, mode=args.mode, the_cache=cache, plan=None, model=None):
        model = model or cm
        e = F.Engine(layers, w["heads"], F.MODE_CODE[mode], F.FPS_BF16, w["L_img"], w["L_txt"],
                     max(len(reqs_dev), 1), w["steps"], deltas, the_cache, mod_table=mod,
                     slots=0, plan_policy=policy, plan=plan, cost_model=model.as_engine_model(),
                     L_ctx=L_ctx, mod_width=MODW, cross_step=bool(args.cross_step),
                     sampler=1 if args.sampler == "flow" else 0, sigmas=sigmas,
                     layer_comp=model.layer_comp)
        F.fps_engine_set_kv_transition(e.h, args.kv_transition)
        return e

    eng = engine(0)
    refine = None
    if args.plan_refine:
        # Alg. 1 picks the plan from the fitted latency models; the models' few-percent error
        # moves the link / compute balance point by a block or two, so the choice is refined
        # by measurement: the planner's suffix plan and its neighbours (k - 2 .. k + 2 cached
        # blocks, extended while the best sits at an edge and keeps improving), a few steps
        # each on this GPU, the fastest kept (an online correction of the planner, made before
        # the timed region; every rank does the same on its own batch)
        run_engine_timed(F, eng, reqs_dev, 1, 1, stream, load_stream, rank, world)
        p0, pred0 = eng.last_plan()
        N = len(p0)
        suffix = all(p0[i] <= p0[i + 1] for i in range(N - 1))
        if suffix:
            k0 = int(sum(p0))
            refine = {"planner_cached_blocks": k0, "planner_predicted_ms": pred0, "measured_ms": {}}
            def measure(k):
                e_k = engine(3, plan=[0] * (N - k) + [1] * k)
                ms_k, _ = run_engine_timed(F, e_k, reqs_dev, 4, 2, stream, load_stream, rank, world)
                refine["measured_ms"][k] = ms_k
                del e_k
                return ms_k
            for k in range(max(0, k0 - 2), min(N, k0 + 2) + 1):
                measure(k)
            # the best at an edge of the window: keep walking that way while it improves
            while True:
                kb = min(refine["measured_ms"], key=refine["measured_ms"].get)
                lo, hi = min(refine["measured_ms"]), max(refine["measured_ms"])
                nxt = kb - 1 if (kb == lo and lo > 0) else kb + 1 if (kb == hi and hi < N) else None
                if nxt is None or len(refine["measured_ms"]) >= 12:
                    break
                if measure(nxt) >= refine["measured_ms"][kb]:
                    break
            kb = min(refine["measured_ms"], key=refine["measured_ms"].get)
            best = (refine["measured_ms"][kb], kb)
            if best[1] != k0:
                del eng
                eng = engine(3, plan=[0] * (N - best[1]) + [1] * best[1])
            refine["chosen_cached_blocks"] = best[1]
            log(f"[rank {rank}] plan refinement {refine}")
    F.fps_engine_set_admission_reuse(eng.h, args.admission_reuse)
    log(f"[rank {rank}] timed run")
    with Clocks(local % n_dev) as clk:
        step_ms, launches = run_engine_timed(F, eng, reqs_dev, K, W, stream, load_stream, rank, world,
                                             ranged=True)
    plan, pred_ms = eng.last_plan()
    imgs = sum(len(a) for a in assign)
    value = imgs / (step_ms * 1e-3 * S_IMG)

    extras = {}
    if not args.no_extras:
        log(f"[rank {rank}] extras")
        # same batch, every block dense (all tokens, no cache): the compute-saving reference
        log(f"[rank {rank}] extras: dense")
        eng_d = engine(2)
        dense_ms, _ = run_engine_timed(F, eng_d, reqs_dev, K, W, stream, load_stream, rank, world)
        del eng_d
        # all blocks cached (no planner) and the HBM-resident "ideal" (no loads at all)
        log(f"[rank {rank}] extras: all cached")
        eng_c = engine(1)
        cached_ms, _ = run_engine_timed(F, eng_c, reqs_dev, K, W, stream, load_stream, rank, world)
        del eng_c
        extras.update(dense_ms_per_step=dense_ms, all_cached_ms_per_step=cached_ms)
        # the same plan, same engine and cache, with the loads switched off
        # (fps_engine_set_skip_loads: ready events still recorded, no bytes moved; the staging
        # slots keep an earlier step's rows): the step without host-link load. Exposed load =
        # this step - that step, signed
        log(f"[rank {rank}] extras: same plan, loads skipped")
        eng_n = engine(3, plan=list(plan))
        F.fps_engine_set_skip_loads(eng_n.h, 1)
        noload_ms, _ = run_engine_timed(F, eng_n, reqs_dev, K, W, stream, load_stream, rank, world)
        del eng_n
        extras["same_plan_no_load_ms_per_step"] = noload_ms
        extras["exposed_load_ms_per_step"] = step_ms - noload_ms
        # the other caching mode, and both modes with the other cache tier, on the same batch
        other = "y" if args.mode == "kv" else "kv"
        other_loc = 0 if location == 1 else 1
        wl = WORKLOADS[args.config]

        def default_cm(md, loc):     # the bench's default H2D method of a mode on a tier
            return wl.get("kv_copy_method", 2) if (md == "kv" and loc != 1) else 2
        other_cm = default_cm(other, other_loc)
        for md, loc, cmeth in ((other, location, args.copy_method if cm_given
                                else default_cm(other, location)),
                               (args.mode, other_loc, default_cm(args.mode, other_loc)),
                               (other, other_loc, other_cm),
                               (args.mode, location, 2 if args.copy_method != 2 else 1)):
            if loc == 1 and cmeth == 1:
                continue
            loc = 0 if loc == 3 else loc        # the shared arena file belongs to `cache`
            log(f"[rank {rank}] extras: mode {md} location {loc} copy method {cmeth}")
            ctas_saved = COPY_CTAS
            ls_o = load_stream
            if cmeth == 3 and not cm_given:   # that mode's default gather setting (C4 KV-mode)
                COPY_CTAS = wl.get("kv_copy_ctas", 0)
                ls_o = torch.cuda.Stream(device=device, priority=-5)
            c2 = make_cache(F, w, md, n_entries, loc, cmeth)
            COPY_CTAS = ctas_saved
            cm2, _ = calibrate(F, w, md, layers, c2, [dict()] * w["batch"], device)
            eng_o = engine(0, mode=md, the_cache=c2, model=cm2)
            o_ms, _ = run_engine_timed(F, eng_o, reqs_dev, K, W, stream, ls_o, rank, world)
            tag = f"{md}_mode_{['host', 'hbm', 'host_hugepage', 'host_shared'][loc]}"
            if cmeth != default_cm(md, loc):
                tag += "_" + ["row_gather", "run_dma", "whole_entry_dma", "tma_row_gather"][cmeth]
            extras[f"{tag}_ms_per_step"] = o_ms
            extras[f"{tag}_cached_blocks"] = int(sum(eng_o.last_plan()[0]))
            del eng_o
            c2.close()

    # per-kernel-class device time over the same timed region (CUDA events on each kernel's
    # own stream), for the roofline of the dominant kernel
    log(f"[rank {rank}] profile pass")
    F.fps_profile_enable(1)
    run_engine_timed(F, eng, reqs_dev, K, W, stream, load_stream, rank, world)
    ms = (torch.zeros(7, dtype=torch.float64)).numpy()
    fl, by = ms.copy(), ms.copy()
    cnt = np.zeros(7, dtype=np.int64)
    import ctypes as C
    P = C.POINTER(C.c_double)
    F.fps_profile_read(ms.ctypes.data_as(P), fl.ctypes.data_as(P), by.ctypes.data_as(P),
                       cnt.ctypes.data_as(C.POINTER(C.c_int64)))
    names = ["gemm_tcgen05", "attention", "rownorm", "row_copy", "cache_prefetch", "sampler", "mask_index"]
    # launch timeline of the same pass: the compute stream's and the load stream's classes
    # separately (the load stream overlaps the compute stream, so only the compute stream's
    # classes add up to the step)
    nmax = 400000
    st_, en_ = np.zeros(nmax), np.zeros(nmax)
    kd_, sid_ = np.zeros(nmax, np.int32), np.zeros(nmax, np.int64)
    ntr = F.fps_profile_trace(st_.ctypes.data_as(P), en_.ctypes.data_as(P),
                              kd_.ctypes.data_as(C.POINTER(C.c_int32)),
                              sid_.ctypes.data_as(C.POINTER(C.c_int64)), nmax)
    F.fps_profile_enable(0)
    comp_sid = stream.cuda_stream
    on_comp = sid_[:ntr] == comp_sid
    dur = en_[:ntr] - st_[:ntr]
    stream_split = {
        "compute_stream_ms_per_step": float(dur[on_comp].sum()) / (W + K),
        "load_stream_ms_per_step": float(dur[~on_comp].sum()) / (W + K),
        "compute_stream_by_class": {names[k]: float(dur[on_comp & (kd_[:ntr] == k)].sum()) / (W + K)
                                    for k in range(7) if (on_comp & (kd_[:ntr] == k)).any()},
        "note": "CUDA events around every library launch on its own stream (the events break "
                "PDL overlap, so the profiled step runs a little longer than the timed one); "
                "per-class times of the undisturbed step come from the ncu launch list "
                "(kernels_ncu)"}
    # the profiled pass covers warm-up + timed steps; report per step of the timed region share
    per = {names[k]: {"ms_per_step": ms[k] / (W + K), "launches_per_step": cnt[k] / (W + K),
                      "tflops": (fl[k] / (ms[k] * 1e-3) / 1e12) if ms[k] > 0 and fl[k] > 0 else None,
                      "gbs": (by[k] / (ms[k] * 1e-3) / 1e9) if ms[k] > 0 and by[k] > 0 else None}
           for k in range(7)}
    hbm, bf16_burst, bf16_sust, src = peaks()
    gemm_avg_ms = ms[0] / max(cnt[0], 1)
    gemm_achieved = fl[0] / (ms[0] * 1e-3) / 1e12 if ms[0] > 0 else 0.0
    roofline = {"bound": "tensor", "kernel": "gemm_tcgen05 (a5/a7/a8 projections + MLP)",
                "achieved": gemm_achieved, "peak": bf16_sust, "unit": "TFLOP/s",
                "frac": gemm_achieved / bf16_sust, "peak_source": f"{src} bf16_tflops_sustained",
                "traffic": None, "traffic_source": None,
                "algorithmic_bytes_per_launch": by[0] / max(cnt[0], 1),
                "avg_launch_ms": gemm_avg_ms,
                "flops_per_launch": fl[0] / max(cnt[0], 1)}
    tr = ncu_summary(args.config, "traffic")
    if tr and "gemm_tcgen05" in tr:
        roofline["traffic"] = tr["gemm_tcgen05"]["dram_bytes_per_launch"]
        roofline["traffic_source"] = tr["source"]
    # step roofline for the chosen plan: the slower of the tensor work at the sustained peak,
    # the exact unmasked rows over the host link at its measured rate, and one pass of the
    # weights over HBM
    step_flops = (fl[0] + fl[1]) / (W + K)
    n_cached = int(sum(plan))
    Wl = (2 if args.mode == "kv" else 1) * w["H"] * 2
    u_rows = sum(w["L_img"] - (p["n_active"] - w["L_txt"]) for p in mine)   # unmasked rows U
    exact_bytes = n_cached * u_rows * Wl + ((u_rows * w["H"] * 2) if (args.mode == "kv" and n_cached) else 0)
    # the link's rate: the probe of a pinned torch buffer, or the load rate fitted on the arena
    # itself (whole-entry DMA, or the row gather's useful bytes) when higher -- the probe buffer
    # can land on the far NUMA node (27 vs 55 GB/s seen), and a measured rate bounds the peak
    link_gbs = max(fit.get("link_gbs") or 0.0, fit.get("load_gbs") or 0.0) or None
    t_comp = step_flops / (bf16_sust * 1e12) * 1e3
    t_link = exact_bytes / (link_gbs * 1e9) * 1e3 if (location != 1 and link_gbs) else 0.0
    t_hbm = weight_bytes(w) / (hbm * 1e9) * 1e3
    ideal = max(t_comp, t_link, t_hbm)
    step_roofline = {"ideal_ms": ideal, "frac": ideal / step_ms, "compute_ms": t_comp,
                     "link_ms": t_link, "hbm_ms": t_hbm, "step_tflop": step_flops / 1e12,
                     "exact_row_link_bytes": exact_bytes, "link_gbs": link_gbs,
                     "link_source": "host-link rate measured in the calibration (max of a pinned-buffer "
                                    "copy-engine probe and the load rate fitted on the arena itself)",
                     "bound": ["tensor", "host link", "hbm"][[t_comp, t_link, t_hbm].index(ideal)]}

    log(f"[rank {rank}] e2e")
    # e2e through the public call with HOST buffers: per step H2D latents, one step, D2H latents
    host_x = [torch.empty(L, w["H"], dtype=torch.bfloat16).pin_memory() for _ in reqs_dev]
    for h, r in zip(host_x, reqs_dev):
        h.copy_(r["x"])
    for r in reqs_dev:
        r["step"] = 0
    eng.run_batch(reqs_dev, W, stream=stream, load_stream=load_stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(K):
        for h, r in zip(host_x, reqs_dev):
            r["x"].copy_(h, non_blocking=True)
        eng.run_batch(reqs_dev, 1, stream=stream, load_stream=load_stream)
        for h, r in zip(host_x, reqs_dev):
            h.copy_(r["x"], non_blocking=True)
    e1.record(stream)
    torch.cuda.synchronize()
    e2e_ms = e0.elapsed_time(e1) / K
    if world > 1:
        e2e_ms = dist_max(e2e_ms)
    bytes_io = len(reqs_dev) * L * w["H"] * 2
    e2e = {"value": imgs / (e2e_ms * 1e-3 * S_IMG), "unit": metric_unit,
           "ms_per_step": e2e_ms, "h2d_bytes_per_step": bytes_io, "d2h_bytes_per_step": bytes_io}

    if rank == 0:
        cpu = None
        if not args.no_cpu and world == 1:
            # the oracle's FLOP rate on one mask-aware block of each kind in the stack, then the
            # timed plan's FLOPs (dense prefix, transition block, cached suffix) at that rate
            kinds = ["double", "par"] if args.block == "flux" else [args.block]
            secs, flops = 0.0, 0.0
            for i, kd in enumerate(kinds):
                t, f = oracle_block_sample(w, args.mode, float(w["ratios"][0]), seed=11 + i, kind=kd)
                secs += t
                flops += f
            rate = flops / secs
            cpu_step_ms = step_flops / rate * 1e3
            cpu = {"value": imgs / (cpu_step_ms * 1e-3 * S_IMG), "unit": metric_unit,
                   "cores": cpu_threads(), "kind": "oracle",
                   "sample": f"{len(kinds)} mask-aware block(s) ({'/'.join(kinds)}) x 1 request, fp64 "
                             f"numpy, m={w['ratios'][0]}: {secs:.1f} s for {flops / 1e9:.0f} GFLOP; "
                             f"the timed plan's {step_flops / 1e12:.2f} TFLOP/step ({n_cached} cached "
                             f"of {len(plan)} blocks) priced at that rate, x{S_IMG} steps",
                   "oracle_gflops": rate / 1e9, "step_ms": cpu_step_ms}
        mean_n = statistics.mean(p["n_active"] for p in mine) if mine else 0
        out = {
            "metric": metric_name,
            "value": value, "unit": metric_unit, "n_gpus": world, "steps": K, "warmup": W,
            "ms_per_step": step_ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "bf16", "data": "synthetic (random-init weights, blob masks)",
            "config": dict(base_cfg, parallelism=f"request-parallel x{world} (Alg. 2 routing)",
                           mask_ratios=sorted({p["ratio"] for p in mine}), mean_active_rows=mean_n),
            "clocks": clk.summary(),
            "gpu_launches": int(launches),
            "e2e": e2e,
            "roofline": roofline,
            "cpu_baseline": cpu,
            "plan": {"cached_blocks": int(sum(plan)), "blocks": len(plan),
                     "predicted_ms_per_step": pred_ms, "fit": fit, "refinement": refine},
            "kernels": per,
            "kernels_stream_split": stream_split,
            "kernels_ncu": ncu_summary(args.config, "classes"),
            "step_roofline": step_roofline,
            "extras": extras,
        }
        if extras.get("dense_ms_per_step"):
            dms = extras["dense_ms_per_step"]
            out["extras"]["speedup_vs_dense"] = dms / step_ms
            out["extras"]["time_fraction_of_dense"] = step_ms / dms
            # north_star: saving >= 0.7 x the ideal saving dense * m (literal reading, image
            # tokens) and dense * n/L (text rows always active); report the achieved fraction
            m = float(w["ratios"][0]) if len(w["ratios"]) == 1 else None
            if m is not None:
                frac_active = (synth.n_masked_for(m, w["L_img"]) + w["L_txt"]) / L
                out["extras"]["saving_vs_ideal_literal"] = (dms - step_ms) / (dms * (1 - m))
                out["extras"]["saving_vs_ideal_active_rows"] = (dms - step_ms) / (dms * (1 - frac_active))
        if "exposed_load_ms_per_step" in extras:
            load_ms = stream_split["load_stream_ms_per_step"]
            ex = extras["exposed_load_ms_per_step"]
            out["extras"]["load_ms_per_step"] = load_ms
            # hidden share of the load time; a negative exposed time (the step with loads ran
            # faster than the one without, i.e. within run-to-run noise) is reported as is
            out["extras"]["load_overlap_frac"] = (1 - max(ex, 0.0) / load_ms) if load_ms > 0 else None
        print(json.dumps(out), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
