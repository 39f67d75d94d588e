"""§4.4 mask-aware scheduling on top of the library's Alg. 1 planner.

  * latency models (L255-L257): Comp(FLOPs) = a*FLOPs + b and Load(bytes) = c*bytes + e, fitted
    by least squares on measurements taken on this GPU (`calibrate`);
  * CalcCost (Alg. 2 lines 1-4): the Alg. 1 pipeline latency of worker.running_batch + request,
    computed by fps_plan_pipeline in libflashps;
  * route (Alg. 2 lines 5-11): the candidate worker with slack and the lowest cost wins; ties go
    to the worker with fewer requests, then the lower id (reading R15).
Host-side bookkeeping only; the data path never leaves the GPU worker that owns a request.
"""
from __future__ import annotations

import math

import numpy as np

from . import FPS_MODE_KV, FPS_MODE_Y, plan_pipeline


def block_flops(mode, n, L, H, F, kind="seq", Lc=0):
    """Exact FLOPs of one block for one request with n active of L rows (Table 1, per mode);
    the SDXL block (R24) adds cross-attention (4H^2 + 4 Lc H) and the GEGLU's 2HF per row."""
    rows = L if mode == "dense" else n
    extra = rows * (4.0 * H * H + 4.0 * Lc * H + 2.0 * H * F) if kind == "sdxl" else 0.0
    if mode == "dense":
        return 8.0 * L * H * H + 4.0 * L * H * F + 4.0 * L * L * H + extra
    attn = 4.0 * n * L * H
    if mode == "kv":
        return 8.0 * n * H * H + 4.0 * n * H * F + attn + extra
    return 4.0 * n * H * H + 4.0 * L * H * H + 4.0 * n * H * F + attn + extra


def cache_bytes(mode, u, H, elt=2):
    return (2.0 if mode == "kv" else 1.0) * u * H * elt


def fit_linear(x, y):
    """Least squares y ~ a x + b; returns (a, b, R^2) (L257 reports R^2)."""
    x = np.asarray(x, np.float64)
    y = np.asarray(y, np.float64)
    A = np.stack([x, np.ones_like(x)], 1)
    (a, b), *_ = np.linalg.lstsq(A, y, rcond=None)
    res = y - (a * x + b)
    tot = ((y - y.mean()) ** 2).sum()
    return float(a), float(b), float(1.0 - (res ** 2).sum() / tot) if tot > 0 else 1.0


class Request:
    """What the scheduler knows about a request: its active rows n and unmasked rows u."""

    def __init__(self, rid, n_active, L, arrival=0.0, steps=28, tokens=None, model="flux",
                 ratio=None):
        self.rid, self.n, self.L, self.arrival, self.steps = rid, int(n_active), int(L), arrival, steps
        # token-granularity load (§6.5): masked image tokens (defaults to the active rows)
        self.tokens = int(n_active if tokens is None else tokens)
        # which model's stack serves it, and its image-token mask ratio (multi-level models)
        self.model, self.ratio = model, ratio

    @property
    def u(self):
        return self.L - self.n


class CostModel:
    """Per-block costs of a batch for Alg. 1 from the two fitted linear models."""

    def __init__(self, n_layers, H, F, mode, comp=(1e-12, 0.01), load=(2e-8, 0.01), elt=2,
                 full_entry_rows=None, kind="seq", Lc=0, layer_comp=None):
        self.n_layers, self.H, self.F, self.mode, self.elt = n_layers, H, F, mode, elt
        self.kind, self.Lc = kind, Lc
        self.comp, self.load = comp, load
        # per-block compute models (a_l, b_l), e.g. fitted per block kind; None = comp for all
        self.layer_comp = layer_comp
        # whole-entry DMA loads (copy_method 2) move L_img rows whatever the mask
        self.full_entry_rows = full_entry_rows

    def _rows(self, r):
        return self.full_entry_rows if (self.full_entry_rows and r.u > 0) else r.u

    def costs(self, batch):
        a, b = self.comp
        c, e = self.load
        fm = sum(block_flops(self.mode, r.n, r.L, self.H, self.F, self.kind, self.Lc) for r in batch)
        fd = sum(block_flops("dense", r.n, r.L, self.H, self.F, self.kind, self.Lc) for r in batch)
        by = sum(cache_bytes(self.mode, self._rows(r), self.H, self.elt) for r in batch)
        byf = sum(cache_bytes("y", self._rows(r), self.H, self.elt) for r in batch)
        N = self.n_layers
        ab = self.layer_comp or [(a, b)] * N
        Cw = [al * fm + bl for al, bl in ab]
        Cwo = [al * fd + bl for al, bl in ab]
        Lm = [c * by + e if by > 0 else 0.0] * N
        fin = (c * byf + e) if (self.mode == "kv" and byf > 0) else 0.0
        return Cw, Cwo, Lm, fin

    def step_latency(self, batch):
        """dp(batch).pipeline_latency of Alg. 2 line 3 (library planner)."""
        if not batch:
            return 0.0
        Cw, Cwo, Lm, fin = self.costs(batch)
        mode = FPS_MODE_KV if self.mode == "kv" else FPS_MODE_Y
        return plan_pipeline(Cw, Cwo, Lm, mode, fin)[1]

    def as_engine_model(self):
        """(a, b, c, e) in the units fps_engine_desc.cost_model expects (ms/FLOP, ms, ms/B, ms)."""
        return (self.comp[0], self.comp[1], self.load[0], self.load[1])


class SdxlCost:
    """SDXL's transformer blocks sit at two UNet levels (reading R19): a
    request's step runs the 64 x 64 level's stack (640 channels) and the 32 x 32 level's (1280
    channels), each with the request's mask pooled to that level (fps_mask_to_tokens, R8).  The
    step latency is the sum of the two levels' Alg. 1 pipeline latencies under their own fitted
    models; a request's mask ratio sets its active rows at each level."""

    def __init__(self, level_models, level_tokens):
        self.levels = list(zip(level_models, level_tokens))

    def step_latency(self, batch):
        if not batch:
            return 0.0
        t = 0.0
        for cm, Lv in self.levels:
            t += cm.step_latency([Request(r.rid, max(1, round(r.ratio * Lv)), Lv) for r in batch])
        return t


class MixedCost:
    """A worker holding both models' stacks (Flux 12.9 GB + SDXL 2.4 GB of weights
    in 180 GB of HBM) runs each model's sub-batch of its running batch in turn every step; the
    step latency is their sum (configs[4]: mixed SDXL / Flux traffic)."""

    def __init__(self, models):
        self.models = models          # model name -> object with step_latency(batch)

    def step_latency(self, batch):
        by = {}
        for r in batch:
            by.setdefault(r.model, []).append(r)
        return sum(self.models[m].step_latency(b) for m, b in by.items())


def route(req, workers, cost_fn, max_batch):
    """Alg. 2 lines 6-11. workers: list of lists of assigned requests. Returns an index or None."""
    best, key = None, None
    for wid, assigned in enumerate(workers):
        if len(assigned) >= max_batch:
            continue
        k = (cost_fn(assigned + [req]), len(assigned), wid)
        if key is None or k < key:
            best, key = wid, k
    return best


def shard_requests(n_active, L, world, rank, cost_model, max_batch):
    """Request-parallel sharding for `world` GPU workers (§8(e)): every rank routes the same
    pool with Alg. 2 (deterministic, so no communication is needed) and keeps its share.
    Returns (indices of this rank's requests, the full assignment, held requests)."""
    reqs = [Request(i, n, L) for i, n in enumerate(n_active)]
    workers, held = assign_all(reqs, world, cost_model.step_latency, max_batch)
    return [r.rid for r in workers[rank]], [[r.rid for r in w] for w in workers], [r.rid for r in held]


def assign_all(reqs, n_workers, cost_fn, max_batch):
    """Route a pool of simultaneously arriving requests one by one (arrival order)."""
    workers = [[] for _ in range(n_workers)]
    held = []
    for r in reqs:
        w = route(r, workers, cost_fn, max_batch)
        if w is None:
            held.append(r)
        else:
            workers[w].append(r)
    return workers, held


def simulate_serving(reqs, n_workers, max_batch, step_latency, policy="mask_aware",
                     batching="continuous", interrupt_ms=0.0):
    """Cluster of `n_workers` step-level continuous-batching workers (Fig. 8 workflow, L191-L199;
    L237: join / leave at step boundaries) fed by a router (Alg. 2, or a baseline policy:
    "round_robin" = request-level, "least_requests" = fewest assigned requests, "least_tokens" =
    fewest masked tokens assigned, §6.5).  Worker batching (§4.3, §6.4, reading R27):
    "continuous" (FlashPS, pre/post-processing disaggregated), "strawman" (each join and leave
    costs `interrupt_ms` of the worker's main process before its next step), "static" (a batch
    forms only on an idle worker and runs until all its requests finish).

    reqs: Request objects with .arrival (ms) and .steps, sorted by arrival.
    step_latency(batch) -> ms of one denoising step of that batch (e.g. CostModel.step_latency,
    the Alg. 1 pipeline latency from latency models fitted on this GPU).
    Returns {rid: (arrival, finish)}; requests no worker can take are held FIFO (reading R15)."""
    import heapq
    workers = [[] for _ in range(n_workers)]
    running = [[] for _ in range(n_workers)]
    remaining, busy, held, out, ev = {}, [False] * n_workers, [], {}, []
    started = set()
    seq = 0
    for r in reqs:
        heapq.heappush(ev, (r.arrival, 1, seq, "arr", r))
        seq += 1
    rr = [0]

    def start_step(wid, now, finished=0):
        nonlocal seq
        cur = [r for r in running[wid] if remaining.get(r.rid, 0) > 0]
        # static batching admits nobody while its batch still runs
        running[wid] = cur if (batching == "static" and cur) else list(workers[wid])
        busy[wid] = bool(running[wid])
        if busy[wid]:
            joining = [r for r in running[wid] if r.rid not in started]
            started.update(r.rid for r in joining)
            pause = interrupt_ms * (len(joining) + finished) if batching == "strawman" else 0.0
            heapq.heappush(ev, (now + pause + step_latency(running[wid]), 0, seq, "step", wid))
            seq += 1

    def assign(r, now):
        free = [w for w in range(n_workers) if len(workers[w]) < max_batch]
        if policy == "mask_aware":
            wid = route(r, workers, step_latency, max_batch)
        elif not free:
            wid = None
        elif policy == "round_robin":
            wid = min(free, key=lambda w: (w - rr[0]) % n_workers)
            rr[0] = (wid + 1) % n_workers
        elif policy == "least_tokens":
            wid = min(free, key=lambda w: (sum(q.tokens for q in workers[w]), w))
        else:
            wid = min(free, key=lambda w: (len(workers[w]), w))
        if wid is None:
            held.append(r)
            return
        workers[wid].append(r)
        remaining[r.rid] = r.steps
        if not busy[wid]:
            start_step(wid, now)

    while ev:
        now, _, _, kind, obj = heapq.heappop(ev)
        if kind == "arr":
            assign(obj, now)
            continue
        wid = obj
        finished = 0
        for r in running[wid]:
            remaining[r.rid] -= 1
            if remaining[r.rid] == 0:
                workers[wid].remove(r)
                out[r.rid] = (r.arrival, now)
                finished += 1
        while held and len(workers[wid]) < max_batch:
            assign(held.pop(0), now)
        start_step(wid, now, finished)
    return out


def latency_stats(out):
    lat = sorted(f - a for a, f in out.values())
    if not lat:
        return {}
    pick = lambda q: lat[min(len(lat) - 1, int(math.ceil(q * len(lat))) - 1)]
    return {"mean_ms": sum(lat) / len(lat), "p50_ms": pick(0.5), "p95_ms": pick(0.95),
            "makespan_ms": max(f for _, f in out.values()) - min(a for a, _ in out.values())}
