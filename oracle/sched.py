"""§4.4: latency models, Alg. 2 routing and a discrete-event simulator
of step-level continuous batching across workers (oracle; test infrastructure only).

  * L255-L257: "linear regression models to estimate computation latency and cache loading
    latency"; "we compute FLOPs ... based on their mask ratios, which are mapped to inference
    latency by the regression models" -> Comp(FLOPs) = a*FLOPs + b, Load(bytes) = c*bytes + e
    fitted by ordinary least squares, R^2 reported (reading R14).
  * Alg. 2 (L263-L287): CalcCost(req, worker) = dp(worker.running_batch + req).pipeline_latency;
    candidates = workers with slack (batch < max_batch, L326); best = argmin cost; ties -> fewer
    assigned requests, then lowest worker id; no candidate -> FIFO hold (reading R15).
  * L237 (§4.3): requests join/leave the running batch only at denoising-step boundaries (R16).
"""
from __future__ import annotations

import heapq
import math

import numpy as np

from .counters import block_flops, cache_bytes
from .pipeline import plan_bruteforce, plan_suffix_scan, simulate


def fit_linear(x, y):
    """OLS fit y ~ a*x + b. Returns (a, b, r2)."""
    x = np.asarray(x, dtype=np.float64)
    y = np.asarray(y, dtype=np.float64)
    A = np.stack([x, np.ones_like(x)], axis=1)
    (a, b), *_ = np.linalg.lstsq(A, y, rcond=None)
    pred = a * x + b
    ss_res = float(((y - pred) ** 2).sum())
    ss_tot = float(((y - y.mean()) ** 2).sum())
    r2 = 1.0 - ss_res / ss_tot if ss_tot > 0 else 1.0
    return float(a), float(b), r2


class CostModel:
    """Per-block costs of a batch from the two linear models (L257).

    layers: list of (L, H, F) per block; comp=(a, b) ms per FLOP; load=(c, e) ms per byte.
    A request is described by its active-row count per distinct (L) level: n_of(req, L)."""

    def __init__(self, layers, comp, load, mode, elt=2):
        self.layers, self.comp, self.load, self.mode, self.elt = layers, comp, load, mode, elt

    def costs(self, batch):
        a, b = self.comp
        c, e = self.load
        Cw, Cwo, Lm = [], [], []
        for (L, H, F) in self.layers:
            fm = sum(block_flops(self.mode, r.n_active(L), L, H, F) for r in batch)
            fd = sum(block_flops("dense", L, L, H, F) for r in batch)
            by = sum(cache_bytes(self.mode, L - r.n_active(L), H, self.elt) for r in batch)
            Cw.append(a * fm + b)
            Cwo.append(a * fd + b)
            Lm.append(c * by + e if by > 0 else 0.0)
        final = 0.0
        if self.mode == "kv" and self.layers:
            L, H, _ = self.layers[-1]
            by = sum(cache_bytes("y", L - r.n_active(L), H, self.elt) for r in batch)
            final = c * by + e if by > 0 else 0.0
        return Cw, Cwo, Lm, final

    def step_latency(self, batch, exact=False):
        if not batch:
            return 0.0
        Cw, Cwo, Lm, final = self.costs(batch)
        if self.mode == "kv" or not exact:
            lat, _ = plan_suffix_scan(Cw, Cwo, Lm, self.mode, final)
        else:
            lat, _ = plan_bruteforce(Cw, Cwo, Lm, self.mode, final)
        return lat


class Req:
    def __init__(self, rid, arrival, ratio, steps, L_img, L_txt=0):
        self.rid, self.arrival, self.ratio, self.steps = rid, arrival, ratio, steps
        self.L_img, self.L_txt = L_img, L_txt

    def n_active(self, L):
        # exact-count masks (R18) at the level with L tokens (text rows only at the top level)
        if L == self.L_img + self.L_txt:
            return int(math.floor(self.ratio * self.L_img + 0.5)) + self.L_txt
        return int(math.floor(self.ratio * L + 0.5))


def route(req, workers, cost_fn, max_batch):
    """Alg. 2 lines 6-11: pick the candidate with the lowest CalcCost; None if none has slack.
    workers: list of lists (requests assigned and unfinished)."""
    best, best_key = None, None
    for wid, assigned in enumerate(workers):
        if len(assigned) >= max_batch:
            continue
        cost = cost_fn(assigned + [req])            # CalcCost (Alg. 2 lines 1-4)
        key = (cost, len(assigned), wid)
        if best_key is None or key < best_key:
            best, best_key = wid, key
    return best


def masked_tokens(r):
    """Token-granularity load of a request (§6.5): its masked image tokens."""
    return int(math.floor(r.ratio * r.L_img + 0.5))


def simulate_serving(reqs, n_workers, max_batch, step_latency, policy="mask_aware",
                     batching="continuous", interrupt_ms=0.0):
    """Discrete-event simulation of the cluster (Fig. 8 workflow, L191-L199).

    reqs: list of Req sorted by arrival. step_latency(batch) -> ms of one denoising step.
    policy (router, §6.5): "mask_aware" (Alg. 2), "round_robin" and "least_requests"
    (request granularity), "least_tokens" (token granularity: fewest masked tokens assigned).
    batching (worker, §4.3, §6.4; reading R27):
      "continuous"  FlashPS: requests join / leave the running batch at step boundaries (L237),
                    pre- / post-processing run in other processes (disaggregated, L235);
      "strawman"    the same, but each request's preprocessing (when it joins) and
                    postprocessing (when it leaves) run in the worker's main process: every
                    such event adds `interrupt_ms` before the worker's next step (L233);
      "static"      a batch is formed only when the worker is idle and runs until all of its
                    requests finish; later requests wait (L228).
    Returns {rid: (arrival, finish of its last denoising step)}."""
    workers = [[] for _ in range(n_workers)]         # assigned, unfinished
    running = [[] for _ in range(n_workers)]         # joined the running batch
    remaining = {}
    busy = [False] * n_workers
    joined = set()
    held = []
    out = {}
    ev = []
    seq = 0
    for r in reqs:
        heapq.heappush(ev, (r.arrival, 1, seq, "arr", r))
        seq += 1
    rr = [0]

    def assign(r, now):
        if policy == "mask_aware":
            wid = route(r, workers, step_latency, max_batch)
        else:
            free = [w for w in range(n_workers) if len(workers[w]) < max_batch]
            if not free:
                wid = None
            elif policy == "round_robin":
                wid = min(free, key=lambda w: ((w - rr[0]) % n_workers))
                rr[0] = (wid + 1) % n_workers
            elif policy == "least_tokens":
                wid = min(free, key=lambda w: (sum(masked_tokens(q) for q in workers[w]), w))
            else:
                wid = min(free, key=lambda w: (len(workers[w]), w))
        if wid is None:
            held.append(r)
            return
        workers[wid].append(r)
        remaining[r.rid] = r.steps
        if not busy[wid]:
            start_step(wid, now, 0)

    def start_step(wid, now, n_left):
        nonlocal seq
        if batching == "static":
            batch = [r for r in running[wid] if remaining[r.rid] > 0]   # no newcomers ...
            if not batch:
                batch = list(workers[wid])           # ... until the whole batch is done
        else:
            batch = list(workers[wid])               # join at the step boundary (L237)
        new = [r for r in batch if r.rid not in joined]
        joined.update(r.rid for r in new)
        running[wid] = batch
        if not batch:
            busy[wid] = False
            return
        busy[wid] = True
        extra = interrupt_ms * (len(new) + n_left) if batching == "strawman" else 0.0
        heapq.heappush(ev, (now + extra + step_latency(batch), 0, seq, "step", wid))
        seq += 1

    while ev:
        now, _, _, kind, obj = heapq.heappop(ev)
        if kind == "arr":
            assign(obj, now)
            continue
        wid = obj
        n_left = 0
        for r in running[wid]:
            remaining[r.rid] -= 1
            if remaining[r.rid] == 0:
                workers[wid].remove(r)               # leave at the step boundary (L237)
                out[r.rid] = (r.arrival, now)
                n_left += 1
        while held and len(workers[wid]) < max_batch:
            assign(held.pop(0), now)
        start_step(wid, now, n_left)
    return out
