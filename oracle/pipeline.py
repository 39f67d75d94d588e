"""Alg. 1 (§4.2, Fig. 9): pipeline latency and block selection (oracle).

The body of Alg. 1 is lost in extraction; only its I/O survives (L213-L217): inputs N,
C_w^m (block latency with cache), C_w/o (without), L^m (load latency); outputs useCache and
pipeline_latency; complexity O(N) (L211). Reading R11 fixes the pipeline model:

  * one load stream issues the loads of the cached blocks in block order, back to back from
    t = 0; with `slots` staging buffers the j-th load also waits until the consumer of load
    j - slots has finished (slot reuse); slots=None means unbounded;
  * one compute stream runs blocks in order; block l starts at max(end(l-1), dep(l)) and lasts
    C_w^m[l] if cached else C_w/o[l] (L211: uncached blocks compute all tokens, load nothing);
  * KV-mode: dep(l) = end of block l's load (Fig. 9, "load i ... compute i"); the plan must be
    monotone (R11) and, if any block is cached, a final load of the last block's Y rows
    (`final_load`, R22) is issued last and must land before the step ends;
  * Y-mode: block l's cached output rows feed block l+1 (R4), so dep(l+1) = end of block l's
    load, and the step ends no earlier than the load of block N-1 if it is cached.

`simulate` is that definition; `plan_bruteforce` is the optimum by exhaustion (all 2^N plans,
or the N+1 feasible suffix plans in KV-mode); `plan_suffix_scan` evaluates only the N+1
suffix plans (the paper's O(N) claim is exact for KV-mode, whose feasible set is exactly them).
"""
from __future__ import annotations

import itertools
import math


def _feasible(use, mode):
    if mode != "kv":
        return True
    seen = False
    for u in use:
        if u:
            seen = True
        elif seen:
            return False
    return True


def simulate(use, Cw, Cwo, Lm, mode, final_load=0.0, slots=None):
    """Pipeline latency of plan `use` (R11). Infeasible KV plans return +inf."""
    N = len(use)
    if not _feasible(use, mode):
        return math.inf
    loads = [l for l in range(N) if use[l]]
    if mode == "kv" and loads:
        loads.append(N)                     # N stands for the final Y-rows load (R22)
    dur = [Lm[l] if l < N else final_load for l in loads]
    pos = {l: j for j, l in enumerate(loads)}
    end = [None] * N
    load_end = []
    state = {"t": 0.0}

    def consumer(l):
        if mode == "kv":
            return l if l < N else None
        return l + 1 if l + 1 < N else None

    def ensure(j):
        while len(load_end) <= j:
            k = len(load_end)
            start = state["t"]
            if slots is not None and k >= slots:
                c = consumer(loads[k - slots])
                assert c is not None and end[c] is not None
                start = max(start, end[c])
            state["t"] = start + dur[k]
            load_end.append(state["t"])
        return load_end[j]

    t = 0.0
    for l in range(N):
        dep = 0.0
        if mode == "kv" and use[l]:
            dep = ensure(pos[l])
        elif mode == "y" and l > 0 and use[l - 1]:
            dep = ensure(pos[l - 1])
        t = max(t, dep) + (Cw[l] if use[l] else Cwo[l])
        end[l] = t
    if mode == "kv" and loads:
        t = max(t, ensure(len(loads) - 1))
    if mode == "y" and N and use[N - 1]:
        t = max(t, ensure(pos[N - 1]))
    return t


def plan_bruteforce(Cw, Cwo, Lm, mode, final_load=0.0, slots=None):
    """Exhaustive optimum: (latency, plan). Ties -> the plan found first in this order:
    KV-mode by fewest cached blocks, Y-mode in lexicographic order of the 0/1 tuple."""
    N = len(Cw)
    if mode == "kv":
        cands = [tuple([0] * (N - k) + [1] * k) for k in range(N + 1)]
    else:
        cands = itertools.product((0, 1), repeat=N)
    best, best_plan = math.inf, None
    for p in cands:
        v = simulate(p, Cw, Cwo, Lm, mode, final_load, slots)
        if v < best:
            best, best_plan = v, list(p)
    return best, best_plan


def plan_suffix_scan(Cw, Cwo, Lm, mode, final_load=0.0, slots=None):
    """Best of the N+1 plans 'uncached prefix, cached suffix'."""
    N = len(Cw)
    best, best_plan = math.inf, None
    for k in range(N + 1):
        p = [0] * (N - k) + [1] * k
        v = simulate(p, Cw, Cwo, Lm, mode, final_load, slots)
        if v < best:
            best, best_plan = v, p
    return best, best_plan


def simulate_steps(use, Cw, Cwo, Lm, mode, final_load=0.0, steps=1, cross_step=False):
    """End time of `steps` consecutive denoising steps under plan `use` (R11 per step).

    cross_step=False: each step's two streams start when the previous step has ended (the
    per-step pipeline of Fig. 9).  cross_step=True (NEXT-2 "cross-step prefetch", reading R26):
    the load stream runs on continuously -- load j of step s starts as soon as the stream is
    free and its staging slot has been consumed in step s-1 (one slot per load; the final Y
    rows' slot is consumed by the step-end replenish) -- while compute still runs the steps in
    order (step s+1 starts after step s's last block and final load, i.e. its sampler update).
    Returns (total end time, list of per-step end times)."""
    N = len(use)
    if not _feasible(use, mode):
        return math.inf, []
    loads = [l for l in range(N) if use[l]]
    if mode == "kv" and loads:
        loads.append(N)
    dur = [Lm[l] if l < N else final_load for l in loads]
    pos = {l: j for j, l in enumerate(loads)}
    t_load, t_comp = 0.0, 0.0
    prev_consumed = [0.0] * len(loads)     # when step s-1 released slot j
    ends = []
    for s in range(steps):
        start = t_comp
        if not cross_step:
            t_load = max(t_load, start)
        load_end = []
        for j in range(len(loads)):         # the load stream issues in order
            st = max(t_load, prev_consumed[j] if cross_step else start)
            t_load = st + dur[j]
            load_end.append(t_load)
        t = start
        end = [0.0] * N
        for l in range(N):
            dep = 0.0
            if mode == "kv" and use[l]:
                dep = load_end[pos[l]]
            elif mode == "y" and l > 0 and use[l - 1]:
                dep = load_end[pos[l - 1]]
            t = max(t, dep) + (Cw[l] if use[l] else Cwo[l])
            end[l] = t
        if mode == "kv" and loads:
            t = max(t, load_end[-1])
        if mode == "y" and N and use[N - 1]:
            t = max(t, load_end[pos[N - 1]])
        for j, l in enumerate(loads):       # consumers: KV block l; Y block l+1 (or the end)
            if l == N:
                prev_consumed[j] = t
            elif mode == "kv":
                prev_consumed[j] = end[l]
            else:
                prev_consumed[j] = end[l + 1] if l + 1 < N else t
        t_comp = t
        ends.append(t)
    return t_comp, ends


STEADY_STEPS = 16


def steady_step_latency(use, Cw, Cwo, Lm, mode, final_load=0.0, steps=STEADY_STEPS):
    """Long-run per-step time with cross-step prefetch (R26): the mean step time over the
    second half of `steps` simulated steps (past the pipeline's fill transient).  At least the
    busier stream's total, max(sum of block times, sum of load times); more when a slot's
    reuse cycle (its load in step s+1 waits for its consumer in step s) binds."""
    if not _feasible(use, mode):
        return math.inf
    _, ends = simulate_steps(use, Cw, Cwo, Lm, mode, final_load, steps, cross_step=True)
    h = steps // 2
    return (ends[-1] - ends[h - 1]) / (steps - h)


def plan_steady_suffix(Cw, Cwo, Lm, mode, final_load=0.0):
    """Cross-step planner (R26): the suffix plan minimising steady_step_latency; ties -> fewer
    cached blocks."""
    N = len(Cw)
    best, best_plan = math.inf, None
    for k in range(N + 1):
        p = [0] * (N - k) + [1] * k
        v = steady_step_latency(p, Cw, Cwo, Lm, mode, final_load)
        if v < best:
            best, best_plan = v, p
    return best, best_plan


def plan_transition_suffix(Cw, Cwo, Ct, Lm, final_load=0.0, cross_step=False):
    """KV-mode Alg. 1 with the transition block (reading R28): the N+1 plans
    'uncached prefix, cached suffix', each priced with the prefix's last block at Ct[l] (it runs
    as a masked block over the fresh full input) instead of Cwo[l] when both parts are
    non-empty; latency = simulate (R11) or steady_step_latency (R26, cross_step).  Ties ->
    fewer cached blocks.  Returns (latency, plan)."""
    N = len(Cw)
    best, best_plan = math.inf, None
    for k in range(N + 1):
        p = [0] * (N - k) + [1] * k
        c = list(Cwo)
        if 0 < k < N:
            c[N - k - 1] = Ct[N - k - 1]
        v = (steady_step_latency(p, Cw, c, Lm, "kv", final_load) if cross_step
             else simulate(p, Cw, c, Lm, "kv", final_load))
        if v < best:
            best, best_plan = v, p
    return best, best_plan
