"""Pins for oracle/pipeline.py (Alg. 1 reading R11) and oracle/counters.py (Table 1)."""
import json
import math
import os

import numpy as np
import pytest

import synth
from oracle import counters as C
from oracle import pipeline as P


def _golden():
    return json.load(open(os.path.join(os.path.dirname(__file__), "golden",
                                       "pipeline_cases.json")))["cases"]


@pytest.mark.parametrize("case", _golden(), ids=lambda c: c["name"])
def test_hand_timelines(case):
    v = P.simulate(case["use"], case["Cw"], case["Cwo"], case["Lm"], case["mode"],
                   case["final"], case.get("slots"))
    assert v == pytest.approx(case["latency"])


def test_limits():
    """L^m = 0 -> caching every block is optimal; C_w^m >= C_w/o -> caching nothing is."""
    g = synth.rng(0)
    for mode in ("kv", "y"):
        Cw = g.uniform(1, 2, 8); Cwo = Cw + g.uniform(0.5, 2, 8)
        lat, plan = P.plan_bruteforce(Cw, Cwo, np.zeros(8), mode)
        assert plan == [1] * 8 and lat == pytest.approx(Cw.sum())
        lat, plan = P.plan_bruteforce(Cwo + 1, Cwo, g.uniform(0, 1, 8), mode, 0.1)
        assert plan == [0] * 8 and lat == pytest.approx(Cwo.sum())


def test_naive_sequential_is_sum():
    """Fig. 9-Top: with one staging slot and loads as long as compute, nothing overlaps."""
    Cw, Lm = [1.0, 2.0, 3.0], [1.5, 0.5, 2.0]
    v = P.simulate([1, 1, 1], Cw, [9, 9, 9], Lm, "kv", 0.0, slots=1)
    assert v == pytest.approx(sum(Cw) + sum(Lm))


def test_kv_suffix_scan_is_exact():
    """KV-mode feasible plans are exactly the N+1 suffixes, so the O(N) scan is optimal."""
    g = synth.rng(1)
    for _ in range(100):
        N = int(g.integers(1, 11))
        Cw, Cwo, Lm = g.uniform(0.5, 2, N), g.uniform(1, 4, N), g.uniform(0, 3, N)
        fin = float(g.uniform(0, 1))
        a = P.plan_bruteforce(Cw, Cwo, Lm, "kv", fin)[0]
        # exhaustive over ALL 2^N plans (infeasible ones score +inf)
        import itertools
        b = min(P.simulate(p, Cw, Cwo, Lm, "kv", fin) for p in itertools.product((0, 1), repeat=N))
        assert a == pytest.approx(b)
        assert P.plan_suffix_scan(Cw, Cwo, Lm, "kv", fin)[0] == pytest.approx(a)


def test_y_bruteforce_beats_or_ties_suffix():
    g = synth.rng(2)
    worse = 0
    for _ in range(60):
        N = int(g.integers(2, 10))
        Cw, Cwo, Lm = g.uniform(0.2, 2, N), g.uniform(1, 4, N), g.uniform(0, 4, N)
        a = P.plan_bruteforce(Cw, Cwo, Lm, "y")[0]
        b = P.plan_suffix_scan(Cw, Cwo, Lm, "y")[0]
        assert a <= b + 1e-12
        worse += b > a + 1e-9
    assert worse > 0          # heterogeneous Y-mode stacks do need the exhaustive/DP planner


def test_more_slots_never_slower():
    g = synth.rng(3)
    for _ in range(50):
        N = 6
        Cw, Cwo, Lm = g.uniform(0.5, 2, N), g.uniform(1, 4, N), g.uniform(0, 3, N)
        use = [int(v) for v in g.integers(0, 2, N)]
        for mode in ("y",):
            vals = [P.simulate(use, Cw, Cwo, Lm, mode, 0.0, s) for s in (1, 2, 3, None)]
            assert all(vals[i] >= vals[i + 1] - 1e-12 for i in range(3))


def test_table1_scaling():
    """Table 1 (L165-L173): with image-only tokens, FFN, projection and QK^T FLOPs of the
    KV-mode block are exactly m times the dense ones; cache shape is ((1-m)L, H)."""
    L, H, F = 4096, 3072, 12288
    for m in (0.05, 0.2, 0.5):
        n = synth.n_masked_for(m, L)
        ratio = n / L
        assert C.gemm_flops("kv", n, L, H, F) == pytest.approx(ratio * C.gemm_flops("dense", L, L, H, F))
        attn_m = C.block_flops("kv", n, L, H, F) - C.gemm_flops("kv", n, L, H, F)
        attn_d = C.block_flops("dense", L, L, H, F) - C.gemm_flops("dense", L, L, H, F)
        assert attn_m == pytest.approx(ratio * attn_d)
        assert C.cache_bytes("y", L - n, H, 2) == (L - n) * H * 2
        assert C.cache_bytes("kv", L - n, H, 2) == 2 * C.cache_bytes("y", L - n, H, 2)  # L161
        # Y-mode keeps the K/V projections of the unmasked rows (R5): exactly 4uH^2 more
        assert C.block_flops("y", n, L, H, F) - C.block_flops("kv", n, L, H, F) == 4 * (L - n) * H * H


def test_flops_match_matmul_shapes():
    """Count 2*m*n*k over the matmuls oracle/block.py performs (instrumented linear/attention)."""
    from oracle import block as B
    g = synth.rng(4)
    H, heads, F, L = 16, 2, 40, 24
    w = synth.block_weights(g, H, F, "f32")
    x = synth.latent(g, L, H, "f32")
    mod = B.identity_mod(H)
    M = np.arange(0, L, 3); U = np.setdiff1d(np.arange(L), M)
    count = {"f": 0}
    orig = B.linear, B.attention

    def lin(h, W, b):
        count["f"] += 2 * h.shape[0] * W.shape[0] * W.shape[1]
        return orig[0](h, W, b)

    def att(Q, K, V, heads_):
        count["f"] += 2 * Q.shape[0] * K.shape[0] * Q.shape[1] * 2
        return orig[1](Q, K, V, heads_)

    B.linear, B.attention = lin, att
    try:
        B.dense_block(x, w, mod, heads)
        assert count["f"] == C.block_flops("dense", L, L, H, F); count["f"] = 0
        B.masked_block_kv(x[M], M, U, x[U], x[U], w, mod, heads, L)
        assert count["f"] == C.block_flops("kv", len(M), L, H, F); count["f"] = 0
        B.masked_block_y(x[M], M, U, x[U], w, mod, heads, L)
        assert count["f"] == C.block_flops("y", len(M), L, H, F)
    finally:
        B.linear, B.attention = orig


def test_sdxl_flops_match_matmul_shapes():
    """The SDXL block's counts (R24) against the matmuls oracle/block.py performs."""
    from oracle import block as B
    g = synth.rng(5)
    H, heads, F, L, Lc, D = 16, 2, 32, 24, 5, 12
    w = synth.block_weights(g, H, F, "f32", "sdxl", D_ctx=D)
    x = synth.latent(g, L, H, "f32")
    ctx = synth.context(g, Lc, D, "f32")
    M = np.arange(0, L, 3); U = np.setdiff1d(np.arange(L), M)
    count = {"f": 0}
    orig = B.linear, B.attention

    def lin(h, W, b):
        count["f"] += 2 * h.shape[0] * W.shape[0] * W.shape[1]
        return orig[0](h, W, b)

    def att(Q, K, V, heads_):
        count["f"] += 2 * Q.shape[0] * K.shape[0] * Q.shape[1] * 2
        return orig[1](Q, K, V, heads_)

    B.linear, B.attention = lin, att
    cf = C.context_flops(Lc, D, H)
    try:
        B.dense_block(x, w, None, heads, ctx)
        assert count["f"] == C.block_flops("dense", L, L, H, F, "sdxl", Lc) + cf; count["f"] = 0
        B.masked_block_kv(x[M], M, U, x[U], x[U], w, None, heads, L, ctx)
        assert count["f"] == C.block_flops("kv", len(M), L, H, F, "sdxl", Lc) + cf; count["f"] = 0
        B.masked_block_y(x[M], M, U, x[U], w, None, heads, L, ctx)
        assert count["f"] == C.block_flops("y", len(M), L, H, F, "sdxl", Lc) + cf
    finally:
        B.linear, B.attention = orig


def test_multistep_without_cross_step_is_steps_times_alg1_model():
    """cross_step=False: consecutive steps are independent copies of the pinned R11 model."""
    g = synth.rng(61)
    for mode in ("kv", "y"):
        for _ in range(30):
            N = int(g.integers(1, 9))
            Cw, Cwo, Lm = g.uniform(0.1, 1, N), g.uniform(1, 2, N), g.uniform(0, 2, N)
            fin = float(g.uniform(0, 0.5))
            plan = [0] * int(g.integers(0, N + 1))
            plan += [1] * (N - len(plan))
            one = P.simulate(plan, Cw, Cwo, Lm, mode, fin)
            tot, ends = P.simulate_steps(plan, Cw, Cwo, Lm, mode, fin, steps=4)
            assert tot == pytest.approx(4 * one, rel=1e-12)
            assert ends == pytest.approx([one * (s + 1) for s in range(4)], rel=1e-12)


def test_cross_step_never_slower_and_converges_to_busier_stream():
    """cross_step=True: never slower than per-step pipelines, and the long-run step time is
    the busier stream's total (closed form) -- the link never idles when load-bound and the
    compute stream never waits when compute-bound."""
    g = synth.rng(62)
    for mode in ("kv", "y"):
        for _ in range(40):
            N = int(g.integers(2, 10))
            Cw, Cwo, Lm = g.uniform(0.1, 1, N), g.uniform(1, 2, N), g.uniform(0, 2.5, N)
            fin = float(g.uniform(0, 0.5))
            k = int(g.integers(1, N + 1))
            plan = [0] * (N - k) + [1] * k
            base, _ = P.simulate_steps(plan, Cw, Cwo, Lm, mode, fin, steps=40)
            tot, ends = P.simulate_steps(plan, Cw, Cwo, Lm, mode, fin, steps=40, cross_step=True)
            assert tot <= base + 1e-9
            steady = P.steady_step_latency(plan, Cw, Cwo, Lm, mode, fin)
            comp = sum(Cw[l] if plan[l] else Cwo[l] for l in range(N))
            load = sum(Lm[l] for l in range(N) if plan[l]) + (fin if mode == "kv" else 0.0)
            assert max(comp, load) - 1e-9 <= steady <= P.simulate(plan, Cw, Cwo, Lm, mode, fin) + 1e-9
            # no load time at all: the compute stream alone sets the pace (closed form)
            z = P.steady_step_latency(plan, Cw, Cwo, np.zeros(N), mode, 0.0)
            assert z == pytest.approx(comp, rel=1e-12)


def test_cross_step_busy_link_closed_form():
    """Load-bound with a dense prefix long enough to cover every slot's reuse cycle: the link
    never idles, one step = all loads + the final load (hand-derived)."""
    N = 6
    Cw, Cwo = [0.1] * N, [1.0] * N
    Lm = [2.0] * N
    plan = [0, 0, 0, 1, 1, 1]            # prefix compute 3.0, loads 6.0 + final 0.5
    assert P.steady_step_latency(plan, Cw, Cwo, Lm, "kv", 0.5) == pytest.approx(6.5)
    # all cached, Cw 0.5, loads 0.6: per step block l waits for load l -> 6 x 0.6 + 0.5 = 4.1;
    # across steps the loads of step s+1 run under step s's compute -> the link's 3.6
    Cw2, Lm2 = [0.5] * N, [0.6] * N
    assert P.simulate([1] * N, Cw2, Cwo, Lm2, "kv", 0.0) == pytest.approx(4.1)
    assert P.steady_step_latency([1] * N, Cw2, Cwo, Lm2, "kv", 0.0) == pytest.approx(3.6)


def test_steady_planner_is_exhaustive_optimum_over_suffixes():
    g = synth.rng(63)
    for _ in range(50):
        N = int(g.integers(1, 12))
        Cw, Cwo, Lm = g.uniform(0.1, 1, N), g.uniform(1, 2, N), g.uniform(0, 2, N)
        best, plan = P.plan_steady_suffix(Cw, Cwo, Lm, "kv", 0.2)
        for k in range(N + 1):
            p = [0] * (N - k) + [1] * k
            assert best <= P.steady_step_latency(p, Cw, Cwo, Lm, "kv", 0.2) + 1e-12


def test_transition_planner_hand_case_flips_the_plan():
    """KV-mode transition block (R28), a timeline derived by hand under the R11 model: N = 2,
    C_w = [1, 1], C_w/o = [3, 3], C_t = [1.5, 1.5], loads [1, 1], no final load.
    Without the transition: [0,0] = 6; [0,1]: block 0 ends 3, block 1 at max(3, 1) -> 4;
    [1,1]: loads end 1, 2; block 0 1 -> 2, block 1 max(2, 2) -> 3  => [1,1] at 3.
    With it, [0,1]: block 0 (transition) ends 1.5, block 1 at max(1.5, 1) -> 2.5  => [0,1]."""
    Cw, Cwo, Ct, Lm = [1.0, 1.0], [3.0, 3.0], [1.5, 1.5], [1.0, 1.0]
    assert P.plan_suffix_scan(Cw, Cwo, Lm, "kv") == (3.0, [1, 1])
    assert P.plan_transition_suffix(Cw, Cwo, Ct, Lm) == (2.5, [0, 1])
    # cross-step (R26): the [0,1] plan's loads hide (1 per step against 2.5 of compute), so its
    # steady step is the compute stream's sum 1.5 + 1
    lat, plan = P.plan_transition_suffix(Cw, Cwo, Ct, Lm, cross_step=True)
    assert P.steady_step_latency([0, 1], Cw, [1.5, 3.0], Lm, "kv") == pytest.approx(2.5)
    assert lat <= 2.5 + 1e-12


@pytest.mark.parametrize("cross", [False, True])
def test_transition_planner_reduces_to_alg1_and_never_loses(cross):
    """With C_t = C_w/o the transition planner is the suffix planner (R11 / R26); with
    C_t <= C_w/o it is never slower."""
    g = synth.rng(28)
    for _ in range(60):
        N = int(g.integers(1, 10))
        Cw = list(g.uniform(0.1, 1.0, N))
        Cwo = [c + float(g.uniform(0.2, 2.0)) for c in Cw]
        Lm = list(g.uniform(0.05, 1.5, N))
        fin = float(g.uniform(0, 0.5))
        ref = (P.plan_steady_suffix if cross else P.plan_suffix_scan)(Cw, Cwo, Lm, "kv", fin)
        same = P.plan_transition_suffix(Cw, Cwo, Cwo, Lm, fin, cross)
        assert same[0] == pytest.approx(ref[0], rel=1e-12) and same[1] == ref[1]
        Ct = [c + float(g.uniform(0, 1)) * (d - c) for c, d in zip(Cw, Cwo)]
        lat, plan = P.plan_transition_suffix(Cw, Cwo, Ct, Lm, fin, cross)
        assert lat <= ref[0] + 1e-12
