"""Pins for oracle/sched.py (§4.4 regression models, Alg. 2 routing, serving DES)."""
import numpy as np
import pytest

import synth
from oracle import sched as SC


def test_fit_exact_recovery_and_vs_polyfit():
    g = synth.rng(0)
    x = g.uniform(1e9, 1e12, 50)
    a, b, r2 = SC.fit_linear(x, 3e-9 * x + 0.7)
    assert a == pytest.approx(3e-9) and b == pytest.approx(0.7) and r2 == pytest.approx(1.0)
    y = 2e-9 * x + 1 + g.normal(0, 50, 50)
    a, b, r2 = SC.fit_linear(x, y)
    pa, pb = np.polyfit(x, y, 1)                               # library routine
    assert a == pytest.approx(pa, rel=1e-6) and b == pytest.approx(pb, rel=1e-6, abs=1e-6)
    assert 0.0 < r2 < 1.0


def _model(mode="kv"):
    # Flux-like single level, 4 blocks; ms per FLOP / per byte
    return SC.CostModel([(4608, 3072, 12288)] * 4, (1 / 1.0e9, 0.01), (1 / 55e6, 0.005), mode)


def test_route_spreads_identical_requests():
    cm = _model()
    workers = [[] for _ in range(4)]
    for i in range(8):
        r = SC.Req(i, 0.0, 0.2, 28, 4096, 512)
        wid = SC.route(r, workers, cm.step_latency, 8)
        workers[wid].append(r)
    assert [len(w) for w in workers] == [2, 2, 2, 2]


def test_route_heavy_request_avoids_loaded_worker():
    cm = _model()
    workers = [[SC.Req(0, 0, 0.6, 28, 4096, 512), SC.Req(1, 0, 0.6, 28, 4096, 512)],
               [SC.Req(2, 0, 0.05, 28, 4096, 512), SC.Req(3, 0, 0.05, 28, 4096, 512)]]
    # request-count balancing would see a tie; the mask-aware cost does not
    assert SC.route(SC.Req(9, 0, 0.5, 28, 4096, 512), workers, cm.step_latency, 8) == 1


def test_route_respects_slack():
    cm = _model()
    workers = [[SC.Req(i, 0, 0.05, 28, 4096, 512) for i in range(2)], []]
    assert SC.route(SC.Req(9, 0, 0.05, 28, 4096, 512), workers, cm.step_latency, 2) == 1
    workers[1] = [SC.Req(5, 0, 0.5, 28, 4096, 512), SC.Req(6, 0, 0.5, 28, 4096, 512)]
    assert SC.route(SC.Req(9, 0, 0.05, 28, 4096, 512), workers, cm.step_latency, 2) is None


def test_des_single_request_closed_form():
    cm = _model()
    r = SC.Req(0, 5.0, 0.2, 10, 4096, 512)
    out = SC.simulate_serving([r], 2, 8, cm.step_latency)
    assert out[0][1] == pytest.approx(5.0 + 10 * cm.step_latency([r]))


def test_des_continuous_batching_joins_at_step_boundary():
    """L237: a request arriving mid-step joins at the next step boundary, not at batch end."""
    lat = lambda b: 10.0 * len(b)
    r0 = SC.Req(0, 0.0, 0.2, 3, 4096, 0)
    r1 = SC.Req(1, 5.0, 0.2, 1, 4096, 0)
    out = SC.simulate_serving([r0, r1], 1, 8, lat)
    # r0 step0 0..10 alone; r1 joins at 10: step 10..30 (batch 2) -> r1 done at 30
    assert out[1][1] == pytest.approx(30.0)
    # r0: steps end 10, 30, then alone 30..40
    assert out[0][1] == pytest.approx(40.0)


def test_des_mask_aware_not_worse_on_skewed_load():
    g = synth.rng(5)
    cm = _model()
    ratios = synth.sample_mask_ratios(g, 40)
    t = np.cumsum(g.exponential(60.0, 40))
    reqs = [SC.Req(i, float(t[i]), float(ratios[i]), 8, 4096, 512) for i in range(40)]
    lat = lambda pol: np.mean([f - a for a, f in SC.simulate_serving(reqs, 4, 8, cm.step_latency, pol).values()])
    assert lat("mask_aware") <= lat("round_robin") * 1.05


# ---- NEXT-3: worker batching policies (§4.3, §6.4) and token-granularity routing (§6.5) ----
def _reqs(spec):
    """spec: list of (arrival ms, steps); ratio 0.2 each."""
    return [SC.Req(i, a, 0.2, s, 64) for i, (a, s) in enumerate(spec)]


def test_static_batching_closed_form():
    """1 worker, max batch 2, step latency = 10 ms x batch size; a request arriving at an idle
    worker starts a step at once.  r0 (2 steps) at 0, r1 (4 steps) at 5, r2 (1 step) at 6 (held:
    no slack).  Continuous: r1 joins at the boundary 10 -> step 10..30 ends r0; r2 joins ->
    30..50 ends r2; r1 alone 50..60..70.  Static: nobody joins r0's batch (0..10..20); then
    {r1, r2} 20..40 ends r2; r1 alone 40..50..60..70."""
    lat = lambda b: 10.0 * len(b)
    reqs = _reqs([(0, 2), (5, 4), (6, 1)])
    c = SC.simulate_serving(reqs, 1, 2, lat, "least_requests", "continuous")
    assert {k: v[1] for k, v in c.items()} == {0: 30.0, 1: 70.0, 2: 50.0}
    st = SC.simulate_serving(reqs, 1, 2, lat, "least_requests", "static")
    assert {k: v[1] for k, v in st.items()} == {0: 20.0, 1: 70.0, 2: 40.0}


def test_static_equals_continuous_without_overlap():
    """Requests that never meet (each arrives after the previous one finished): every worker
    batching policy gives the same result, interruption-free."""
    lat = lambda b: 7.0 + 3.0 * len(b)
    reqs = _reqs([(0, 5), (100, 3), (200, 4)])
    ref = SC.simulate_serving(reqs, 1, 8, lat, "least_requests", "continuous")
    assert SC.simulate_serving(reqs, 1, 8, lat, "least_requests", "static") == ref
    assert SC.simulate_serving(reqs, 1, 8, lat, "least_requests", "strawman") == ref


def test_strawman_interruptions_closed_form():
    """r0 (3 steps) at 0, r1 (1 step) at 15, step 10 ms, interruption 4 ms.  Strawman: r0's
    preprocessing precedes its first step (0..4..14); r1 has not arrived at 14, so 14..24 runs
    r0 alone; at 24 r1 joins (+4 preprocessing) -> 28..38 ends both.  Disaggregated
    (continuous): 0..10, 10..20, then {r0, r1} 20..30."""
    lat = lambda b: 10.0
    reqs = _reqs([(0, 3), (15, 1)])
    s = SC.simulate_serving(reqs, 1, 8, lat, "least_requests", "strawman", interrupt_ms=4.0)
    assert {k: v[1] for k, v in s.items()} == {0: 38.0, 1: 38.0}
    c = SC.simulate_serving(reqs, 1, 8, lat, "least_requests", "continuous", interrupt_ms=4.0)
    assert {k: v[1] for k, v in c.items()} == {0: 30.0, 1: 30.0}


def test_least_tokens_routing():
    """Token granularity (§6.5): a heavy request (ratio 0.6) stays alone and the two light ones
    (0.1) share the other worker; request granularity splits the light ones instead."""
    def batches(policy):
        seen = []

        def lat(b):
            seen.append(tuple(sorted(r.rid for r in b)))
            return 1e6                                   # nobody finishes: routing only
        reqs = [SC.Req(0, 0.0, 0.6, 5, 100), SC.Req(1, 1.0, 0.1, 5, 100), SC.Req(2, 2.0, 0.1, 5, 100)]
        SC.simulate_serving(reqs, 2, 8, lat, policy)
        return set(seen)
    assert (1, 2) in batches("least_tokens")
    assert (0, 2) in batches("least_requests")
