"""Product-side scheduling (paper_conf_..._b200/sched.py: Alg. 2 routing on the library's Alg. 1
planner, serving DES) vs the oracle's independent implementation (oracle/sched.py)."""
import numpy as np
import pytest

import synth
from oracle import sched as OS
from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched as PS


def _pool(seed, n, rate_ms):
    g = synth.rng(seed)
    ratios = synth.sample_mask_ratios(g, n)
    t = np.cumsum(g.exponential(rate_ms, n))
    return ratios, t


@pytest.mark.parametrize("policy,batching", [("mask_aware", "continuous"),
                                              ("round_robin", "continuous"),
                                              ("least_requests", "continuous"),
                                              ("least_tokens", "continuous"),
                                              ("mask_aware", "static"),
                                              ("mask_aware", "strawman"),
                                              ("least_requests", "strawman")])
def test_des_matches_oracle(policy, batching):
    ratios, t = _pool(3, 30, 40.0)
    L_img, L_txt = 4096, 512
    # one latency function for both sides: the oracle's cost model (suffix scan == library
    # planner in KV-mode, test_lib_cpu pins that), so the comparison isolates the DES + routing
    ocm = OS.CostModel([(4608, 3072, 12288)] * 57, (1 / 1.2e9, 0.05), (1 / 4.6e7, 0.01), "kv")
    oreqs = [OS.Req(i, float(t[i]), float(ratios[i]), 6, L_img, L_txt) for i in range(30)]
    pcm = PS.CostModel(57, 3072, 12288, "kv", comp=(1 / 1.2e9, 0.05), load=(1 / 4.6e7, 0.01))
    preqs = [PS.Request(i, synth.n_masked_for(float(ratios[i]), L_img) + L_txt, L_img + L_txt,
                        arrival=float(t[i]), steps=6,
                        tokens=synth.n_masked_for(float(ratios[i]), L_img)) for i in range(30)]
    o = OS.simulate_serving(oreqs, 3, 4, ocm.step_latency, policy, batching, interrupt_ms=25.0)
    p = PS.simulate_serving(preqs, 3, 4, pcm.step_latency, policy, batching, interrupt_ms=25.0)
    assert set(o) == set(p)
    for k in o:
        assert p[k][1] == pytest.approx(o[k][1], rel=1e-9)


def test_library_cost_equals_oracle_cost():
    ocm = OS.CostModel([(4608, 3072, 12288)] * 57, (1 / 1.2e9, 0.05), (1 / 4.6e7, 0.01), "kv")
    pcm = PS.CostModel(57, 3072, 12288, "kv", comp=(1 / 1.2e9, 0.05), load=(1 / 4.6e7, 0.01))
    for ratios in ([0.2], [0.05, 0.6], [0.1, 0.2, 0.3, 0.4]):
        ob = [OS.Req(i, 0, m, 28, 4096, 512) for i, m in enumerate(ratios)]
        pb = [PS.Request(i, synth.n_masked_for(m, 4096) + 512, 4608) for i, m in enumerate(ratios)]
        assert pcm.step_latency(pb) == pytest.approx(ocm.step_latency(ob), rel=1e-9)


def test_stats():
    s = PS.latency_stats({0: (0, 10), 1: (0, 20), 2: (5, 45)})
    assert s["p50_ms"] == 20 and s["p95_ms"] == 40 and s["mean_ms"] == pytest.approx(70 / 3)


@pytest.mark.parametrize("kind,Lc", [("sdxl", 77), ("seq", 0)])
def test_product_flops_match_oracle_counters(kind, Lc):
    """The product's per-block FLOP count (planner / balancer cost input) equals the oracle's
    Table 1 counters, including the SDXL block's cross-attention and GEGLU terms (R24)."""
    from oracle import counters as OC
    for mode in ("kv", "y", "dense"):
        for n, L, H, F in ((410, 4096, 640, 2560), (307, 1024, 1280, 5120), (1331, 4608, 3072, 12288)):
            assert PS.block_flops(mode, n, L, H, F, kind, Lc) == pytest.approx(
                OC.block_flops(mode, n, L, H, F, kind, Lc), rel=1e-12)


def test_mixed_and_sdxl_costs_are_sums_of_their_parts():
    """configs[4] mixed traffic: a worker's step over a mixed batch = the Flux sub-batch's
    latency + the SDXL sub-batch's, and an SDXL step = its two UNet levels' pipeline latencies
    with the request's mask ratio pooled to each level (R19, R8)."""
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    flux = sched.CostModel(57, 3072, 12288, "kv", comp=(7e-13, 0.1), load=(1 / 5.5e7, 0.003))
    A = sched.CostModel(10, 640, 2560, "kv", comp=(1.6e-12, 0.08), load=(1 / 5.4e7, 0.002),
                        kind="sdxl", Lc=77)
    Bm = sched.CostModel(60, 1280, 5120, "kv", comp=(1.0e-12, 0.1), load=(1 / 5.3e7, 0.004),
                         kind="sdxl", Lc=77)
    sd = sched.SdxlCost([A, Bm], [4096, 1024])
    mix = sched.MixedCost({"flux": flux, "sdxl": sd})
    f = [sched.Request(0, 1331, 4608, model="flux"), sched.Request(1, 900, 4608, model="flux")]
    s = [sched.Request(2, 0, 4096, model="sdxl", ratio=0.25)]
    assert mix.step_latency(f + s) == pytest.approx(flux.step_latency(f) + sd.step_latency(s))
    assert sd.step_latency(s) == pytest.approx(
        A.step_latency([sched.Request(2, 1024, 4096)]) + Bm.step_latency([sched.Request(2, 256, 1024)]))
    assert mix.step_latency([]) == 0.0
    # Alg. 2 over a mixed pool sends an SDXL request to the worker whose batch it costs least
    workers = [list(f), list(s)]
    w = sched.route(sched.Request(3, 0, 4096, model="sdxl", ratio=0.1), workers, mix.step_latency, 8)
    costs = [mix.step_latency(wk + [sched.Request(3, 0, 4096, model="sdxl", ratio=0.1)]) for wk in workers]
    assert w == int(np.argmin(costs))
