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
