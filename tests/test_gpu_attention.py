"""GPU parity of a6 alone (fps_masked_attention) vs the oracle's attention: varlen requests with
ragged query tiles and key lengths that are not multiples of the 128-key tile, d = 64 / 128,
tensor-core and SIMT kernels."""
import numpy as np
import pytest
import torch

import synth
from oracle.block import attention
from gpu_util import TOL, check_close, to_dev, to_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as fps
    fps.require_gpu()
    return fps


KERNEL_FLAGS = {"auto": 0, "pair": 4096, "p_tmem": 48, "two_tile": 32, "one_tile": 16, "simt": 2}


@pytest.mark.parametrize("d,heads", [(128, 3), (64, 4)])
@pytest.mark.parametrize("kernel", list(KERNEL_FLAGS))
def test_varlen_attention(F, d, heads, kernel):
    g = synth.rng(d * 10 + heads)
    H = d * heads
    n_active = [1, 130, 257, 64, 384, 200]
    L = [5, 300, 1000, 129, 700, 256]
    q = synth.latent(g, sum(n_active), H, "bf16")
    kv = synth.latent(g, sum(L), 2 * H, "bf16") * 2.0       # larger logits exercise the max
    kv = synth.bf16_round(kv)
    F.fps_set_disable_tc(KERNEL_FLAGS[kernel])
    try:
        out = F.masked_attention(to_dev(q, "bf16"), to_dev(kv, "bf16"), n_active, L, heads)
        torch.cuda.synchronize()
    finally:
        F.fps_set_disable_tc(0)
    got = to_np(out)
    qo, ko = 0, 0
    for n, l in zip(n_active, L):
        ref = attention(q[qo:qo + n], kv[ko:ko + l, :H], kv[ko:ko + l, H:], heads)
        check_close(got[qo:qo + n], ref, TOL["bf16"], f"attention n={n} L={l}")
        qo += n
        ko += l


@pytest.mark.parametrize("kernel", ["auto", "pair", "p_tmem", "two_tile", "one_tile"])
def test_attention_large_logits_lazy_rescale(F, kernel):
    """Keys whose scores grow along the sequence force the lazy-max rescale of O in TMEM."""
    g = synth.rng(5)
    heads, d = 2, 128
    H = heads * d
    n, L = 128, 1024
    q = synth.bf16_round(np.ones((n, H), np.float32) * 0.25)
    k = synth.bf16_round(np.linspace(-4, 4, L, dtype=np.float32)[:, None] * np.ones((1, H), np.float32))
    v = synth.latent(g, L, H, "bf16")
    kv = np.concatenate([k, v], 1)
    F.fps_set_disable_tc(KERNEL_FLAGS[kernel])
    try:
        q2 = np.concatenate([q, q], 0)                      # 256 query rows: both tiles of a pair
        out = F.masked_attention(to_dev(q2, "bf16"), to_dev(kv, "bf16"), [2 * n], [L], heads)
        torch.cuda.synchronize()
    finally:
        F.fps_set_disable_tc(0)
    ref = attention(q, k, v, heads)
    check_close(to_np(out)[:n], ref, TOL["bf16"], "rescale")
    check_close(to_np(out)[n:], ref, TOL["bf16"], "rescale (second tile of the pair)")


@pytest.mark.parametrize("d,heads", [(128, 3), (64, 10)])
def test_short_key_sets(F, d, heads):
    """Every request <= 128 keys (the SDXL cross-attention over a 77-token prompt): the
    register-tile kernel, with key counts off every 8 / 16 boundary, ragged query tiles, an
    empty request and large logits."""
    g = synth.rng(700 + d)
    H = d * heads
    n_active = [300, 1, 0, 129, 77, 16]
    L = [77, 1, 5, 128, 120, 33]
    q = synth.latent(g, sum(n_active), H, "bf16")
    kv = synth.bf16_round(synth.latent(g, sum(L), 2 * H, "bf16") * 3.0)
    out = F.masked_attention(to_dev(q, "bf16"), to_dev(kv, "bf16"), n_active, L, heads)
    torch.cuda.synchronize()
    got = to_np(out)
    qo, ko = 0, 0
    for n, l in zip(n_active, L):
        if n:
            ref = attention(q[qo:qo + n], kv[ko:ko + l, :H], kv[ko:ko + l, H:], heads)
            check_close(got[qo:qo + n], ref, TOL["bf16"], f"short attention n={n} L={l}")
        qo += n
        ko += l
