"""Pins for oracle/stack.py: the paper's degenerate cases over whole stacks and steps."""
import numpy as np
import pytest

import synth
from oracle import stack as S


def _setup(N=3, steps=2, H=32, heads=2, F=64, L_img=36, L_txt=4, seed=0, kind="seq"):
    g = synth.rng(seed)
    if kind == "flux":       # double-stream blocks then a single-stream block (R25, R23)
        W = synth.stack_weights(g, N - 1, H, F, "f32", "double") + \
            synth.stack_weights(g, 1, H, F, "f32", "par")
    else:
        W = synth.stack_weights(g, N, H, F, "f32", kind, D_ctx=24)
    mods = synth.mod_table(g, N, steps, H, "f32", streams=2 if kind == "flux" else 1)
    if kind == "flux":       # the single-stream block reads the first 6H of the 12H row
        mods = [[mods[l][s] if l < N - 1 else mods[l][s][:6 * H] for s in range(steps)]
                for l in range(N)]
    x0 = synth.latent(g, L_img + L_txt, H, "f32")
    return g, W, mods, x0, synth.delta_table(steps)


PLANS_KV = [[1, 1, 1], [0, 1, 1], [0, 0, 1], [0, 0, 0]]
PLANS_Y = PLANS_KV + [[1, 0, 1], [1, 1, 0], [0, 1, 0], [1, 0, 0]]


@pytest.mark.parametrize("mode,plan", [("kv", p) for p in PLANS_KV] + [("y", p) for p in PLANS_Y])
@pytest.mark.parametrize("kind", ["seq", "par", "sdxl", "flux"])
def test_identical_input_cache_reproduces_template(mode, plan, kind):
    """L144/L157 + L211: with the cache from the template run on the identical input, every
    feasible plan reproduces the dense trajectory over a whole stack and several steps (every
    block kind; SDXL with a prompt context, Flux-like double-stream + single-stream)."""
    g, W, mods, x0, deltas = _setup(kind=kind)
    ctx = synth.context(g, 5, 24, "f32") if kind == "sdxl" else None
    cache, xs = S.template_run(x0, W, mods, deltas, 2, 2, ctx=ctx, L_txt=4)
    mask = synth.token_mask(synth.mask_blobs(g, 6, 6, 0.3), 4)
    x = S.masked_run(x0, mask, W, mods, deltas, plan, mode, cache, 2, 2, ctx=ctx, L_txt=4)
    assert np.allclose(x, xs[2], rtol=0, atol=1e-11)


def test_empty_mask_returns_cache():
    """No active token: the output is entirely replenished from the cache (L157)."""
    g, W, mods, x0, deltas = _setup(L_txt=0)
    cache, _ = S.template_run(synth.latent(g, 36, 32, "f32"), W, mods, deltas, 2, 1)
    mask = np.zeros(36, dtype=np.uint8)
    for mode in ("kv", "y"):
        y = S.masked_stack(x0, mask, W, [mods[l][0] for l in range(3)], [1, 1, 1], mode,
                           cache[0], 2)
        assert np.array_equal(y, cache[0][2]["Y"])


def test_kv_equals_y_under_identical_cache_different_request():
    """Both caching modes agree whenever the cache is consistent with the request input."""
    g, W, mods, x0, deltas = _setup(seed=3)
    cache, xs = S.template_run(x0, W, mods, deltas, 2, 2)
    mask = synth.token_mask(synth.mask_random(g, 36, 0.2), 4)
    a = S.masked_run(x0, mask, W, mods, deltas, [1, 1, 1], "kv", cache, 2, 2)
    b = S.masked_run(x0, mask, W, mods, deltas, [1, 1, 1], "y", cache, 2, 2)
    assert np.allclose(a, b, atol=1e-11)


def test_edit_changes_only_through_masked_rows():
    """A request whose input differs from the template only on masked rows: unmasked output rows
    equal the template's (replenished), masked rows differ (they are recomputed)."""
    g, W, mods, x0, deltas = _setup(seed=5)
    cache, _ = S.template_run(x0, W, mods, deltas, 2, 1)
    mask = synth.token_mask(synth.mask_blobs(g, 6, 6, 0.25), 4)
    x_req = x0.astype(np.float64).copy()
    M = np.flatnonzero(mask)
    x_req[M] += synth.latent(g, len(M), 32, "f32")
    for mode in ("kv", "y"):
        y = S.masked_stack(x_req, mask, W, [mods[l][0] for l in range(3)], [1, 1, 1], mode,
                           cache[0], 2)
        U = np.flatnonzero(mask == 0)
        assert np.array_equal(y[U], cache[0][2]["Y"][U])
        assert not np.allclose(y[M], cache[0][2]["Y"][M], atol=1e-3)


def test_kv_nonmonotone_rejected():
    with pytest.raises(ValueError):
        S.check_plan([1, 0, 1], "kv")
    S.check_plan([1, 0, 1], "y")
