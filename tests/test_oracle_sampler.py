"""Pins for the sampler update after the stack (a9): the synthetic Euler update of reading R21
and the flow-matching Euler sampler with inpainting blend of reading R29 (oracle/sampler.py).

Each pin is fixed by hand arithmetic or a closed form, not by re-running the oracle's formula:
a wrong step index of delta / sigma / the modulation row / the cache entry, a wrong sign, or a
blend applied to the wrong rows fails one of them."""
import math

import numpy as np
import pytest

import synth
from oracle import sampler as SM
from oracle import stack as S


def _zero_block(H, b_o, b_down):
    """A sequential block with zero weights: Q = K = V = 0, so the attention output does not
    matter (W_o = 0) and the block is y = x + gate1 * b_o + gate2 * b_down exactly."""
    z = lambda *s: np.zeros(s)
    return {"w_qkv": z(3 * H, H), "b_qkv": z(3 * H), "w_o": z(H, H), "b_o": np.array(b_o, float),
            "w_up": z(4 * H, H), "b_up": z(4 * H), "w_down": z(H, 4 * H),
            "b_down": np.array(b_down, float)}


def _mod(g1, g2, H=2):
    return np.concatenate([np.zeros(H), np.zeros(H), np.full(H, g1), np.zeros(H), np.zeros(H),
                           np.full(H, g2)])


def test_r21_hand_case_two_steps():
    """One zero-weight block, two steps, hand-derived (R21): step s uses delta_s and
    block l's modulation row of step s.
      step 0: y0 = x0 + 1*[1,0] + 1*[0,2];   x1 = x0 - 0.5 y0 = [[0,0],[1,1],[2,2]]
      step 1: y1 = x1 + 2*[1,0] + 0.5*[0,2]; x2 = x1 - 0.25 y1 = [[-.5,-.25],[.25,.5],[1,1.25]]"""
    W = [_zero_block(2, [1, 0], [0, 2])]
    mods = [[_mod(1.0, 1.0), _mod(2.0, 0.5)]]
    deltas = [-0.5, -0.25]
    x0 = np.array([[1, 2], [3, 4], [5, 6]], float)
    cache, xs = S.template_run(x0, W, mods, deltas, 1, 2)
    assert np.array_equal(xs[1], [[0, 0], [1, 1], [2, 2]])
    assert np.array_equal(xs[2], [[-0.5, -0.25], [0.25, 0.5], [1.0, 1.25]])


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_r21_hand_case_masked_uses_cache_of_its_step(mode):
    """The masked run of the same block with token 0 active: row 0 as in the dense hand case,
    rows U = {1, 2} take the cache entry of THAT step (cache[s], reading R7):
      x1[1] = [3,4] - 0.5 [10,10] = [-2,-1]     x2[1] = x1[1] - 0.25 [8,8]  = [-4,-3]
      x1[2] = [5,6] - 0.5 [11,11] = [-.5,.5]    x2[2] = x1[2] - 0.25 [1,-1] = [-.75,.75]"""
    W = [_zero_block(2, [1, 0], [0, 2])]
    mods = [[_mod(1.0, 1.0), _mod(2.0, 0.5)]]
    deltas = [-0.5, -0.25]
    x0 = np.array([[1, 2], [3, 4], [5, 6]], float)
    Y = [np.array([[9, 9], [10, 10], [11, 11]], float), np.array([[7, 7], [8, 8], [1, -1]], float)]
    rnd = np.random.default_rng(0)
    cache = [[{"K": rnd.normal(size=(3, 2)), "V": rnd.normal(size=(3, 2)), "Y": Y[s]}]
             for s in range(2)]
    mask = np.array([1, 0, 0], np.uint8)
    x2 = S.masked_run(x0, mask, W, mods, deltas, [1], mode, cache, 1, 2)
    assert np.array_equal(x2, [[-0.5, -0.25], [-4, -3], [-0.75, 0.75]])


def test_flow_sigmas_closed_forms():
    """R29 schedule: linear at shift 1; hand values at S = 4, shift 3 (t = 1, .75, .5, .25 ->
    3t / (1 + 2t) = 1, .9, .75, .5, then 0); endpoints, monotone; Flux's shift e^1.15."""
    assert np.allclose(SM.flow_sigmas(5, 1.0), [1, 0.8, 0.6, 0.4, 0.2, 0], atol=1e-15)
    assert np.allclose(SM.flow_sigmas(4, 3.0), [1, 0.9, 0.75, 0.5, 0], atol=1e-15)
    s = SM.flow_sigmas(28, SM.FLUX_SHIFT)
    assert s[0] == 1.0 and s[-1] == 0.0 and len(s) == 29 and np.all(np.diff(s) < 0)
    assert SM.FLUX_SHIFT == pytest.approx(3.1581929, rel=1e-7)


@pytest.mark.parametrize("shift", [1.0, 3.0])
def test_flow_euler_integrates_the_straight_path_exactly(shift):
    """Every row masked and a constant velocity y = eps - z (the exact flow from the template
    latent z to the noise eps): Euler from x_0 = eps follows x_s = (1 - sigma_s) z + sigma_s eps
    at every step and ends at z -- pins the sign of (sigma_{s+1} - sigma_s) and its step index."""
    g = np.random.default_rng(1)
    z, eps = g.normal(size=(6, 3)), g.normal(size=(6, 3))
    sig = SM.flow_sigmas(7, shift)
    x = eps.copy()
    for s in range(7):
        x = SM.flow_blend_update(x, eps - z, np.ones(6, np.uint8), z, eps, sig[s], sig[s + 1], 6)
        assert np.allclose(x, (1 - sig[s + 1]) * z + sig[s + 1] * eps, atol=1e-13)
    assert np.allclose(x, z, atol=1e-13)


def test_flow_blend_rows_hand_case():
    """L_img = 2 image rows (row 0 masked, row 1 not) and one text row, sigma 0.8 -> 0.5:
      masked row   x + (0.5 - 0.8) y       = [1,1] - 0.3 [2,4]          = [0.4, -0.2]
      unmasked row 0.5 z + 0.5 eps         = 0.5 [4,6] + 0.5 [2,0]      = [3, 3]   (y ignored)
      text row     unchanged                                           = [7, 8]"""
    x = np.array([[1, 1], [9, 9], [7, 8]], float)
    y = np.array([[2, 4], [100, -100], [5, 5]], float)
    z = np.array([[0, 0], [4, 6]], float)
    eps = np.array([[0, 0], [2, 0]], float)
    out = SM.flow_blend_update(x, y, np.array([1, 0, 1], np.uint8), z, eps, 0.8, 0.5, 2)
    assert np.allclose(out, [[0.4, -0.2], [3, 3], [7, 8]], atol=1e-15)


def test_flow_blend_unmasked_region_ends_at_the_template():
    """Whatever the stack computes, after the last step (sigma_S = 0) every unmasked image row
    of a masked run equals the template latent z, and the text rows are the prompt rows."""
    g = synth.rng(5)
    H, L_img, L_txt, N, steps = 16, 16, 2, 2, 3
    W = synth.stack_weights(g, N, H, 32, "f32")
    mods = synth.mod_table(g, N, steps, H, "f32")
    z, eps = synth.latent(g, L_img, H, "f32"), synth.latent(g, L_img, H, "f32")
    txt = synth.latent(g, L_txt, H, "f32")
    sig = SM.flow_sigmas(steps, 3.0)
    samp = {"sigmas": sig, "z": z, "eps": eps}
    x0 = SM.flow_init(z, eps, sig[0], txt)
    cache, _ = S.template_run(x0, W, mods, synth.delta_table(steps), 2, steps, L_txt=L_txt,
                              sampler=samp)
    mask = synth.token_mask(synth.mask_blobs(g, 4, 4, 0.3), L_txt)
    x = S.masked_run(x0, mask, W, mods, None, [1] * N, "kv", cache, 2, steps, L_txt=L_txt,
                     sampler=samp)
    U = np.flatnonzero(mask[:L_img] == 0)
    assert np.array_equal(x[U], z[U])
    assert np.array_equal(x[L_img:], txt)
    # the template run itself (nothing masked) reconstructs z exactly on every image row
    _, xs = S.template_run(x0, W, mods, None, 2, steps, L_txt=L_txt, sampler=samp)
    assert np.array_equal(xs[-1][:L_img], z)


def test_flow_blend_identical_input_invariant():
    """L144/L157 under the flow-blend sampler: a request identical to the template run (its
    cache) reproduces the template trajectory for every feasible KV plan -- the sampler keeps
    the masked rows' dependence on the stack and the invariant of the R21 update."""
    g = synth.rng(9)
    H, L_img, L_txt, N, steps = 16, 16, 2, 3, 2
    W = synth.stack_weights(g, N, H, 32, "f32")
    mods = synth.mod_table(g, N, steps, H, "f32")
    z, eps = synth.latent(g, L_img, H, "f32"), synth.latent(g, L_img, H, "f32")
    sig = SM.flow_sigmas(steps, SM.FLUX_SHIFT)
    samp = {"sigmas": sig, "z": z, "eps": eps}
    x0 = SM.flow_init(z, eps, sig[0], synth.latent(g, L_txt, H, "f32"))
    mask = synth.token_mask(synth.mask_blobs(g, 4, 4, 0.4), L_txt)
    # the "template" here is a dense run of the same request (same mask in the blend)
    x, cache = np.array(x0), []
    for s in range(steps):
        cur, ent = x, []
        for l, w in enumerate(W):
            y, K, V = S.dense_block(cur, w, mods[l][s], 2)
            ent.append({"K": K, "V": V, "Y": y})
            cur = y
        cache.append(ent)
        x = SM.flow_blend_update(x, cur, mask, z, eps, sig[s], sig[s + 1], L_img)
    for plan in ([1, 1, 1], [0, 1, 1], [0, 0, 0]):
        got = S.masked_run(x0, mask, W, mods, None, plan, "kv", cache, 2, steps, L_txt=L_txt,
                           sampler=samp)
        assert np.allclose(got, x, rtol=0, atol=1e-11), plan
