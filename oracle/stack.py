"""a3 / a9 / a10 data flow over a stack of N blocks and S denoising steps (oracle; tests only).

PAPER.md L203-L207 (§4.2): activations are cached "at the granularity of transformer blocks";
L211 (§4.2, Fig. 9-Bottom): blocks that do not use cached activations "compute all tokens --
both masked and unmasked"; L157: unmasked output rows are "replenished" from the cache;
L230 (§4.3): iterative denoising, so a cache entry is keyed (template, step, block) (R7).

Readings used here: R4 (Y = block output), R6 (Y-mode block 0 takes rows U from
the fresh stack input), R11 (KV-mode plans are monotone: uncached prefix, cached suffix),
R12 (`use_cache` is an explicit input), the synthetic sampler update x <- x + delta_s * y over
the full latent (R21), and the KV-mode final replenish from the cached final-block Y (R22).
"""
from __future__ import annotations

import numpy as np

from .block import dense_block, f64, masked_block_kv, masked_block_y
from .index import build_mask_index, gather_rows, scatter_rows
from .sampler import flow_blend_update


def template_run(x0, weights, mods, deltas, heads, steps, ctx=None, L_txt=0, sampler=None):
    """Full (dense) inference of the template: the producer of the activation cache (L130,
    L203). mods[l][s] is block l's adaLN vector at step s.

    ctx: the request's prompt encoding (SDXL blocks only); L_txt: text rows (double-stream).
    sampler: None = the synthetic update (R21); {"sigmas", "z", "eps"} = the flow-blend sampler
    (R29) with no image row masked, i.e. the template's own latent re-noised along the schedule.
    Returns (cache, xs): cache[s][l] = {"K", "V", "Y"} full-L arrays; xs[s] = latent entering
    step s (xs[steps] = final latent)."""
    x = f64(x0)
    cache, xs = [], []
    for s in range(steps):
        xs.append(x)
        cur = x
        entries = []
        for l, w in enumerate(weights):
            y, K, V = dense_block(cur, w, mods[l][s], heads, ctx, L_txt)
            entries.append({"K": K, "V": V, "Y": y})
            cur = y
        cache.append(entries)
        if sampler is None:
            x = x + float(deltas[s]) * cur
        else:
            L = x.shape[0]
            x = flow_blend_update(x, cur, np.zeros(L, np.uint8), sampler["z"], sampler["eps"],
                                  sampler["sigmas"][s], sampler["sigmas"][s + 1], L - L_txt)
    xs.append(x)
    return cache, xs


def check_plan(use_cache, mode):
    """KV-mode needs an uncached prefix then a cached suffix (R11): an uncached block after a
    cached one would need x[U], which KV-mode never materialises."""
    if mode == "kv":
        seen = False
        for u in use_cache:
            if u:
                seen = True
            elif seen:
                raise ValueError("KV-mode plan must be monotone (0..0 1..1)")


def masked_stack(x, mask, weights, mods_s, use_cache, mode, cache_s, heads, ctx=None, L_txt=0):
    """One denoising step's block stack for one request (a2-a9).

    x: full latent [L, H] entering the step; mask: [L] (text rows set); mods_s[l]: block l's
    adaLN vector at this step; cache_s[l] = {"K","V","Y"} of the template run at this step.
    Returns the full output y [L, H]: rows M computed, rows U replenished from the cache."""
    check_plan(use_cache, mode)
    M, U = build_mask_index(mask)
    L = len(mask)
    N = len(weights)
    rep, cur, act = "full", f64(x), None
    for l in range(N):
        if not use_cache[l]:
            if rep == "act":                      # Y-mode only: rebuild the full input (R11)
                full = np.empty_like(cur)
                scatter_rows(act, M, full)
                scatter_rows(gather_rows(cache_s[l - 1]["Y"], U), U, full)
                cur = full
            cur, _, _ = dense_block(cur, weights[l], mods_s[l], heads, ctx, L_txt)   # L211: all tokens
            rep = "full"
            continue
        if rep == "full":
            act = gather_rows(cur, M)                                     # a2
            x_U = gather_rows(cur, U)                                     # R6 (Y-mode input)
        else:
            x_U = gather_rows(cache_s[l - 1]["Y"], U) if mode == "y" else None
        if mode == "kv":
            act, _, _ = masked_block_kv(act, M, U, gather_rows(cache_s[l]["K"], U),
                                        gather_rows(cache_s[l]["V"], U), weights[l],
                                        mods_s[l], heads, L, ctx, L_txt)
        else:
            act = masked_block_y(act, M, U, x_U, weights[l], mods_s[l], heads, L, ctx, L_txt)
        rep = "act"
    if rep == "full":
        return cur
    y = np.empty_like(f64(x))
    scatter_rows(act, M, y)                                               # a9
    scatter_rows(gather_rows(cache_s[N - 1]["Y"], U), U, y)               # replenish (L157)
    return y


def euler_update(x, y, delta):
    """Synthetic sampler update over the full latent (R21): x <- x + delta * y."""
    return f64(x) + float(delta) * f64(y)


def masked_run(x0, mask, weights, mods, deltas, use_cache, mode, cache, heads, steps,
               step0=0, ctx=None, L_txt=0, sampler=None):
    """Steps step0..step0+steps-1 of one request against the template cache.  sampler: None =
    the synthetic update (R21), or {"sigmas", "z", "eps"} for the flow-blend sampler (R29)."""
    x = f64(x0)
    for s in range(step0, step0 + steps):
        mods_s = [mods[l][s] for l in range(len(weights))]
        y = masked_stack(x, mask, weights, mods_s, use_cache, mode, cache[s], heads, ctx, L_txt)
        if sampler is None:
            x = euler_update(x, y, deltas[s])
        else:
            x = flow_blend_update(x, y, mask, sampler["z"], sampler["eps"], sampler["sigmas"][s],
                                  sampler["sigmas"][s + 1], len(mask) - L_txt)
    return x
