"""Pins for oracle/index.py (a1, a2, a9): hand-derived golden case, library routine, invariants."""
import os

import numpy as np

import synth
from oracle.index import build_mask_index, gather_rows, scatter_rows


def _golden():
    path = os.path.join(os.path.dirname(__file__), "golden", "mask_index_tiny.txt")
    rows = [l.split() for l in open(path) if l.strip() and not l.startswith("#")]
    return [np.array(list(map(int, r))) for r in rows]


def test_golden_tiny():
    mask, m_ids, u_ids = _golden()
    M, U = build_mask_index(mask)
    assert M.tolist() == m_ids.tolist()
    assert U.tolist() == u_ids.tolist()


def test_vs_flatnonzero_and_invariants():
    g = synth.rng(7)
    for L in (1, 2, 31, 32, 33, 256, 1000, 4608):
        for m in (0.0, 0.05, 0.2, 0.6, 1.0):
            mask = synth.mask_random(g, L, m)
            M, U = build_mask_index(mask)
            assert M.tolist() == np.flatnonzero(mask).tolist()       # library routine
            assert U.tolist() == np.flatnonzero(mask == 0).tolist()
            assert len(M) == int(mask.sum())                          # n = popcount
            assert len(np.intersect1d(M, U)) == 0                     # disjoint
            assert sorted(M.tolist() + U.tolist()) == list(range(L))  # union = [0, L)
            assert np.all(np.diff(M) > 0) and np.all(np.diff(U) > 0)  # ascending


def test_exact_count_masks():
    g = synth.rng(3)
    for m in (0.05, 0.1, 0.2, 0.35, 0.6):
        assert synth.mask_random(g, 4096, m).sum() == synth.n_masked_for(m, 4096)
        assert synth.mask_blobs(g, 64, 64, m).sum() == synth.n_masked_for(m, 4096)


def test_gather_scatter_roundtrip_bit_exact():
    g = synth.rng(11)
    x = synth.latent(g, 300, 40, "bf16")
    mask = synth.mask_blobs(g, 15, 20, 0.3)
    M, U = build_mask_index(mask)
    xm, xu = gather_rows(x, M), gather_rows(x, U)
    assert np.array_equal(xm, x[M]) and np.array_equal(xu, x[U])     # numpy fancy indexing
    out = np.full_like(x, np.nan)
    scatter_rows(xm, M, out)
    scatter_rows(xu, U, out)
    assert np.array_equal(out.view(np.uint32), x.view(np.uint32))    # identity, bit-exact


# ---- NEXT-4: pixel mask -> token mask (reading R8) -------------------------------------------
from oracle.index import pixel_to_token_mask


def test_pixel_to_token_golden():
    # hand-derived: 4 x 6 pixels, f = 2 -> 2 x 3 tokens; pixels set at (0,0), (3,5), (2,2)
    pix = np.zeros((4, 6), np.uint8)
    pix[0, 0] = pix[3, 5] = pix[2, 2] = 1
    # token (0,0) covers rows 0-1 cols 0-1 -> 1; (1,2) covers rows 2-3 cols 4-5 -> 1;
    # (1,1) covers rows 2-3 cols 2-3 -> 1; all others 0; then 2 text tokens
    assert pixel_to_token_mask(pix, 2, 2).tolist() == [1, 0, 0, 0, 1, 1, 1, 1]


def test_pixel_to_token_vs_reshape_max_and_identities():
    g = synth.rng(21)
    for (Hp, Wp, f) in ((32, 48, 4), (30, 45, 3), (64, 64, 16), (16, 16, 1), (40, 8, 8)):
        pix = (g.random((Hp, Wp)) < 0.02).astype(np.uint8)
        tok = pixel_to_token_mask(pix, f, 3)
        ref = pix.reshape(Hp // f, f, Wp // f, f).max(axis=(1, 3)).reshape(-1)  # library max-pool
        assert tok[:-3].tolist() == (ref != 0).astype(np.uint8).tolist()
        assert tok[-3:].tolist() == [1, 1, 1]
        if f == 1:
            assert tok[:-3].tolist() == (pix.reshape(-1) != 0).tolist()       # identity
    # monotone: adding masked pixels never clears a token; empty / full masks
    pix = np.zeros((64, 64), np.uint8)
    assert pixel_to_token_mask(pix, 16).sum() == 0
    assert pixel_to_token_mask(pix + 1, 16).sum() == 16
    pix[5, 7] = 1
    a = pixel_to_token_mask(pix, 16)
    pix[40, 60] = 1
    b = pixel_to_token_mask(pix, 16)
    assert np.all(b >= a) and a.sum() == 1 and b.sum() == 2
