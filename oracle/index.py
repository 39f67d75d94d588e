"""a1 / a2 / a9: token categorisation and row selection (oracle; test infrastructure only).

PAPER.md L130 (§3.1): "Leveraging the mask, we can categorize the tokens as masked tokens and
unmasked tokens". L157 (§3.1, Fig. 5-Bottom): "extract the matrix of masked tokens ... while
replenishing cached activations for the unmasked tokens".
"""
from __future__ import annotations

import numpy as np


def build_mask_index(mask):
    """Return (masked_ids, unmasked_ids): ascending token ids with mask != 0 / == 0.

    Plain loop in token order (L130). Text tokens are expected to be set active by the caller
    (reading R9).
    """
    masked, unmasked = [], []
    for t in range(len(mask)):
        if mask[t]:
            masked.append(t)
        else:
            unmasked.append(t)
    return np.array(masked, dtype=np.int32), np.array(unmasked, dtype=np.int32)


def gather_rows(x, ids):
    """x_M = rows of x at ids, in ids order (L157 "extract the matrix of masked tokens")."""
    out = np.empty((len(ids),) + x.shape[1:], dtype=x.dtype)
    for i, t in enumerate(ids):
        out[i] = x[t]
    return out


def scatter_rows(rows, ids, out):
    """out[ids[i]] = rows[i] (L157 "replenishing" / writing back). Returns out."""
    for i, t in enumerate(ids):
        out[t] = rows[i]
    return out


def pixel_to_token_mask(pix, f, L_txt=0):
    """Pixel-level editing mask -> token mask (NEXT-4; reading R8 of DESIGN.md).

    PAPER.md L79 (§2.1): "a latent of shape (B, C, H, W) is reshaped to (B, H x W, C)", i.e. one
    token per latent position; a token covers an f x f block of mask pixels (VAE down-sampling
    x patchify; f = 16 for Flux-scale 1024^2 -> 64 x 64 tokens, 16 / 32 for the SDXL-scale 64^2 /
    32^2 levels).  Reading R8: the token is masked iff ANY covered pixel is masked (so every
    edited pixel is regenerated).  Text tokens (reading R9) are appended, always active.
    pix: 2-D array [Hp, Wp], nonzero = masked; Hp, Wp multiples of f.  Returns uint8 [T + L_txt].
    """
    Hp, Wp = pix.shape
    Ht, Wt = Hp // f, Wp // f
    out = np.zeros(Ht * Wt + L_txt, dtype=np.uint8)
    for i in range(Ht):
        for j in range(Wt):
            hit = 0
            for y in range(i * f, (i + 1) * f):
                for x in range(j * f, (j + 1) * f):
                    if pix[y, x]:
                        hit = 1
                        break
                if hit:
                    break
            out[i * Wt + j] = hit
    out[Ht * Wt:] = 1
    return out
