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
