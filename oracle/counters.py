"""Table 1 (§3.2): FLOPs and cache bytes per block (oracle; tests only).

Table 1 gives orders: FFN O(BmLH^2), linear projection O(BmLH^2), QK^T O(BmL^2H), cache shape
(B, (1-m)L, H). These are the exact per-mode counts for the block in oracle/block.py
(a multiply-add = 2 FLOPs; n = active rows, u = L - n cached rows, F = MLP width):

  dense : QKV 6LH^2 + O 2LH^2 + MLP 4LHF              + attention 4L^2H
  KV    : QKV 6nH^2 + O 2nH^2 + MLP 4nHF              + attention 4nLH
  Y     : Q 2nH^2 + KV 4LH^2 + O 2nH^2 + MLP 4nHF     + attention 4nLH   (R5)
Cache bytes loaded per block: KV 2*u*H*elt (K and V), Y 1*u*H*elt (Table 1 cache shape).

SDXL block (R24) adds, per row that runs the token-wise part (n, or L when dense): the
cross-attention Q and output projections 4H^2, its attention over Lc prompt tokens 4LcH, and
the GEGLU's doubled input projection 2HF (4HF -> 6HF for the feed-forward).  The prompt's K|V
projection, 4 Lc D_ctx H, is per request and admission, not per step (context_flops).
"""
from __future__ import annotations


def block_flops(mode, n, L, H, F, kind="seq", Lc=0):
    """FLOPs of one block for one request with n active rows out of L (Lc prompt tokens for
    the SDXL block's cross-attention)."""
    attn = 4 * n * L * H
    rows = L if mode == "dense" else n
    extra = rows * (4 * H * H + 4 * Lc * H + 2 * H * F) if kind == "sdxl" else 0
    if mode == "dense":
        return 6 * L * H * H + 2 * L * H * H + 4 * L * H * F + 4 * L * L * H + extra
    if mode == "kv":
        return 6 * n * H * H + 2 * n * H * H + 4 * n * H * F + attn + extra
    if mode == "y":
        return 2 * n * H * H + 4 * L * H * H + 2 * n * H * H + 4 * n * H * F + attn + extra
    raise ValueError(mode)


def context_flops(Lc, D_ctx, H):
    """SDXL block: the prompt's cross-attention K|V projection, once per request."""
    return 4 * Lc * D_ctx * H


def gemm_flops(mode, n, L, H, F):
    """The dense-contraction part only (projections + MLP), i.e. block_flops minus attention."""
    if mode == "dense":
        return block_flops("dense", L, L, H, F) - 4 * L * L * H
    return block_flops(mode, n, L, H, F) - 4 * n * L * H


def cache_bytes(mode, u, H, elt=2):
    """Bytes of cached activations one block loads for one request (Table 1 cache shape)."""
    if mode == "kv":
        return 2 * u * H * elt
    if mode == "y":
        return u * H * elt
    if mode == "dense":
        return 0
    raise ValueError(mode)
