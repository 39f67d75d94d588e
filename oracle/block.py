"""a4-a8: the transformer block, dense and mask-aware (oracle; test infrastructure only).

Block definition (§3.1 "Mask-aware attention", Fig. 5; L134-L138 token-wise
LayerNorm/GeLU/dropout; Table 1 "(XW1)W2" feed-forward with W1 in R^{H x 4H}):

    h1 = LN(x)(1 + scale1) + shift1                       LN eps 1e-6, no affine   (R3, R2)
    Q, K, V = h1 Wq^T + bq, h1 Wk^T + bk, h1 Wv^T + bv    split into `heads` heads  (R1)
    A_j = softmax(Q_j K_j^T / sqrt(d)) V_j                per head j, d = H/heads   (R1)
    x1 = x + gate1 * (concat_j A_j  Wo^T + bo)
    h2 = LN(x1)(1 + scale2) + shift2
    y  = x1 + gate2 * (GELU_tanh(h2 W1^T + b1) W2^T + b2)                          (R3)

Weights use the nn.Linear layout W[out, in]; w_qkv stacks Wq, Wk, Wv as rows [0,H),[H,2H),[2H,3H).
`mod` is the per-request adaLN vector [6H] = (shift1, scale1, gate1, shift2, scale2, gate2);
the identity modulation (0, 0, 1, 0, 0, 1) gives plain pre-LN + residual.

Mask-aware block (L157 §3.1, Fig. 5-Bottom; L161 Fig. 7): given the ascending active ids M and
unmasked ids U of one request (index.build_mask_index),
  * KV-mode (Fig. 7): compute Q, K, V for rows M only; keys/values of rows U are the
    cached K[U], V[U] of the template run; attention uses Q_M against the merged key set in
    original token order (R10); the rest of the block runs on rows M only.
  * Y-mode (Fig. 5-Bottom): the block input on rows U is the cached previous-block output
    Y (R4); K, V are projected over all L rows; Q, O-projection and MLP on rows M only.
Everything is float64.

Parallel block variant (NEXT-2, weights["kind"] == "par"; reading R23): the Flux single-stream
block, where attention and MLP read the same normalised input and share one input and one
output projection (Flux is a stack of such transformer blocks, L79 / L92 footnote):

    h  = LN(x)(1 + scale1) + shift1
    [Q | K | V | Z] = h W1^T + b1                         W1 in R^{(3H+F) x H}
    y  = x + gate1 * ([A | GELU_tanh(Z)] W2^T + b2)       A = concat_j A_j, W2 in R^{H x (H+F)}

Only (shift1, scale1, gate1) of `mod` are used.  Its FLOPs per row equal the sequential block's
(12 H^2 multiply-adds with F = 4H), and the same masked modes apply: Z is token-wise (rows M
only), K/V follow KV- or Y-mode exactly as above.

SDXL block variant (NEXT-2, weights["kind"] == "sdxl"; reading R24): the UNet transformer
block of the SDXL model the paper evaluates (L65, L305), i.e. self-attention, cross-attention
to the request's prompt encoding ctx [L_ctx, D_ctx], and a GEGLU feed-forward, each pre-norm
with an affine LayerNorm (gamma, beta) and an ungated residual; `mod` is not used:

    h1 = LN(x) g1 + b1 ;  Q, K, V = h1 Wqkv^T (+ b) ;  x1 = x + (A(Q, K, V) Wo^T + bo)
    h2 = LN(x1) g2 + b2 ; Q2 = h2 Wq2^T (+ bq2) ; [Kc | Vc] = ctx Wkv2^T (+ bkv2)
                          x2 = x1 + (A(Q2, Kc, Vc) Wo2^T + bo2)
    h3 = LN(x2) g3 + b3 ; [P | G] = h3 Wup^T + bup      Wup in R^{2F x H}: rows [0,F) -> P,
                          y  = x2 + ((P * GELU_tanh(G)) Wdown^T + bdown)    rows [F,2F) -> G

Cross-attention and GEGLU are token-wise in the latent (each row's output depends only on that
row and ctx), so on a masked block they run on rows M only; the self-attention's K/V follow
KV- or Y-mode exactly as for the sequential block.

Double-stream block variant (NEXT-2, weights["kind"] == "double"; reading R25): Flux's
MM-DiT block, where image rows [0, L_img) and text rows [L_img, L) keep their own weights
(w["img"], w["txt"], each a sequential block's set) and adaLN vectors (mod [12H] = image 6H,
then text 6H) and meet only in one joint attention over all L rows:

    per stream s of the row:  h1 = LN(x)(1 + scale1_s) + shift1_s ;  Q, K, V = h1 W_s^T + b_s
    A = softmax(Q K^T / sqrt(d)) V over all rows (joint)
    per stream:  x1 = x + gate1_s (A Wo_s^T + bo_s) ;  y = x1 + gate2_s MLP_s(LN(x1)(1+scale2_s)+shift2_s)

Text rows are always active (R9), so a masked block has fresh text rows and cached image rows U.
"""
from __future__ import annotations

import math

import numpy as np

LN_EPS = 1e-6


def f64(a):
    return np.asarray(a, dtype=np.float64)


def layer_norm(x, eps=LN_EPS):
    """Row-wise LayerNorm without affine (L134 token-wise; R3)."""
    x = f64(x)
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps)


def layer_norm_affine(x, gamma, beta):
    """LayerNorm with per-channel affine (the SDXL block's norms, R24): LN(x) * gamma + beta."""
    return layer_norm(x) * f64(gamma) + f64(beta)


def gelu_tanh(x):
    """GELU, tanh approximation (L134 "GeLU activation"; R3)."""
    x = f64(x)
    return 0.5 * x * (1.0 + np.tanh(math.sqrt(2.0 / math.pi) * (x + 0.044715 * x ** 3)))


def split_mod(mod, H):
    mod = f64(mod).reshape(6, H)
    return mod[0], mod[1], mod[2], mod[3], mod[4], mod[5]


def identity_mod(H):
    m = np.zeros((6, H))
    m[2] = 1.0
    m[5] = 1.0
    return m.reshape(-1)


def linear(h, W, b):
    """h W^T + b (L146 "a linear projection maps X into Q, K, V")."""
    out = f64(h) @ f64(W).T
    if b is not None:
        out = out + f64(b)
    return out


def softmax_rows(s):
    s = f64(s)
    s = s - s.max(axis=-1, keepdims=True)
    e = np.exp(s)
    return e / e.sum(axis=-1, keepdims=True)


def attention(Q, K, V, heads):
    """Per head j: softmax(Q_j K_j^T / sqrt(d)) V_j  (L146; scale 1/sqrt(d), reading R1).

    Q: [n, H] rows of queries; K, V: [Lk, H]. Returns [n, H] = concat_j A_j.
    """
    Q, K, V = f64(Q), f64(K), f64(V)
    n, H = Q.shape
    d = H // heads
    out = np.empty((n, H))
    for j in range(heads):
        sl = slice(j * d, (j + 1) * d)
        S = Q[:, sl] @ K[:, sl].T / math.sqrt(d)
        out[:, sl] = softmax_rows(S) @ V[:, sl]
    return out


def is_parallel(w):
    return w.get("kind", "seq") == "par"


def is_sdxl(w):
    return w.get("kind", "seq") == "sdxl"


def is_double(w):
    return w.get("kind", "seq") == "double"


def _per_stream(f, ids, L_img, mod, H):
    """Row-wise op of the double-stream block (R25): f(stream weights key, stream mod [6H])
    evaluated for both streams, each row taking its own stream's result (ids >= L_img: text)."""
    mod = f64(mod).reshape(-1)
    img, txt = f("img", mod[:6 * H]), f("txt", mod[6 * H:])
    return np.where((np.asarray(ids) >= L_img)[:, None], txt, img)


def _double_block(x_rows, ids, w, mod, heads, L_img, K_U=None, V_U=None, U=None, x_U=None,
                  L=None):
    """Double-stream block on rows `ids` (ascending) of one request.  Dense: ids = all rows.
    KV-mode: K_U / V_U cached at rows U.  Y-mode: x_U = cached input rows U.  Returns (y, K, V)
    over the rows `ids`."""
    x_rows = f64(x_rows)
    H = x_rows.shape[1]
    ln1 = lambda xr: (lambda s, m: layer_norm(xr) * (1.0 + split_mod(m, H)[1]) + split_mod(m, H)[0])
    proj = lambda hr, j: (lambda s, m: linear(hr, *_qkv_weights(w[s], H)[j]))
    h1 = _per_stream(ln1(x_rows), ids, L_img, mod, H)
    Q, K, V = (_per_stream(proj(h1, j), ids, L_img, mod, H) for j in range(3))
    if U is None or len(U) == 0:
        Kall, Vall = K, V
    else:
        L = L if L is not None else len(ids) + len(U)
        Kall, Vall = np.empty((L, H)), np.empty((L, H))
        Kall[ids], Vall[ids] = K, V
        if x_U is None:                                            # KV-mode: cached K/V rows U
            Kall[U], Vall[U] = f64(K_U), f64(V_U)
        else:                                                      # Y-mode: project x[U]
            hU = _per_stream(ln1(f64(x_U)), U, L_img, mod, H)
            Kall[U] = _per_stream(proj(hU, 1), U, L_img, mod, H)
            Vall[U] = _per_stream(proj(hU, 2), U, L_img, mod, H)
    a = attention(Q, Kall, Vall, heads)
    y = _per_stream(lambda s, m: _attn_out_and_mlp(x_rows, a, w[s], m, H), ids, L_img, mod, H)
    return y, K, V


def geglu(h, W, b):
    """GEGLU feed-forward input (R24): [P | G] = h W^T + b with P the first F output rows of W,
    G the last F; returns P * GELU_tanh(G)."""
    pg = linear(h, W, b)
    F = pg.shape[1] // 2
    return pg[:, :F] * gelu_tanh(pg[:, F:])


def context_kv(ctx, w):
    """Cross-attention keys / values of the prompt encoding: ctx Wkv2^T + bkv2 -> (Kc, Vc)."""
    kv = linear(ctx, w["w_kv2"], w.get("b_kv2"))
    H = kv.shape[1] // 2
    return kv[:, :H], kv[:, H:]


def _norm1(x, w, mod, H):
    """The block's first normalised input: affine LN (SDXL) or adaLN-modulated LN."""
    if is_sdxl(w):
        return layer_norm_affine(x, w["ln1_w"], w["ln1_b"])
    sh1, sc1, _, _, _, _ = split_mod(mod, H)
    return layer_norm(x) * (1.0 + sc1) + sh1


def _sdxl_out(x_rows, a_rows, w, ctx, heads):
    """SDXL block after the self-attention, on the given rows (all token-wise in the latent)."""
    x1 = f64(x_rows) + linear(a_rows, w["w_o"], w.get("b_o"))
    h2 = layer_norm_affine(x1, w["ln2_w"], w["ln2_b"])
    Kc, Vc = context_kv(ctx, w)
    a2 = attention(linear(h2, w["w_q2"], w.get("b_q2")), Kc, Vc, heads)
    x2 = x1 + linear(a2, w["w_o2"], w.get("b_o2"))
    h3 = layer_norm_affine(x2, w["ln3_w"], w["ln3_b"])
    return x2 + linear(geglu(h3, w["w_up"], w.get("b_up")), w["w_down"], w.get("b_down"))


def _qkv_weights(w, H):
    if is_parallel(w):
        W, b = f64(w["w_1"]), f64(w["b_1"])
    else:
        W = f64(w["w_qkv"])
        b = f64(w["b_qkv"]) if w.get("b_qkv") is not None else np.zeros(3 * H)
    return (W[0:H], b[0:H]), (W[H:2 * H], b[H:2 * H]), (W[2 * H:3 * H], b[2 * H:3 * H])


def _block_out(x_rows, h_rows, a_rows, w, mod, H, ctx=None, heads=None):
    """The block output on the given rows from their input x, normalised input h and attention
    output A: the sequential block's O projection + MLP, the parallel block's fused output, or
    the SDXL block's O projection + cross-attention + GEGLU."""
    if is_sdxl(w):
        return _sdxl_out(x_rows, a_rows, w, ctx, heads)
    if not is_parallel(w):
        return _attn_out_and_mlp(x_rows, a_rows, w, mod, H)
    _, _, g1, _, _, _ = split_mod(mod, H)
    W1, b1 = f64(w["w_1"]), f64(w["b_1"])
    z = gelu_tanh(linear(h_rows, W1[3 * H:], b1[3 * H:]))          # MLP branch, token-wise
    cat = np.concatenate([f64(a_rows), z], axis=1)                  # [A | GELU(Z)]
    return f64(x_rows) + g1 * linear(cat, w["w_2"], w["b_2"])


def _attn_out_and_mlp(x_rows, a_rows, w, mod, H):
    """x1 = x + gate1 (A Wo^T + bo);  y = x1 + gate2 (GELU(h2 W1^T + b1) W2^T + b2)."""
    _, _, g1, sh2, sc2, g2 = split_mod(mod, H)
    x1 = f64(x_rows) + g1 * linear(a_rows, w["w_o"], w["b_o"])
    h2 = layer_norm(x1) * (1.0 + sc2) + sh2
    y = x1 + g2 * linear(gelu_tanh(linear(h2, w["w_up"], w["b_up"])), w["w_down"], w["b_down"])
    return y


def dense_block(x, w, mod, heads, ctx=None, L_txt=0):
    """Standard block over all L tokens (Fig. 5-Top). Returns (y, K, V).
    ctx: the request's prompt encoding [L_ctx, D_ctx] (SDXL block only); L_txt: text rows at
    the end of x (double-stream block only)."""
    x = f64(x)
    H = x.shape[1]
    if is_double(w):
        L = x.shape[0]
        return _double_block(x, np.arange(L), w, mod, heads, L - L_txt)
    h1 = _norm1(x, w, mod, H)
    (Wq, bq), (Wk, bk), (Wv, bv) = _qkv_weights(w, H)
    Q, K, V = linear(h1, Wq, bq), linear(h1, Wk, bk), linear(h1, Wv, bv)
    a = attention(Q, K, V, heads)
    return _block_out(x, h1, a, w, mod, H, ctx, heads), K, V


def masked_block_kv(x_M, M, U, K_U, V_U, w, mod, heads, L, ctx=None, L_txt=0):
    """KV-cache mode (Fig. 7): fresh Q/K/V on rows M, cached K/V on rows U.

    x_M: [n, H] block input rows M (ascending ids M). K_U, V_U: [u, H] cached keys/values of the
    template run at rows U. Returns (y_M, K_M, V_M).
    """
    if is_double(w):
        return _double_block(x_M, M, w, mod, heads, L - L_txt, K_U, V_U, U, L=L)
    x_M = f64(x_M)
    H = x_M.shape[1]
    h1_M = _norm1(x_M, w, mod, H)                              # token-wise (L134, L144)
    (Wq, bq), (Wk, bk), (Wv, bv) = _qkv_weights(w, H)
    Q_M, K_M, V_M = linear(h1_M, Wq, bq), linear(h1_M, Wk, bk), linear(h1_M, Wv, bv)
    # merged key set in original token order (R10): fresh rows M, cached rows U
    K_all = np.empty((L, H))
    V_all = np.empty((L, H))
    K_all[M], V_all[M] = K_M, V_M
    K_all[U], V_all[U] = f64(K_U), f64(V_U)
    a_M = attention(Q_M, K_all, V_all, heads)                  # queries from masked rows only (L159)
    return _block_out(x_M, h1_M, a_M, w, mod, H, ctx, heads), K_M, V_M


def masked_block_y(x_M, M, U, x_U, w, mod, heads, L, ctx=None, L_txt=0):
    """Y-cache mode (Fig. 5-Bottom): block input rows U are the cached activations Y of
    the previous block (R4); K/V over all L rows; Q, O and MLP on rows M. Returns y_M."""
    if is_double(w):
        return _double_block(x_M, M, w, mod, heads, L - L_txt, U=U, x_U=x_U, L=L)[0]
    x_M = f64(x_M)
    H = x_M.shape[1]
    x_full = np.empty((L, H))
    x_full[M] = x_M
    x_full[U] = f64(x_U)
    h1 = _norm1(x_full, w, mod, H)
    (Wq, bq), (Wk, bk), (Wv, bv) = _qkv_weights(w, H)
    Q_M = linear(h1[M], Wq, bq)
    K, V = linear(h1, Wk, bk), linear(h1, Wv, bv)
    a_M = attention(Q_M, K, V, heads)
    return _block_out(x_M, h1[M], a_M, w, mod, H, ctx, heads)
