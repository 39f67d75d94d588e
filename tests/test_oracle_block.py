"""Pins for oracle/block.py (a4-a8) against library routines, closed forms and the paper's
degenerate cases (PAPER.md L134/L144 token-wise ops, L146 all-masked = standard block, L157
mask-aware block, L161 KV variant)."""
import math

import numpy as np
import pytest
import torch
import torch.nn.functional as Fn

import synth
from oracle import block as B
from oracle.index import build_mask_index

torch.set_default_dtype(torch.float64)


def _setup(seed=0, H=48, heads=3, F=80, L=40, dtype="f32", mod=True):
    g = synth.rng(seed)
    w = synth.block_weights(g, H, F, dtype)
    x = synth.latent(g, L, H, dtype)
    m = synth.mod_table(g, 1, 1, H, dtype, enabled=mod)[0, 0]
    return g, w, x, m


def test_layer_norm_vs_torch_and_moments():
    g = synth.rng(1)
    x = g.standard_normal((17, 33)) * 3 + 1
    ref = Fn.layer_norm(torch.tensor(x), (33,), eps=1e-6).numpy()
    out = B.layer_norm(x)
    assert np.allclose(out, ref, rtol=0, atol=1e-12)
    assert np.allclose(out.mean(-1), 0, atol=1e-12)
    assert np.allclose(out.var(-1), 1 / (1 + 1e-6 / x.var(-1)), atol=1e-9)


def test_gelu_vs_torch():
    x = np.linspace(-8, 8, 1001)
    ref = Fn.gelu(torch.tensor(x), approximate="tanh").numpy()
    assert np.allclose(B.gelu_tanh(x), ref, rtol=0, atol=1e-14)


def test_attention_vs_sdpa_and_uniform_case():
    g = synth.rng(2)
    n, Lk, heads, d = 7, 19, 3, 16
    Q, K, V = (g.standard_normal((r, heads * d)) for r in (n, Lk, Lk))
    out = B.attention(Q, K, V, heads)
    t = lambda a, r: torch.tensor(a).view(r, heads, d).transpose(0, 1)
    ref = Fn.scaled_dot_product_attention(t(Q, n), t(K, Lk), t(V, Lk))  # scale 1/sqrt(d)
    assert np.allclose(out, ref.transpose(0, 1).reshape(n, heads * d).numpy(), atol=1e-12)
    # Q = 0 -> uniform weights -> every output row is the mean of V (closed form)
    out0 = B.attention(np.zeros_like(Q), K, V, heads)
    assert np.allclose(out0, np.broadcast_to(V.mean(0), out0.shape), atol=1e-12)


def _torch_block(x, w, mod, heads):
    """The same block assembled from torch library modules (nn.MultiheadAttention, LayerNorm,
    Linear, GELU(tanh)) in float64 -- an implementation independent of oracle/block.py."""
    H = x.shape[1]
    mha = torch.nn.MultiheadAttention(H, heads, bias=True, batch_first=True)
    with torch.no_grad():
        mha.in_proj_weight.copy_(torch.tensor(w["w_qkv"]))
        mha.in_proj_bias.copy_(torch.tensor(w["b_qkv"]))
        mha.out_proj.weight.copy_(torch.tensor(w["w_o"]))
        mha.out_proj.bias.copy_(torch.tensor(w["b_o"]))
        up = torch.nn.Linear(H, w["w_up"].shape[0])
        up.weight.copy_(torch.tensor(w["w_up"])); up.bias.copy_(torch.tensor(w["b_up"]))
        dn = torch.nn.Linear(w["w_up"].shape[0], H)
        dn.weight.copy_(torch.tensor(w["w_down"])); dn.bias.copy_(torch.tensor(w["b_down"]))
        sh1, sc1, g1, sh2, sc2, g2 = torch.tensor(np.asarray(mod, np.float64)).view(6, H)
        xt = torch.tensor(np.asarray(x, np.float64))[None]
        h1 = Fn.layer_norm(xt, (H,), eps=1e-6) * (1 + sc1) + sh1
        a, _ = mha(h1, h1, h1, need_weights=False)
        x1 = xt + g1 * a
        h2 = Fn.layer_norm(x1, (H,), eps=1e-6) * (1 + sc2) + sh2
        y = x1 + g2 * dn(Fn.gelu(up(h2), approximate="tanh"))
    return y[0].numpy()


@pytest.mark.parametrize("mod", [True, False])
def test_dense_block_vs_torch_modules(mod):
    _, w, x, m = _setup(mod=mod)
    y, _, _ = B.dense_block(x, w, m, 3)
    assert np.allclose(y, _torch_block(x, w, m, 3), rtol=0, atol=1e-10)


def test_dense_block_zero_weights_closed_form():
    """W = 0: Q, K const -> uniform attention -> A = bv; o = bo; y = x + g1*bo + g2*b2."""
    g, w, x, m = _setup(seed=5)
    for k in ("w_qkv", "w_o", "w_up", "w_down"):
        w[k] = np.zeros_like(w[k])
    y, _, _ = B.dense_block(x, w, m, 3)
    H = x.shape[1]
    mm = m.astype(np.float64).reshape(6, H)
    assert np.allclose(y, x + mm[2] * w["b_o"] + mm[5] * w["b_down"], atol=1e-12)


def _kv_cache_from_dense(x, w, m, heads, U):
    _, K, V = B.dense_block(x, w, m, heads)
    return K[U], V[U]


@pytest.mark.parametrize("ratio", [0.0, 0.1, 0.5, 1.0])
def test_masked_equals_dense_under_identical_input_cache(ratio):
    """L144/L157: every op but attention is token-wise, so with the cache taken from a dense
    run on the identical input, masked rows reproduce the dense rows (both modes)."""
    g, w, x, m = _setup(seed=9, L=64)
    mask = synth.mask_blobs(g, 8, 8, ratio)
    M, U = build_mask_index(mask)
    y_ref, K, V = B.dense_block(x, w, m, 3)
    y_kv, K_M, V_M = B.masked_block_kv(x[M], M, U, K[U], V[U], w, m, 3, 64)
    y_y = B.masked_block_y(x[M], M, U, x[U], w, m, 3, 64)
    assert np.allclose(y_kv, y_ref[M], rtol=0, atol=1e-12)
    assert np.allclose(y_y, y_ref[M], rtol=0, atol=1e-12)
    assert np.allclose(K_M, K[M], atol=1e-12) and np.allclose(V_M, V[M], atol=1e-12)


def test_all_ones_mask_is_dense():
    """L146: with every token masked, the mask-aware block is the standard block."""
    _, w, x, m = _setup(seed=4)
    L = x.shape[0]
    M, U = np.arange(L), np.arange(0)
    y_ref, _, _ = B.dense_block(x, w, m, 3)
    e = np.zeros((0, x.shape[1]))
    y_kv, _, _ = B.masked_block_kv(x, M, U, e, e, w, m, 3, L)
    assert np.allclose(y_kv, y_ref, rtol=0, atol=1e-12)
    assert np.allclose(B.masked_block_y(x, M, U, e, w, m, 3, L), y_ref, rtol=0, atol=1e-12)


def test_cache_is_actually_used():
    """With a cache from a DIFFERENT template input, masked rows differ from the request's own
    dense rows, and perturbing one cached key/value row changes the output."""
    g, w, x, m = _setup(seed=12, L=64)
    mask = synth.mask_random(g, 64, 0.25)
    M, U = build_mask_index(mask)
    x_t = synth.latent(g, 64, x.shape[1], "f32")
    _, Kt, Vt = B.dense_block(x_t, w, m, 3)
    y_kv, _, _ = B.masked_block_kv(x[M], M, U, Kt[U], Vt[U], w, m, 3, 64)
    y_ref, _, _ = B.dense_block(x, w, m, 3)
    assert not np.allclose(y_kv, y_ref[M], atol=1e-3)
    Vt2 = Vt.copy(); Vt2[U[0]] += 1.0
    y2, _, _ = B.masked_block_kv(x[M], M, U, Kt[U], Vt2[U], w, m, 3, 64)
    assert not np.allclose(y2, y_kv, atol=1e-6)
    # Y-mode: perturbing an unmasked input row changes masked outputs (through K/V only)
    xu = x_t[U].copy(); xu[0, 0] += 1.0          # (a whole-row shift would be LN-invariant)
    assert not np.allclose(B.masked_block_y(x[M], M, U, xu, w, m, 3, 64),
                           B.masked_block_y(x[M], M, U, x_t[U], w, m, 3, 64), atol=1e-6)


def test_key_order_invariance():
    """Softmax attention does not depend on the key order (R10: order is a layout choice)."""
    g = synth.rng(21)
    Q, K, V = g.standard_normal((5, 32)), g.standard_normal((23, 32)), g.standard_normal((23, 32))
    p = g.permutation(23)
    assert np.allclose(B.attention(Q, K, V, 2), B.attention(Q, K[p], V[p], 2), atol=1e-12)


def test_token_wise_rows_independent():
    """L134: outside attention each row's result depends only on that row: two different
    inputs that share rows M and K/V produce identical masked outputs."""
    g, w, x, m = _setup(seed=13, L=32)
    mask = synth.mask_random(g, 32, 0.5)
    M, U = build_mask_index(mask)
    _, K, V = B.dense_block(x, w, m, 3)
    y1, _, _ = B.masked_block_kv(x[M], M, U, K[U], V[U], w, m, 3, 32)
    y2, _, _ = B.masked_block_kv(x[M][::-1].copy(), M[::-1].copy(), U, K[U], V[U], w, m, 3, 32)
    assert np.allclose(y1, y2[::-1], atol=1e-12)


# ---- NEXT-2: parallel (Flux single-stream) block, reading R23 ------------------------------
def _setup_par(seed=0, H=48, heads=3, F=80, L=40, dtype="f32"):
    g = synth.rng(seed)
    w = synth.block_weights(g, H, F, dtype, kind="par")
    x = synth.latent(g, L, H, dtype)
    m = synth.mod_table(g, 1, 1, H, dtype)[0, 0]
    return g, w, x, m


def _torch_parallel_block(x, w, mod, heads):
    """The parallel block from torch library modules in float64: nn.MultiheadAttention takes
    W1's Q/K/V rows and W2's first H columns as its output projection; the MLP branch is two
    nn.Linear layers over W1's last F rows and W2's last F columns."""
    H = x.shape[1]
    F = w["w_1"].shape[0] - 3 * H
    W1, b1 = np.asarray(w["w_1"], np.float64), np.asarray(w["b_1"], np.float64)
    W2 = np.asarray(w["w_2"], np.float64)
    mha = torch.nn.MultiheadAttention(H, heads, bias=True, batch_first=True)
    up, dn = torch.nn.Linear(H, F), torch.nn.Linear(F, H)
    with torch.no_grad():
        mha.in_proj_weight.copy_(torch.tensor(W1[:3 * H])); mha.in_proj_bias.copy_(torch.tensor(b1[:3 * H]))
        mha.out_proj.weight.copy_(torch.tensor(W2[:, :H])); mha.out_proj.bias.zero_()
        up.weight.copy_(torch.tensor(W1[3 * H:])); up.bias.copy_(torch.tensor(b1[3 * H:]))
        dn.weight.copy_(torch.tensor(W2[:, H:])); dn.bias.copy_(torch.tensor(np.asarray(w["b_2"], np.float64)))
        sh1, sc1, g1 = torch.tensor(np.asarray(mod, np.float64)).view(6, H)[:3]
        xt = torch.tensor(np.asarray(x, np.float64))[None]
        h = Fn.layer_norm(xt, (H,), eps=1e-6) * (1 + sc1) + sh1
        a, _ = mha(h, h, h, need_weights=False)
        y = xt + g1 * (a + dn(Fn.gelu(up(h), approximate="tanh")))
    return y[0].numpy()


def test_parallel_block_vs_torch_modules():
    _, w, x, m = _setup_par()
    y, K, V = B.dense_block(x, w, m, 3)
    assert np.allclose(y, _torch_parallel_block(x, w, m, 3), rtol=0, atol=1e-10)
    # K, V are W1's rows [H, 3H) applied to the normalised input
    H = x.shape[1]
    mm = np.asarray(m, np.float64).reshape(6, H)
    h = B.layer_norm(x) * (1 + mm[1]) + mm[0]
    assert np.allclose(K, h @ np.asarray(w["w_1"], np.float64)[H:2 * H].T + w["b_1"][H:2 * H], atol=1e-12)


def test_parallel_block_zero_weights_closed_form():
    """W1 = W2 = 0: y = x + gate1 * b2 (the MLP branch GELU(b1) meets a zero W2)."""
    _, w, x, m = _setup_par(seed=3)
    w["w_1"], w["w_2"] = np.zeros_like(w["w_1"]), np.zeros_like(w["w_2"])
    y, _, _ = B.dense_block(x, w, m, 3)
    H = x.shape[1]
    assert np.allclose(y, x + m.reshape(6, H)[2] * w["b_2"], atol=1e-12)


@pytest.mark.parametrize("ratio", [0.0, 0.3, 1.0])
def test_parallel_masked_equals_dense_under_identical_input_cache(ratio):
    g, w, x, m = _setup_par(seed=19, L=64)
    mask = synth.mask_blobs(g, 8, 8, ratio)
    M, U = build_mask_index(mask)
    y_ref, K, V = B.dense_block(x, w, m, 3)
    y_kv, K_M, V_M = B.masked_block_kv(x[M], M, U, K[U], V[U], w, m, 3, 64)
    y_y = B.masked_block_y(x[M], M, U, x[U], w, m, 3, 64)
    assert np.allclose(y_kv, y_ref[M], rtol=0, atol=1e-12)
    assert np.allclose(y_y, y_ref[M], rtol=0, atol=1e-12)
    assert np.allclose(K_M, K[M], atol=1e-12) and np.allclose(V_M, V[M], atol=1e-12)


def test_parallel_cache_is_actually_used():
    g, w, x, m = _setup_par(seed=23, L=64)
    mask = synth.mask_random(g, 64, 0.25)
    M, U = build_mask_index(mask)
    x_t = synth.latent(g, 64, x.shape[1], "f32")
    _, Kt, Vt = B.dense_block(x_t, w, m, 3)
    y_kv, _, _ = B.masked_block_kv(x[M], M, U, Kt[U], Vt[U], w, m, 3, 64)
    y_ref, _, _ = B.dense_block(x, w, m, 3)
    assert not np.allclose(y_kv, y_ref[M], atol=1e-3)


# ---- NEXT-2: SDXL UNet transformer block (self-attn + cross-attn + GEGLU), reading R24 -----
def _setup_sdxl(seed=0, H=48, heads=3, F=80, L=40, L_ctx=7, D_ctx=24, dtype="f32"):
    g = synth.rng(seed)
    w = synth.block_weights(g, H, F, dtype, kind="sdxl", D_ctx=D_ctx)
    x = synth.latent(g, L, H, dtype)
    ctx = synth.context(g, L_ctx, D_ctx, dtype)
    return g, w, x, ctx


def _torch_sdxl_block(x, w, ctx, heads):
    """The SDXL block assembled from torch library modules in float64, as diffusers'
    BasicTransformerBlock is: nn.LayerNorm (affine), nn.MultiheadAttention for self-attention
    (bias-free in-projection, biased out-projection) and for cross-attention (kdim = vdim =
    D_ctx, separate q/k/v projection weights), and GEGLU as Linear -> chunk(2) -> value *
    gelu(gate) -> Linear."""
    t = lambda a: torch.tensor(np.asarray(a, np.float64))
    H, D = x.shape[1], ctx.shape[1]
    F = w["w_up"].shape[0] // 2
    lns = [torch.nn.LayerNorm(H, eps=1e-6) for _ in range(3)]
    sa = torch.nn.MultiheadAttention(H, heads, bias=True, batch_first=True)
    ca = torch.nn.MultiheadAttention(H, heads, bias=True, batch_first=True, kdim=D, vdim=D)
    up, dn = torch.nn.Linear(H, 2 * F), torch.nn.Linear(F, H)
    with torch.no_grad():
        for i, ln in enumerate(lns, 1):
            ln.weight.copy_(t(w[f"ln{i}_w"])); ln.bias.copy_(t(w[f"ln{i}_b"]))
        sa.in_proj_weight.copy_(t(w["w_qkv"])); sa.in_proj_bias.zero_()
        sa.out_proj.weight.copy_(t(w["w_o"])); sa.out_proj.bias.copy_(t(w["b_o"]))
        ca.q_proj_weight.copy_(t(w["w_q2"]))
        ca.k_proj_weight.copy_(t(w["w_kv2"][:H])); ca.v_proj_weight.copy_(t(w["w_kv2"][H:]))
        ca.in_proj_bias.zero_()
        ca.out_proj.weight.copy_(t(w["w_o2"])); ca.out_proj.bias.copy_(t(w["b_o2"]))
        up.weight.copy_(t(w["w_up"])); up.bias.copy_(t(w["b_up"]))
        dn.weight.copy_(t(w["w_down"])); dn.bias.copy_(t(w["b_down"]))
        xt, ct = t(x)[None], t(ctx)[None]
        h = lns[0](xt)
        x1 = xt + sa(h, h, h, need_weights=False)[0]
        h = lns[1](x1)
        x2 = x1 + ca(h, ct, ct, need_weights=False)[0]
        v, gate = up(lns[2](x2)).chunk(2, dim=-1)
        y = x2 + dn(v * Fn.gelu(gate, approximate="tanh"))
    return y[0].numpy()


def test_sdxl_block_vs_torch_modules():
    _, w, x, ctx = _setup_sdxl()
    y, K, V = B.dense_block(x, w, None, 3, ctx)
    assert np.allclose(y, _torch_sdxl_block(x, w, ctx, 3), rtol=0, atol=1e-10)
    H = x.shape[1]
    h = Fn.layer_norm(torch.tensor(np.asarray(x, np.float64)), (H,),
                      weight=torch.tensor(np.asarray(w["ln1_w"], np.float64)),
                      bias=torch.tensor(np.asarray(w["ln1_b"], np.float64)), eps=1e-6).numpy()
    assert np.allclose(K, h @ np.asarray(w["w_qkv"], np.float64)[H:2 * H].T, atol=1e-12)


def test_sdxl_single_context_token_closed_form():
    """L_ctx = 1: the cross-attention softmax is 1 for every query, so its output is the one
    context value row ctx Wv2^T for every latent row; with W_o2 = I the block's x2 - x1 equals
    that row (checked through y with a zero feed-forward)."""
    _, w, x, ctx = _setup_sdxl(seed=31, L_ctx=1)
    H = x.shape[1]
    w["w_o2"], w["b_o2"] = np.eye(H, dtype=np.float32), np.zeros(H, np.float32)
    w["w_down"], w["b_down"] = np.zeros_like(w["w_down"]), np.zeros_like(w["b_down"])
    y, _, _ = B.dense_block(x, w, None, 3, ctx)
    w0 = dict(w); w0["w_kv2"] = np.zeros_like(w["w_kv2"])   # same block, zero context values
    y0, _, _ = B.dense_block(x, w0, None, 3, ctx)
    v_row = np.asarray(ctx, np.float64) @ np.asarray(w["w_kv2"], np.float64)[H:].T
    assert np.allclose(y - y0, np.broadcast_to(v_row, y.shape), atol=1e-12)


def test_sdxl_geglu_halves_closed_form():
    """GEGLU chunk order: gate weights 0 and gate bias c give P * GELU(c) with P the FIRST F
    output rows; swapping the halves would give GELU(P) * ... instead."""
    g = synth.rng(33)
    h = g.standard_normal((5, 8))
    W = g.standard_normal((12, 8)); W[6:] = 0.0
    b = np.zeros(12); b[6:] = 3.0
    gelu3 = 0.5 * 3.0 * (1 + math.tanh(math.sqrt(2 / math.pi) * (3.0 + 0.044715 * 27.0)))
    assert np.allclose(B.geglu(h, W, b), (h @ W[:6].T) * gelu3, atol=1e-12)


@pytest.mark.parametrize("ratio", [0.0, 0.3, 1.0])
def test_sdxl_masked_equals_dense_under_identical_input_cache(ratio):
    g, w, x, ctx = _setup_sdxl(seed=35, L=64)
    mask = synth.mask_blobs(g, 8, 8, ratio)
    M, U = build_mask_index(mask)
    y_ref, K, V = B.dense_block(x, w, None, 3, ctx)
    y_kv, K_M, V_M = B.masked_block_kv(x[M], M, U, K[U], V[U], w, None, 3, 64, ctx)
    y_y = B.masked_block_y(x[M], M, U, x[U], w, None, 3, 64, ctx)
    assert np.allclose(y_kv, y_ref[M], rtol=0, atol=1e-12)
    assert np.allclose(y_y, y_ref[M], rtol=0, atol=1e-12)
    assert np.allclose(K_M, K[M], atol=1e-12) and np.allclose(V_M, V[M], atol=1e-12)


def test_sdxl_context_and_cache_are_used():
    g, w, x, ctx = _setup_sdxl(seed=37, L=64)
    mask = synth.mask_random(g, 64, 0.25)
    M, U = build_mask_index(mask)
    x_t = synth.latent(g, 64, x.shape[1], "f32")
    _, Kt, Vt = B.dense_block(x_t, w, None, 3, ctx)
    y_kv, _, _ = B.masked_block_kv(x[M], M, U, Kt[U], Vt[U], w, None, 3, 64, ctx)
    y_ref, _, _ = B.dense_block(x, w, None, 3, ctx)
    assert not np.allclose(y_kv, y_ref[M], atol=1e-3)
    ctx2 = ctx.copy(); ctx2[0, 0] += 1.0
    y2, _, _ = B.masked_block_kv(x[M], M, U, Kt[U], Vt[U], w, None, 3, 64, ctx2)
    assert not np.allclose(y2, y_kv, atol=1e-6)


# ---- NEXT-2: Flux double-stream (MM-DiT) block, reading R25 --------------------------------
def _setup_double(seed=0, H=48, heads=3, F=80, L_img=32, L_txt=8, dtype="f32"):
    g = synth.rng(seed)
    w = synth.block_weights(g, H, F, dtype, kind="double")
    x = synth.latent(g, L_img + L_txt, H, dtype)
    m = synth.mod_table(g, 1, 1, H, dtype, streams=2)[0, 0]
    return g, w, x, m


def _torch_double_block(x, w, mod, heads, L_img):
    """The double-stream block from torch library routines in float64: per-stream Linear /
    LayerNorm, and ONE scaled_dot_product_attention over the concatenated streams."""
    t = lambda a: torch.tensor(np.asarray(a, np.float64))
    H = x.shape[1]
    d = H // heads
    m = t(mod).view(2, 6, H)
    xs = [t(x[:L_img]), t(x[L_img:])]
    ws = [w["img"], w["txt"]]
    lin = lambda h, W, b: Fn.linear(h, t(W), t(b))
    hs = [Fn.layer_norm(xs[i], (H,), eps=1e-6) * (1 + m[i, 1]) + m[i, 0] for i in range(2)]
    qkv = [lin(hs[i], ws[i]["w_qkv"], ws[i]["b_qkv"]) for i in range(2)]
    q, k, v = (torch.cat([qkv[0][:, j * H:(j + 1) * H], qkv[1][:, j * H:(j + 1) * H]])
               .view(-1, heads, d).transpose(0, 1) for j in range(3))
    a = Fn.scaled_dot_product_attention(q, k, v).transpose(0, 1).reshape(-1, H)
    a_s = [a[:L_img], a[L_img:]]
    out = []
    for i in range(2):
        x1 = xs[i] + m[i, 2] * lin(a_s[i], ws[i]["w_o"], ws[i]["b_o"])
        h2 = Fn.layer_norm(x1, (H,), eps=1e-6) * (1 + m[i, 4]) + m[i, 3]
        mlp = lin(Fn.gelu(lin(h2, ws[i]["w_up"], ws[i]["b_up"]), approximate="tanh"),
                  ws[i]["w_down"], ws[i]["b_down"])
        out.append(x1 + m[i, 5] * mlp)
    return torch.cat(out).numpy()


def test_double_block_vs_torch():
    _, w, x, m = _setup_double()
    y, K, V = B.dense_block(x, w, m, 3, L_txt=8)
    assert np.allclose(y, _torch_double_block(x, w, m, 3, 32), rtol=0, atol=1e-10)


def test_double_block_same_weights_is_sequential():
    """Both streams with the same weights and modulation reduce to the sequential block."""
    g, w, x, m = _setup_double(seed=41)
    w["txt"] = w["img"]
    H = x.shape[1]
    m[6 * H:] = m[:6 * H]
    y, _, _ = B.dense_block(x, w, m, 3, L_txt=8)
    y_seq, _, _ = B.dense_block(x, w["img"], m[:6 * H], 3)
    assert np.allclose(y, y_seq, rtol=0, atol=1e-12)


def test_double_streams_use_their_own_weights():
    """Changing the text stream's MLP changes only text rows (token-wise outside attention)."""
    g, w, x, m = _setup_double(seed=43)
    y, _, _ = B.dense_block(x, w, m, 3, L_txt=8)
    w2 = {"kind": "double", "img": w["img"], "txt": dict(w["txt"])}
    w2["txt"]["b_down"] = w["txt"]["b_down"] + 1.0
    y2, _, _ = B.dense_block(x, w2, m, 3, L_txt=8)
    assert np.allclose(y2[:32], y[:32], atol=1e-12)
    assert np.allclose(y2[32:] - y[32:], np.asarray(m, np.float64).reshape(2, 6, -1)[1, 5], atol=1e-9)


@pytest.mark.parametrize("ratio", [0.0, 0.3, 1.0])
def test_double_masked_equals_dense_under_identical_input_cache(ratio):
    g, w, x, m = _setup_double(seed=45, L_img=64, L_txt=8)
    mask = synth.token_mask(synth.mask_blobs(g, 8, 8, ratio), 8)
    M, U = build_mask_index(mask)
    y_ref, K, V = B.dense_block(x, w, m, 3, L_txt=8)
    y_kv, K_M, V_M = B.masked_block_kv(x[M], M, U, K[U], V[U], w, m, 3, 72, L_txt=8)
    y_y = B.masked_block_y(x[M], M, U, x[U], w, m, 3, 72, L_txt=8)
    assert np.allclose(y_kv, y_ref[M], rtol=0, atol=1e-12)
    assert np.allclose(y_y, y_ref[M], rtol=0, atol=1e-12)
    assert np.allclose(K_M, K[M], atol=1e-12) and np.allclose(V_M, V[M], atol=1e-12)


def test_double_cache_is_actually_used():
    g, w, x, m = _setup_double(seed=47, L_img=64, L_txt=8)
    mask = synth.token_mask(synth.mask_random(g, 64, 0.25), 8)
    M, U = build_mask_index(mask)
    x_t = synth.latent(g, 72, x.shape[1], "f32")
    _, Kt, Vt = B.dense_block(x_t, w, m, 3, L_txt=8)
    y_kv, _, _ = B.masked_block_kv(x[M], M, U, Kt[U], Vt[U], w, m, 3, 72, L_txt=8)
    y_ref, _, _ = B.dense_block(x, w, m, 3, L_txt=8)
    assert not np.allclose(y_kv, y_ref[M], atol=1e-3)
