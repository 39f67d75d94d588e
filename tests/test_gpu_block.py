"""GPU parity of the block forward (a4-a8) against the oracle, through the C ABI.

Tolerance (BASELINE.json north_star, reading R20): |g - r| <= tol * max(1, |r|), tol = 1e-5 for
the fp32 path, 2e-2 for bf16."""
import numpy as np
import pytest
import torch

import synth
from oracle import block as B
from oracle.index import build_mask_index
from gpu_util import TOL, check_close, to_dev, to_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as fps
    fps.require_gpu()
    return fps


def _problem(seed, dtype, H, heads, Fd, L_img, L_txt, ratios, mod=True, blobs=False, kind="seq"):
    g = synth.rng(seed)
    w = synth.block_weights(g, H, Fd, dtype, kind)
    reqs = []
    for m in ratios:
        L = L_img + L_txt
        if blobs:
            gh = int(np.sqrt(L_img))
            im = synth.mask_blobs(g, gh, L_img // gh, m)
        else:
            im = synth.mask_random(g, L_img, m)
        mask = synth.token_mask(im, L_txt)
        M, U = build_mask_index(mask)
        reqs.append(dict(
            mask=mask, M=M, U=U, L=L,
            x=synth.latent(g, L, H, dtype),                 # block input (all rows)
            K=synth.latent(g, L, H, dtype), V=synth.latent(g, L, H, dtype),   # KV cache
            xu=synth.latent(g, L, H, dtype),                # Y-mode cached input rows
            mod=synth.mod_table(g, 1, 1, H, dtype, enabled=mod)[0, 0]))
    return w, reqs


def _run_masked(F, w, reqs, heads, dtype, mode):
    dt = F.DTYPE_CODE[dtype]
    H = (w["w_2"] if w.get("kind") == "par" else w["w_o"]).shape[0]
    bw = F.BlockWeights(w, heads, dt)
    Ls = [r["L"] for r in reqs]
    cu_k = np.concatenate([[0], np.cumsum(Ls)])
    q_row = np.concatenate([r["M"] + cu_k[i] for i, r in enumerate(reqs)]).astype(np.int32)
    u_row = np.concatenate([r["U"] + cu_k[i] for i, r in enumerate(reqs)]).astype(np.int32)
    x_act = to_dev(np.concatenate([r["x"][r["M"]] for r in reqs]), dtype)
    mod = to_dev(np.stack([r["mod"] for r in reqs]), dtype)
    kv = torch.zeros(int(cu_k[-1]), 2 * H, dtype=x_act.dtype, device="cuda")
    xu = None
    if mode == "kv":
        for i, r in enumerate(reqs):     # the cached rows U (what fps_cache_prefetch delivers)
            full = np.concatenate([r["K"], r["V"]], axis=1)
            kv[cu_k[i] + torch.as_tensor(r["U"]).long().cuda()] = to_dev(full[r["U"]], dtype)
    else:
        xu = to_dev(np.concatenate([r["xu"] for r in reqs]), dtype)     # [sum L, H] source
    qd = torch.as_tensor(q_row).cuda()
    ud = torch.as_tensor(u_row).cuda()
    b = F.VarlenBatch([len(r["M"]) for r in reqs], Ls, q_row=qd, mod=mod, mode=F.MODE_CODE[mode],
                      u_row=ud, u_src=ud, n_unmasked=[len(r["U"]) for r in reqs])
    y = F.masked_block_forward(bw, b, x_act, kv, xu=xu)
    torch.cuda.synchronize()
    return to_np(y), kv


def _ref_masked(w, reqs, heads, mode):
    out = []
    for r in reqs:
        if mode == "kv":
            y, _, _ = B.masked_block_kv(r["x"][r["M"]], r["M"], r["U"], r["K"][r["U"]],
                                        r["V"][r["U"]], w, r["mod"], heads, r["L"])
        else:
            y = B.masked_block_y(r["x"][r["M"]], r["M"], r["U"], r["xu"][r["U"]], w, r["mod"],
                                 heads, r["L"])
        out.append(y)
    return np.concatenate(out)


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_c1_fp32_masked(F, mode):
    """configs[0]: hidden 64, 2 heads, 16x16 latent, 25% random mask, batch 1, fp32."""
    w, reqs = _problem(1001, "f32", 64, 2, 256, 256, 0, [0.25], mod=False)
    y, _ = _run_masked(F, w, reqs, 2, "f32", mode)
    check_close(y, _ref_masked(w, reqs, 2, mode), TOL["f32"], f"C1 {mode}")


def test_c1_fp32_dense(F):
    w, reqs = _problem(1001, "f32", 64, 2, 256, 256, 0, [1.0], mod=True)
    r = reqs[0]
    bw = F.BlockWeights(w, 2, F.FPS_F32)
    b = F.VarlenBatch([256], [256], mod=to_dev(r["mod"][None], "f32"))
    y, _ = F.dense_block_forward(bw, b, to_dev(r["x"], "f32"))
    torch.cuda.synchronize()
    ref, _, _ = B.dense_block(r["x"], w, r["mod"], 2)
    check_close(to_np(y), ref, TOL["f32"], "C1 dense")


@pytest.mark.parametrize("mode", ["kv", "y"])
@pytest.mark.parametrize("simt", [False, True])
def test_bf16_varlen_batch(F, mode, simt):
    """Heterogeneous masks (continuous batch, L237) in one varlen launch; d = 128, ragged rows
    spanning several 128-row tiles, text tokens always active."""
    w, reqs = _problem(2002, "bf16", 256, 2, 1024, 576, 40, [0.05, 0.6, 0.3], blobs=True)
    F.fps_set_disable_tc(3 if simt else 0)
    try:
        y, _ = _run_masked(F, w, reqs, 2, "bf16", mode)
    finally:
        F.fps_set_disable_tc(0)
    check_close(y, _ref_masked(w, reqs, 2, mode), TOL["bf16"], f"bf16 {mode} simt={simt}")


def test_bf16_head64_and_odd_width(F):
    """SDXL-like heads (d = 64) and a hidden size that is not a multiple of 256 (H = 640)."""
    w, reqs = _problem(2003, "bf16", 640, 10, 2560, 256, 0, [0.3, 0.1])
    y, _ = _run_masked(F, w, reqs, 10, "bf16", "kv")
    check_close(y, _ref_masked(w, reqs, 10, "kv"), TOL["bf16"], "bf16 H=640")


def test_all_active_equals_dense(F):
    """L146: all tokens masked -> the masked block is the dense block (GPU vs oracle)."""
    w, reqs = _problem(2004, "bf16", 256, 2, 1024, 300, 0, [1.0])
    y, _ = _run_masked(F, w, reqs, 2, "bf16", "kv")
    r = reqs[0]
    ref, _, _ = B.dense_block(r["x"], w, r["mod"], 2)
    check_close(y, ref, TOL["bf16"], "all-active")


def test_fresh_kv_written_at_token_rows(F):
    """The QKV epilogue writes fresh K|V rows at their original token rows (R10)."""
    w, reqs = _problem(2005, "bf16", 256, 2, 1024, 400, 16, [0.25, 0.5])
    _, kv = _run_masked(F, w, reqs, 2, "bf16", "kv")
    kv = to_np(kv)
    base = 0
    H = 256
    for r in reqs:
        sh1, sc1 = r["mod"][:H], r["mod"][H:2 * H]
        h1 = B.layer_norm(r["x"][r["M"]]) * (1 + sc1) + sh1
        Kr = B.linear(h1, w["w_qkv"][H:2 * H], w["b_qkv"][H:2 * H])
        Vr = B.linear(h1, w["w_qkv"][2 * H:], w["b_qkv"][2 * H:])
        check_close(kv[base + r["M"], :H], Kr, TOL["bf16"], "fresh K")
        check_close(kv[base + r["M"], H:], Vr, TOL["bf16"], "fresh V")
        base += r["L"]


def test_flux_scale_sampled_rows(F):
    """configs[2] shapes (H 3072, 24x128 heads, F 12288, 4096 + 512 tokens, m = 0.2) in the
    launch configuration the bench uses; the oracle checks a sample of output rows."""
    g = synth.rng(3003)
    H, heads, Fd, L_img, L_txt = 3072, 24, 12288, 4096, 512
    L = L_img + L_txt
    w = synth.block_weights(g, H, Fd, "bf16")
    mask = synth.token_mask(synth.mask_blobs(g, 64, 64, 0.2), L_txt)
    M, U = build_mask_index(mask)
    x = synth.latent(g, L, H, "bf16")
    K, V = synth.latent(g, L, H, "bf16"), synth.latent(g, L, H, "bf16")
    mod = synth.mod_table(g, 1, 1, H, "bf16")[0, 0]
    req = dict(mask=mask, M=M, U=U, L=L, x=x, K=K, V=V, xu=None, mod=mod)
    y, _ = _run_masked(F, w, [req], heads, "bf16", "kv")
    # oracle on sampled active rows: fresh K/V of all rows M (needed by every query), then the
    # sampled rows' attention + MLP
    sh1, sc1 = mod[:H], mod[H:2 * H]
    h1 = B.layer_norm(x[M]) * (1 + sc1) + sh1
    Kall, Vall = np.array(K, np.float64), np.array(V, np.float64)
    Kall[M] = B.linear(h1, w["w_qkv"][H:2 * H], w["b_qkv"][H:2 * H])
    Vall[M] = B.linear(h1, w["w_qkv"][2 * H:], w["b_qkv"][2 * H:])
    sample = np.unique(np.concatenate([g.choice(len(M), 40, replace=False), [0, len(M) - 1]]))
    Q = B.linear(h1[sample], w["w_qkv"][:H], w["b_qkv"][:H])
    a = B.attention(Q, Kall, Vall, heads)
    ref = B._attn_out_and_mlp(x[M][sample], a, w, mod, H)
    check_close(y[sample], ref, TOL["bf16"], "flux sampled")


# ---- NEXT-2: parallel (Flux single-stream) block, reading R23 ------------------------------
@pytest.mark.parametrize("mode", ["kv", "y"])
def test_parallel_fp32_masked(F, mode):
    w, reqs = _problem(4001, "f32", 64, 2, 256, 256, 8, [0.25, 0.6], kind="par")
    y, _ = _run_masked(F, w, reqs, 2, "f32", mode)
    check_close(y, _ref_masked(w, reqs, 2, mode), TOL["f32"], f"parallel fp32 {mode}")


@pytest.mark.parametrize("mode", ["kv", "y"])
@pytest.mark.parametrize("simt", [False, True])
def test_parallel_bf16_varlen_batch(F, mode, simt):
    w, reqs = _problem(4002, "bf16", 256, 2, 1024, 576, 40, [0.05, 0.6, 0.3], blobs=True,
                       kind="par")
    F.fps_set_disable_tc(3 if simt else 0)
    try:
        y, _ = _run_masked(F, w, reqs, 2, "bf16", mode)
    finally:
        F.fps_set_disable_tc(0)
    check_close(y, _ref_masked(w, reqs, 2, mode), TOL["bf16"], f"parallel bf16 {mode} simt={simt}")


def test_parallel_dense_and_head64(F):
    w, reqs = _problem(4003, "bf16", 640, 10, 2560, 300, 20, [1.0], kind="par")
    r = reqs[0]
    bw = F.BlockWeights(w, 10, F.FPS_BF16)
    b = F.VarlenBatch([r["L"]], [r["L"]], mod=to_dev(r["mod"][None], "bf16"))
    y, _ = F.dense_block_forward(bw, b, to_dev(r["x"], "bf16"))
    torch.cuda.synchronize()
    ref, _, _ = B.dense_block(r["x"], w, r["mod"], 10)
    check_close(to_np(y), ref, TOL["bf16"], "parallel dense H=640")


def test_parallel_weights_validated(F):
    w, _ = _problem(4004, "bf16", 128, 2, 512, 64, 0, [0.5], kind="par")
    bw = F.BlockWeights(w, 2, F.FPS_BF16)
    bw.c.w_o = bw.c.w_qkv                         # a sequential-only pointer set -> EINVAL
    b = F.VarlenBatch([64], [64])
    with pytest.raises(F.FlashPSError):
        F.dense_block_forward(bw, b, torch.zeros(64, 128, dtype=torch.bfloat16, device="cuda"))


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_c4_continuous_batch_sampled_rows(F, mode):
    """configs[3] in the bench's launch configuration: 16 Flux-scale requests with masks from 5 %
    to 60 % in ONE varlen launch per GEMM / attention; the oracle checks sampled rows of four
    requests (first, last and two inner ones, incl. the smallest and largest masks)."""
    g = synth.rng(3004 + (mode == "y"))
    H, heads, Fd, L_img, L_txt = 3072, 24, 12288, 4096, 512
    L = L_img + L_txt
    w = synth.block_weights(g, H, Fd, "bf16")
    reqs = []
    for m in np.linspace(0.05, 0.60, 16):
        mask = synth.token_mask(synth.mask_blobs(g, 64, 64, float(m)), L_txt)
        M, U = build_mask_index(mask)
        reqs.append(dict(mask=mask, M=M, U=U, L=L, x=synth.latent(g, L, H, "bf16"),
                         K=synth.latent(g, L, H, "bf16"), V=synth.latent(g, L, H, "bf16"),
                         xu=synth.latent(g, L, H, "bf16"),
                         mod=synth.mod_table(g, 1, 1, H, "bf16")[0, 0]))
    y, _ = _run_masked(F, w, reqs, heads, "bf16", mode)
    cu = np.concatenate([[0], np.cumsum([len(r["M"]) for r in reqs])])
    Wq, bq = w["w_qkv"][:H], w["b_qkv"][:H]
    Wk, bk = w["w_qkv"][H:2 * H], w["b_qkv"][H:2 * H]
    Wv, bv = w["w_qkv"][2 * H:], w["b_qkv"][2 * H:]
    for i in (0, 5, 10, 15):
        r = reqs[i]
        M, U = r["M"], r["U"]
        sh1, sc1 = r["mod"][:H], r["mod"][H:2 * H]
        x_in = np.array(r["x"], np.float64)
        if mode == "y":
            x_in[U] = r["xu"][U]
        h1 = B.layer_norm(x_in) * (1 + sc1) + sh1
        if mode == "kv":
            Kall, Vall = np.array(r["K"], np.float64), np.array(r["V"], np.float64)
            Kall[M] = B.linear(h1[M], Wk, bk)
            Vall[M] = B.linear(h1[M], Wv, bv)
        else:
            Kall, Vall = B.linear(h1, Wk, bk), B.linear(h1, Wv, bv)
        sample = np.unique(np.concatenate([g.choice(len(M), 12, replace=False), [0, len(M) - 1]]))
        a = B.attention(B.linear(h1[M][sample], Wq, bq), Kall, Vall, heads)
        ref = B._attn_out_and_mlp(r["x"][M][sample], a, w, r["mod"], H)
        check_close(y[cu[i] + sample], ref, TOL["bf16"], f"C4 {mode} request {i}")


@pytest.mark.parametrize("pair", [0, 1])
@pytest.mark.parametrize("mode,split", [("kv", 2), ("kv", 3), ("y", 2), ("kv", 4)])
def test_split_kv_attention(F, mode, split, pair):
    """Split-KV attention (each CTA's key range in S parts, then a combine pass) inside the
    block: heterogeneous varlen batch with ragged key tiles; the parts must merge to the
    oracle's softmax over all keys."""
    w, reqs = _problem(2010 + split, "bf16", 256, 2, 1024, 1500, 36, [0.05, 0.6, 0.3], blobs=False)
    F.fps_set_disable_tc(split << 8 | pair << 12)      # pair: the CTA-pair kernel (attn_tc4)
    try:
        y, _ = _run_masked(F, w, reqs, 2, "bf16", mode)
    finally:
        F.fps_set_disable_tc(0)
    check_close(y, _ref_masked(w, reqs, 2, mode), TOL["bf16"], f"split {split} {mode}")


@pytest.mark.parametrize("kind,mode", [("seq", "kv"), ("seq", "y"), ("par", "kv"), ("par", "y")])
def test_active_rows_read_from_full_buffer_bit_identical(F, kind, mode):
    """a2 fused into the block (x_full_rows): reading the active input rows straight out of the
    full merged buffer at d_q_row gives the same bits as the compact gathered rows."""
    w, reqs = _problem(4100 + (kind == "par"), "bf16", 256, 2, 1024, 576, 40, [0.05, 0.6, 0.3],
                       blobs=True, kind=kind)
    y_ref, _ = _run_masked(F, w, reqs, 2, "bf16", mode)
    orig = F.masked_block_forward
    full = to_dev(np.concatenate([r["x"] for r in reqs]), "bf16")      # [sum L, H]

    def fused(bw, b, x_act, kv, xu=None, **kw):
        b.c.x_full_rows = 1
        return orig(bw, b, full, kv, xu=xu, y_act=torch.empty_like(x_act), **kw)
    F.masked_block_forward = fused
    try:
        y, _ = _run_masked(F, w, reqs, 2, "bf16", mode)
    finally:
        F.masked_block_forward = orig
    assert np.array_equal(y, y_ref)


@pytest.mark.parametrize("kind,H,heads,Fd,L_img,L_txt,ratios", [
    ("par", 256, 2, 1024, 576, 40, [0.05, 0.6, 0.3]),   # several tiles per problem, ragged
    ("par", 3072, 24, 12288, 4096, 512, [0.2]),         # the C3 single-stream block
    ("seq", 256, 2, 1024, 576, 40, [0.05, 0.6, 0.3]),   # sequential block: Q(M) + K|V(all rows)
    ("seq", 1280, 20, 5120, 1024, 0, [0.1, 0.3, 0.5, 0.3]),   # the C2B level's width
])
def test_y_parallel_grouped_projections_bit_identical(F, kind, H, heads, Fd, L_img, L_txt, ratios):
    """Y-mode projections in ONE grouped launch -- parallel block: W1 over rows M and K|V over
    the cached rows U (per-problem N: 3H + F and 2H); sequential block: Q over rows M and K|V over
    all rows (N: H and 2H) -- give the same bits as two launches (flag bit 15), and match the
    oracle (masked_block_y)."""
    w, reqs = _problem(4200 + H, "bf16", H, heads, Fd, L_img, L_txt, ratios, blobs=True,
                       kind=kind)
    y_grouped, kv_grouped = _run_masked(F, w, reqs, heads, "bf16", "y")
    F.fps_set_disable_tc(1 << 15)
    try:
        y_two, kv_two = _run_masked(F, w, reqs, heads, "bf16", "y")
    finally:
        F.fps_set_disable_tc(0)
    assert np.array_equal(y_grouped, y_two)
    assert torch.equal(kv_grouped, kv_two)
    if H <= 256:
        check_close(y_grouped, _ref_masked(w, reqs, heads, "y"), TOL["bf16"])
