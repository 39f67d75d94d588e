"""GPU parity of the Flux double-stream (MM-DiT) block (NEXT-2, reading R25: per-stream
weights and adaLN, one joint attention) against the oracle, through the C ABI: block level
(dense, KV- and Y-mode over a heterogeneous varlen batch, tcgen05 and SIMT kernels) and through
fps_run_batch in a Flux-like stack of double-stream then single-stream (parallel) blocks."""
import numpy as np
import pytest
import torch

import synth
from oracle import block as B
from oracle import stack as S
from oracle.index import build_mask_index
from gpu_util import TOL, check_close, stack_tol, to_dev, to_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as fps
    fps.require_gpu()
    return fps


def _problem(seed, dtype, H, heads, Fd, L_img, L_txt, ratios):
    g = synth.rng(seed)
    w = synth.block_weights(g, H, Fd, dtype, "double")
    reqs = []
    gh = int(np.sqrt(L_img))
    for m in ratios:
        L = L_img + L_txt
        mask = synth.token_mask(synth.mask_blobs(g, gh, L_img // gh, m), L_txt)
        M, U = build_mask_index(mask)
        reqs.append(dict(mask=mask, M=M, U=U, L=L, x=synth.latent(g, L, H, dtype),
                         K=synth.latent(g, L, H, dtype), V=synth.latent(g, L, H, dtype),
                         xu=synth.latent(g, L, H, dtype),
                         mod=synth.mod_table(g, 1, 1, H, dtype, streams=2)[0, 0]))
    return w, reqs


def _run(F, w, reqs, heads, dtype, mode, L_img, dense=False, inv=True):
    dt = F.DTYPE_CODE[dtype]
    H = w["img"]["w_o"].shape[0]
    bw = F.BlockWeights(w, heads, dt)
    Ls = [r["L"] for r in reqs]
    cu_k = np.concatenate([[0], np.cumsum(Ls)])
    mod = to_dev(np.stack([r["mod"] for r in reqs]), dtype)
    if dense:
        x = to_dev(np.concatenate([r["x"] for r in reqs]), dtype)
        b = F.VarlenBatch(Ls, Ls, mod=mod, act_ids=[np.arange(L) for L in Ls], L_img=L_img,
                          stream_inverse=inv)
        y, _ = F.dense_block_forward(bw, b, x)
        torch.cuda.synchronize()
        return to_np(y)
    q_row = np.concatenate([r["M"] + cu_k[i] for i, r in enumerate(reqs)]).astype(np.int32)
    u_row = np.concatenate([r["U"] + cu_k[i] for i, r in enumerate(reqs)]).astype(np.int32)
    x_act = to_dev(np.concatenate([r["x"][r["M"]] for r in reqs]), dtype)
    kv = torch.zeros(int(cu_k[-1]), 2 * H, dtype=x_act.dtype, device="cuda")
    xu = None
    if mode == "kv":
        for i, r in enumerate(reqs):
            full = np.concatenate([r["K"], r["V"]], axis=1)
            kv[cu_k[i] + torch.as_tensor(r["U"]).long().cuda()] = to_dev(full[r["U"]], dtype)
    else:
        xu = to_dev(np.concatenate([r["xu"] for r in reqs]), dtype)
    qd, ud = torch.as_tensor(q_row).cuda(), torch.as_tensor(u_row).cuda()
    b = F.VarlenBatch([len(r["M"]) for r in reqs], Ls, q_row=qd, mod=mod, mode=F.MODE_CODE[mode],
                      u_row=ud, u_src=ud, n_unmasked=[len(r["U"]) for r in reqs],
                      act_ids=[r["M"] for r in reqs], L_img=L_img, stream_inverse=inv)
    y = F.masked_block_forward(bw, b, x_act, kv, xu=xu)
    torch.cuda.synchronize()
    return to_np(y)


def _ref(w, reqs, heads, mode, L_txt):
    out = []
    for r in reqs:
        if mode == "kv":
            y, _, _ = B.masked_block_kv(r["x"][r["M"]], r["M"], r["U"], r["K"][r["U"]],
                                        r["V"][r["U"]], w, r["mod"], heads, r["L"], L_txt=L_txt)
        else:
            y = B.masked_block_y(r["x"][r["M"]], r["M"], r["U"], r["xu"][r["U"]], w, r["mod"],
                                 heads, r["L"], L_txt=L_txt)
        out.append(y)
    return np.concatenate(out)


@pytest.mark.parametrize("mode", ["kv", "y"])
@pytest.mark.parametrize("flags", [0, 3, 4, 8])
def test_double_masked_varlen_batch(F, mode, flags):
    """Three requests, masks 5-60 %, 40 text rows each: image rows of every request on the
    image weights, text rows on the text weights (one grouped GEMM launch per projection; flags
    4 / 8 force its 1-SM / CTA-pair kernel, 3 the SIMT kernels as two launches), one joint
    attention launch."""
    w, reqs = _problem(7100, "bf16", 256, 2, 1024, 576, 40, [0.05, 0.6, 0.3])
    F.fps_set_disable_tc(flags)
    try:
        y = _run(F, w, reqs, 2, "bf16", mode, 576)
    finally:
        F.fps_set_disable_tc(0)
    check_close(y, _ref(w, reqs, 2, mode, 40), TOL["bf16"], f"double {mode} flags={flags}")


def test_double_fp32_and_dense(F):
    w, reqs = _problem(7101, "f32", 64, 2, 256, 256, 16, [0.25, 1.0])
    y = _run(F, w, reqs, 2, "f32", "kv", 256)
    check_close(y, _ref(w, reqs, 2, "kv", 16), TOL["f32"], "double fp32 kv")
    yd = _run(F, w, reqs, 2, "f32", "kv", 256, dense=True)
    ref = np.concatenate([B.dense_block(r["x"], w, r["mod"], 2, L_txt=16)[0] for r in reqs])
    check_close(yd, ref, TOL["f32"], "double fp32 dense")


def test_double_flux_scale_rows(F):
    """Flux-scale double-stream block (H 3072, 24 x 128 heads, 4096 image + 512 text tokens,
    20 % mask) -- the configs[2] shapes -- checked on sampled output rows of each stream (the
    oracle computes the whole block; the comparison samples rows of both streams)."""
    g = synth.rng(7102)
    H, heads, Fd, L_img, L_txt = 3072, 24, 12288, 4096, 512
    w = synth.block_weights(g, H, Fd, "bf16", "double")
    mask = synth.token_mask(synth.mask_blobs(g, 64, 64, 0.2), L_txt)
    M, U = build_mask_index(mask)
    L = L_img + L_txt
    r = dict(mask=mask, M=M, U=U, L=L, x=synth.latent(g, L, H, "bf16"),
             K=synth.latent(g, L, H, "bf16"), V=synth.latent(g, L, H, "bf16"),
             mod=synth.mod_table(g, 1, 1, H, "bf16", streams=2)[0, 0])
    y = _run(F, w, [r], heads, "bf16", "kv", L_img)
    ref = _ref(w, [r], heads, "kv", L_txt)
    pick = np.concatenate([np.arange(0, len(M) - L_txt, 97), np.arange(len(M) - L_txt, len(M), 61)])
    check_close(y[pick], ref[pick], TOL["bf16"], "double Flux-scale sampled rows")


@pytest.mark.parametrize("mode,policy,plan", [("kv", 1, None), ("y", 3, [1, 0, 1, 1]),
                                              ("kv", 3, [0, 0, 1, 1]), ("y", 2, None)])
def test_flux_stack_run_batch(F, mode, policy, plan):
    """A Flux-like stack (2 double-stream blocks, then 2 single-stream parallel blocks, R23 /
    R25) through fps_run_batch: 2 requests at different steps, 12H modulation rows."""
    g = synth.rng(7200)
    N, steps, H, heads, Fd, L_img, L_txt = 4, 3, 256, 2, 512, 256, 16
    L = L_img + L_txt
    W = [synth.block_weights(g, H, Fd, "bf16", "double") for _ in range(2)] + \
        [synth.block_weights(g, H, Fd, "bf16", "par") for _ in range(2)]
    mods = synth.mod_table(g, N, steps, H, "bf16", streams=2)
    deltas = synth.delta_table(steps)
    cache_np = [[{"K": synth.latent(g, L, H, "bf16"), "V": synth.latent(g, L, H, "bf16"),
                  "Y": synth.latent(g, L, H, "bf16")} for _ in range(N)] for _ in range(steps)]
    m = F.MODE_CODE[mode]
    cache = F.Cache(m, F.FPS_BF16, H, L_img, N, steps)
    for s in range(steps):
        for l in range(N):
            e = cache_np[s][l]
            cache.store(0, s, l, to_dev(np.concatenate([e["K"], e["V"]], 1) if mode == "kv"
                                        else e["Y"], "bf16"))
        if mode == "kv":
            cache.store(0, s, N, to_dev(cache_np[s][N - 1]["Y"], "bf16"))
    torch.cuda.synchronize()
    layers = [F.BlockWeights(w, heads, F.FPS_BF16) for w in W]
    eng = F.Engine(layers, heads, m, F.FPS_BF16, L_img, L_txt, max_batch=4, n_steps=steps,
                   deltas=deltas, cache=cache, mod_table=to_dev(mods, "bf16"), plan_policy=policy,
                   plan=plan, mod_width=12 * H)
    reqs = []
    for i, ratio in enumerate([0.1, 0.45]):
        mask = synth.token_mask(synth.mask_blobs(g, 16, 16, ratio), L_txt)
        x0 = synth.latent(g, L, H, "bf16")
        reqs.append(dict(template_id=0, step=i, n_steps=steps, mask=torch.as_tensor(mask).cuda(),
                         x=to_dev(x0, "bf16"), x0=x0, mask_np=mask, step0=i))
    eng.run_batch(reqs, 2)
    torch.cuda.synchronize()
    used = eng.last_plan()[0]
    # the parallel blocks read the first 6H of each (12H) modulation row
    mods_o = [[mods[l][s] if l < 2 else mods[l][s][:6 * H] for s in range(steps)] for l in range(N)]
    for r in reqs:
        n = min(2, steps - r["step0"])
        ref = S.masked_run(r["x0"], r["mask_np"], W, mods_o, deltas, used, mode, cache_np, heads,
                           n, step0=r["step0"], L_txt=L_txt)
        check_close(to_np(r["x"]), ref, stack_tol("bf16", N), f"Flux stack {mode} plan={used}")


def test_double_c4_continuous_batch(F):
    """configs[3] shapes on the double-stream block: 16 Flux-scale requests with masks 5-60 % in
    one varlen batch (grouped GEMMs over ~21k image and 8k text rows, one joint attention); the
    oracle checks the requests with the smallest and the largest mask, all rows."""
    H, heads, Fd, L_img, L_txt = 3072, 24, 12288, 4096, 512
    g = synth.rng(7300)
    w = synth.block_weights(g, H, Fd, "bf16", "double")
    reqs = []
    for m in np.linspace(0.05, 0.60, 16):
        mask = synth.token_mask(synth.mask_blobs(g, 64, 64, float(m)), L_txt)
        M, U = build_mask_index(mask)
        L = L_img + L_txt
        reqs.append(dict(mask=mask, M=M, U=U, L=L, x=synth.latent(g, L, H, "bf16"),
                         K=synth.latent(g, L, H, "bf16"), V=synth.latent(g, L, H, "bf16"),
                         mod=synth.mod_table(g, 1, 1, H, "bf16", streams=2)[0, 0]))
    y = _run(F, w, reqs, heads, "bf16", "kv", L_img)
    cu = np.concatenate([[0], np.cumsum([len(r["M"]) for r in reqs])])
    for i in (0, 15):
        ref = _ref(w, [reqs[i]], heads, "kv", L_txt)
        check_close(y[cu[i]:cu[i + 1]], ref, TOL["bf16"], f"C4 double request {i}")


@pytest.mark.parametrize("mode,flags", [("kv", 0), ("y", 0), ("kv", 16)])
def test_double_copy_path(F, mode, flags):
    """Without the inverse stream order (or with a forced one-tile attention kernel, which has no
    output row map) the block reorders its rows with explicit copies: same results."""
    w, reqs = _problem(7110, "bf16", 256, 2, 1024, 576, 40, [0.1, 0.5])
    F.fps_set_disable_tc(flags)
    try:
        y = _run(F, w, reqs, 2, "bf16", mode, 576, inv=flags != 0)
    finally:
        F.fps_set_disable_tc(0)
    check_close(y, _ref(w, reqs, 2, mode, 40), TOL["bf16"], f"double copy path {mode} {flags}")
