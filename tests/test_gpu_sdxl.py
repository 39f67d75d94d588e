"""GPU parity of the SDXL UNet transformer block (NEXT-2, reading R24: self-attention,
cross-attention to the prompt encoding, GEGLU) against the oracle, through the C ABI: block
level (dense, KV- and Y-mode over a heterogeneous varlen batch) and through fps_run_batch."""
import numpy as np
import pytest
import torch

import synth
from oracle import block as B
from oracle import stack as S
from oracle.index import build_mask_index
from gpu_util import TOL, bits, check_close, stack_tol, to_dev, to_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as fps
    fps.require_gpu()
    return fps


def test_geglu_pack_is_the_documented_permutation(F):
    """fps_geglu_pack moves rows only (bit-exact): packed row j of group k = j // 64 is value row
    32k + j % 64 (j % 64 < 32) or gate row F + 32k + j % 64 - 32."""
    g = synth.rng(6100)
    Fd, K = 160, 192
    w = to_dev(synth.latent(g, 2 * Fd, K, "bf16"), "bf16")
    b = to_dev(synth.latent(g, 1, 2 * Fd, "bf16")[0], "bf16")
    wp, bp = torch.empty_like(w), torch.empty_like(b)
    F.fps_geglu_pack(F.FPS_BF16, F.ptr(w), F.ptr(b), Fd, K, F.ptr(wp), F.ptr(bp),
                     F.stream_ptr())
    torch.cuda.synchronize()
    j = np.arange(2 * Fd)
    src = np.where(j % 64 < 32, 32 * (j // 64) + j % 64, Fd + 32 * (j // 64) + j % 64 - 32)
    assert torch.equal(bits(wp), bits(w)[torch.as_tensor(src)])
    assert torch.equal(bits(bp), bits(b)[torch.as_tensor(src)])


def _problem(seed, H, heads, Fd, L_img, ratios, L_ctx, D_ctx):
    g = synth.rng(seed)
    w = synth.block_weights(g, H, Fd, "bf16", "sdxl", D_ctx=D_ctx)
    reqs = []
    for i, m in enumerate(ratios):
        gh = int(np.sqrt(L_img))
        mask = synth.mask_blobs(g, gh, L_img // gh, m)
        M, U = build_mask_index(mask)
        reqs.append(dict(mask=mask, M=M, U=U, L=L_img,
                         x=synth.latent(g, L_img, H, "bf16"),
                         K=synth.latent(g, L_img, H, "bf16"), V=synth.latent(g, L_img, H, "bf16"),
                         xu=synth.latent(g, L_img, H, "bf16"),
                         ctx=synth.context(g, L_ctx[i], D_ctx, "bf16")))
    return w, reqs


def _run(F, w, reqs, heads, mode, dense=False):
    H = w["w_o"].shape[0]
    bw = F.BlockWeights(w, heads, F.FPS_BF16)
    ctx = to_dev(np.concatenate([r["ctx"] for r in reqs]), "bf16")
    ctx_kv = bw.context_kv(ctx)
    n_ctx = [r["ctx"].shape[0] for r in reqs]
    Ls = [r["L"] for r in reqs]
    cu_k = np.concatenate([[0], np.cumsum(Ls)])
    if dense:
        x = to_dev(np.concatenate([r["x"] for r in reqs]), "bf16")
        b = F.VarlenBatch(Ls, Ls, ctx_kv=ctx_kv, n_ctx=n_ctx)
        y, _ = F.dense_block_forward(bw, b, x)
        torch.cuda.synchronize()
        return to_np(y), to_np(ctx_kv)
    q_row = np.concatenate([r["M"] + cu_k[i] for i, r in enumerate(reqs)]).astype(np.int32)
    u_row = np.concatenate([r["U"] + cu_k[i] for i, r in enumerate(reqs)]).astype(np.int32)
    x_act = to_dev(np.concatenate([r["x"][r["M"]] for r in reqs]), "bf16")
    kv = torch.zeros(int(cu_k[-1]), 2 * H, dtype=torch.bfloat16, device="cuda")
    xu = None
    if mode == "kv":
        for i, r in enumerate(reqs):
            full = np.concatenate([r["K"], r["V"]], axis=1)
            kv[cu_k[i] + torch.as_tensor(r["U"]).long().cuda()] = to_dev(full[r["U"]], "bf16")
    else:
        xu = to_dev(np.concatenate([r["xu"] for r in reqs]), "bf16")
    qd, ud = torch.as_tensor(q_row).cuda(), torch.as_tensor(u_row).cuda()
    b = F.VarlenBatch([len(r["M"]) for r in reqs], Ls, q_row=qd, mode=F.MODE_CODE[mode],
                      u_row=ud, u_src=ud, n_unmasked=[len(r["U"]) for r in reqs],
                      ctx_kv=ctx_kv, n_ctx=n_ctx)
    y = F.masked_block_forward(bw, b, x_act, kv, xu=xu)
    torch.cuda.synchronize()
    return to_np(y), to_np(ctx_kv)


def _ref(w, reqs, heads, mode):
    out = []
    for r in reqs:
        if mode == "kv":
            y, _, _ = B.masked_block_kv(r["x"][r["M"]], r["M"], r["U"], r["K"][r["U"]],
                                        r["V"][r["U"]], w, None, heads, r["L"], r["ctx"])
        else:
            y = B.masked_block_y(r["x"][r["M"]], r["M"], r["U"], r["xu"][r["U"]], w, None, heads,
                                 r["L"], r["ctx"])
        out.append(y)
    return np.concatenate(out)


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_sdxl_masked_varlen_batch(F, mode):
    """Three requests with different masks (5-60 %) and prompt lengths (77, 20, 77: ragged
    cross-attention key sets) in one launch per kernel; d = 64 heads as in SDXL."""
    w, reqs = _problem(6200, 256, 4, 512, 576, [0.05, 0.6, 0.3], [77, 20, 77], 128)
    y, ctx_kv = _run(F, w, reqs, 4, mode)
    check_close(y, _ref(w, reqs, 4, mode), TOL["bf16"], f"SDXL {mode}")
    Kc, Vc = B.context_kv(reqs[0]["ctx"], w)
    check_close(ctx_kv[:77], np.concatenate([Kc, Vc], 1), TOL["bf16"], "context K|V")


def test_sdxl_dense_block(F):
    w, reqs = _problem(6201, 256, 4, 512, 256, [1.0, 1.0], [77, 77], 128)
    y, _ = _run(F, w, reqs, 4, "kv", dense=True)
    ref = np.concatenate([B.dense_block(r["x"], w, None, 4, r["ctx"])[0] for r in reqs])
    check_close(y, ref, TOL["bf16"], "SDXL dense")


def test_sdxl_scale_level_a(F):
    """SDXL-scale 64x64 level (C2A: C = 640, 10 heads of 64, GEGLU width 2560, prompt 77 x
    2048), batch 2 at 10 % / 30 % masks: several tiles and ragged tails on every GEMM."""
    w, reqs = _problem(6202, 640, 10, 2560, 4096, [0.1, 0.3], [77, 77], 2048)
    y, _ = _run(F, w, reqs, 10, "kv")
    check_close(y, _ref(w, reqs, 10, "kv"), TOL["bf16"], "SDXL C2A")


@pytest.mark.parametrize("mode,policy,plan", [("kv", 1, None), ("y", 3, [1, 0, 1]),
                                              ("kv", 3, [0, 1, 1])])
def test_sdxl_run_batch_matches_oracle(F, mode, policy, plan):
    g = synth.rng(6300)
    N, steps, H, heads, Fd, L_img, L_ctx, D_ctx = 3, 3, 256, 4, 512, 256, 77, 128
    W = synth.stack_weights(g, N, H, Fd, "bf16", "sdxl", D_ctx)
    deltas = synth.delta_table(steps)
    mods = [[None] * steps for _ in range(N)]
    cache_np = [[{"K": synth.latent(g, L_img, H, "bf16"), "V": synth.latent(g, L_img, H, "bf16"),
                  "Y": synth.latent(g, L_img, H, "bf16")} for _ in range(N)] for _ in range(steps)]
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
    eng = F.Engine(layers, heads, m, F.FPS_BF16, L_img, 0, max_batch=4, n_steps=steps,
                   deltas=deltas, cache=cache, plan_policy=policy, plan=plan, L_ctx=L_ctx)
    reqs = []
    for i, ratio in enumerate([0.1, 0.5]):
        mask = synth.mask_blobs(g, 16, 16, ratio)
        x0 = synth.latent(g, L_img, H, "bf16")
        ctx = synth.context(g, L_ctx, D_ctx, "bf16")
        reqs.append(dict(template_id=0, step=i, n_steps=steps, mask=torch.as_tensor(mask).cuda(),
                         x=to_dev(x0, "bf16"), ctx=to_dev(ctx, "bf16"), x0=x0, ctx_np=ctx,
                         mask_np=mask, step0=i))
    eng.run_batch(reqs, 2)
    torch.cuda.synchronize()
    used = eng.last_plan()[0]
    for r in reqs:
        n = min(2, steps - r["step0"])
        ref = S.masked_run(r["x0"], r["mask_np"], W, mods, deltas, used, mode, cache_np, heads,
                           n, step0=r["step0"], ctx=r["ctx_np"])
        check_close(to_np(r["x"]), ref, stack_tol("bf16", N), f"SDXL stack {mode} plan={used}")
