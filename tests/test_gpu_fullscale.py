"""Parity at full Flux scale on the exact path the bench times (configs[2]: H 3072, 24 x 128
heads, MLP 12288, 4096 image + 512 text tokens, m = 0.2, blob masks):

* the single-stream (parallel) block -- 38 of the stack's 57 blocks, every cached block of the
  bench's plan -- against the oracle on sampled rows, KV and Y mode (fused W1 of 3H + F = 21504
  rows with the 3-region epilogue, W2 with K = H + F = 15360);
* the KV-mode transition block (R28) of a double-stream block followed by a cached
  single-stream block, through fps_run_batch with the bench's H2D settings (whole-entry DMA from
  pinned host on its own load stream, cross-step prefetch), against the oracle's dense-prefix
  plan on sampled rows;
* Flux's whole 57-block stack (19 double-stream + 38 single-stream blocks) over two steps with
  the bench's settings -- cache recorded by the engine's own template run, whole-entry DMA from
  pinned host, cross-step prefetch, transition block, the bench's plan shape -- bit-identical to
  the dense run when the request is the template (L144 / L157: masked rows computed from
  identical inputs in identical order reproduce the dense rows).
Sizes follow BASELINE.json configs[2]; the oracle checks rows one by one (PAPER.md L157, L161
§3.1; L211 §4.2)."""
import os
import sys

import numpy as np
import pytest
import torch

import synth
from oracle import block as B
from oracle.index import build_mask_index
from gpu_util import TOL, check_close, stack_tol, to_dev, to_np

pytestmark = pytest.mark.gpu

H, HEADS, FD, L_IMG, L_TXT = 3072, 24, 12288, 4096, 512
L = L_IMG + L_TXT


@pytest.fixture(scope="module")
def F():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as fps
    fps.require_gpu()
    return fps


def _sampled_block_rows(w, x_M, M, U, mod, sample, K_U=None, V_U=None, x_U=None):
    """Oracle block output on the sampled active rows (positions into M): fresh K|V of every
    active row (KV-mode) or of every row (Y-mode), queries of the sampled rows only."""
    h1_M = B._norm1(B.f64(x_M), w, mod, H)
    (Wq, bq), (Wk, bk), (Wv, bv) = B._qkv_weights(w, H)
    Kall, Vall = np.empty((L, H)), np.empty((L, H))
    Kall[M], Vall[M] = B.linear(h1_M, Wk, bk), B.linear(h1_M, Wv, bv)
    if x_U is None:
        Kall[U], Vall[U] = B.f64(K_U), B.f64(V_U)
    else:
        h1_U = B._norm1(B.f64(x_U), w, mod, H)
        Kall[U], Vall[U] = B.linear(h1_U, Wk, bk), B.linear(h1_U, Wv, bv)
    a = B.attention(B.linear(h1_M[sample], Wq, bq), Kall, Vall, HEADS)
    return B._block_out(B.f64(x_M)[sample], h1_M[sample], a, w, mod, H)


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_flux_scale_single_stream_block_sampled_rows(F, mode):
    from test_gpu_block import _run_masked
    g = synth.rng(6001 + (mode == "y"))
    w = synth.block_weights(g, H, FD, "bf16", "par")
    mask = synth.token_mask(synth.mask_blobs(g, 64, 64, 0.2), L_TXT)
    M, U = build_mask_index(mask)
    req = dict(mask=mask, M=M, U=U, L=L, x=synth.latent(g, L, H, "bf16"),
               K=synth.latent(g, L, H, "bf16"), V=synth.latent(g, L, H, "bf16"),
               xu=synth.latent(g, L, H, "bf16"), mod=synth.mod_table(g, 1, 1, H, "bf16")[0, 0])
    y, _ = _run_masked(F, w, [req], HEADS, "bf16", mode)
    # sampled active rows: both ends, text rows, and rows inside the ragged last tiles
    sample = np.unique(np.concatenate([g.choice(len(M), 36, replace=False),
                                       [0, 1, len(M) - 513, len(M) - 512, len(M) - 1],
                                       np.arange(1280, 1290)]))
    x = req["x"]
    if mode == "kv":
        ref = _sampled_block_rows(w, x[M], M, U, req["mod"], sample, K_U=req["K"][U], V_U=req["V"][U])
    else:
        ref = _sampled_block_rows(w, x[M], M, U, req["mod"], sample, x_U=req["xu"][U])
    check_close(y[sample], ref, TOL["bf16"], f"flux single-stream {mode}")


def _flux_engine(F, W_np, mods_np, cache, plan, deltas, cross_step=True, steps=1):
    layers = [F.BlockWeights(w, HEADS, F.FPS_BF16) for w in W_np]
    return F.Engine(layers, HEADS, F.FPS_MODE_KV, F.FPS_BF16, L_IMG, L_TXT, 1, steps,
                    deltas, cache, mod_table=to_dev(mods_np, "bf16"),
                    plan_policy=3, plan=plan, mod_width=12 * H, cross_step=cross_step)


def test_flux_scale_transition_block_sampled_rows(F):
    """Plan [dense, cached] over a double-stream block then a single-stream block: the
    double-stream block runs as the transition block (R28) -- K|V of every row of the fresh
    input, attention / O / MLP on the active rows only -- and the single-stream block reads its
    rows U's K|V from the pinned-host cache (whole-entry DMA on a load stream, cross-step on).
    Oracle: the dense-prefix plan (block 0 dense over all rows), checked on sampled rows M of
    the final latent, plus rows U (x0 + delta * cached Y)."""
    g = synth.rng(6010)
    W = [synth.block_weights(g, H, FD, "bf16", "double"), synth.block_weights(g, H, FD, "bf16", "par")]
    mods = synth.mod_table(g, 2, 1, H, "bf16", streams=2)
    mask = synth.token_mask(synth.mask_blobs(g, 64, 64, 0.2), L_TXT)
    M, U = build_mask_index(mask)
    x0 = synth.latent(g, L, H, "bf16")
    K1, V1, Yf = (synth.latent(g, L, H, "bf16") for _ in range(3))
    cache = F.Cache(F.FPS_MODE_KV, F.FPS_BF16, H, L_IMG, 2, 1, copy_method=2)
    cache.store(0, 0, 0, to_dev(np.concatenate([K1, V1], 1), "bf16"))      # unused by the plan
    cache.store(0, 0, 1, to_dev(np.concatenate([K1, V1], 1), "bf16"))
    cache.store(0, 0, 2, to_dev(Yf, "bf16"))
    torch.cuda.synchronize()
    # Euler coefficient +1 (R21's update with another coefficient): x0 + y keeps the check on the
    # stack output y itself; the schedule's -1/S at S = 1 would leave x0 - y = minus the two
    # blocks' residual increments, a cancellation that measures bf16 rounding of |y| instead
    delta = 1.0
    eng = _flux_engine(F, W, mods, cache, [0, 1], [delta])
    req = dict(template_id=0, step=0, n_steps=1, mask=torch.as_tensor(mask).cuda(), x=to_dev(x0, "bf16"))
    eng.run_batch([req], 1, load_stream=torch.cuda.Stream())
    torch.cuda.synchronize()
    assert eng.last_plan()[0] == [0, 1]
    got = to_np(req["x"])
    # block 0 over all rows, read on rows M only (the cached block after it takes rows U's K|V
    # from the cache): the dense block's rows M = the oracle's masked Y-mode block fed the fresh
    # input rows U (pinned by the oracle's all-ones / identical-input invariants)
    y0_M = B.masked_block_y(x0[M], M, U, x0[U], W[0], mods[0][0], HEADS, L, L_txt=L_TXT)
    sample = np.unique(np.concatenate([g.choice(len(M), 30, replace=False), [0, len(M) - 1],
                                       np.arange(len(M) - 512, len(M) - 505)]))
    y1 = _sampled_block_rows(W[1], y0_M, M, U, mods[1][0][:6 * H], sample, K_U=K1[U], V_U=V1[U])
    ref = B.f64(x0)[M][sample] + delta * y1
    check_close(got[M][sample], ref, stack_tol("bf16", 2), "transition block rows M")
    su = g.choice(len(U), 64, replace=False)
    check_close(got[U][su], B.f64(x0)[U][su] + delta * B.f64(Yf)[U][su], TOL["bf16"], "rows U")
    eng.close()
    cache.close()


@pytest.mark.parametrize("copy_method", [2, 3])
def test_flux_stack_57_blocks_bench_settings_bit_identical(F, copy_method):
    """Flux's stack (19 double-stream + 38 single-stream blocks) at configs[2] size, two steps.
    The template's cache is recorded by the engine's own dense run of the request
    (fps_engine_set_record); the mask-aware runs use the bench's settings -- whole-entry DMA
    from pinned host on a separate load stream, cross-step prefetch, the KV-mode transition
    block, a 20-block dense prefix + 37 cached blocks (the bench's plan shape) and the
    all-cached plan -- and must reproduce the dense run's latents bit for bit.  Also with the
    TMA row gather (copy method 3, reserved SMs)."""
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench
    dev = torch.device("cuda")
    steps, N = 2, 57
    w = dict(bench.WORKLOADS["C3"], block="flux", steps=steps)
    layers, mod, scratch = bench.build_engine_inputs(F, w, "kv", dev, 2, 0, 2)
    scratch.close()
    cache = F.Cache(F.FPS_MODE_KV, F.FPS_BF16, H, L_IMG, N, steps, n_templates=1,
                    copy_method=copy_method)
    mask = torch.as_tensor(synth.token_mask(synth.mask_blobs(synth.rng(57), 64, 64, 0.2), L_TXT)).to(dev)
    x0 = torch.randn(L, H, generator=torch.Generator(device=dev).manual_seed(58), device=dev).to(torch.bfloat16)
    deltas = synth.delta_table(steps)
    ls = torch.cuda.Stream()

    def run(policy, plan=None, record=False):
        eng = F.Engine(layers, HEADS, F.FPS_MODE_KV, F.FPS_BF16, L_IMG, L_TXT, 1, steps, deltas,
                       cache, mod_table=mod, plan_policy=policy, plan=plan, mod_width=12 * H,
                       cross_step=True)
        F.fps_engine_set_record(eng.h, int(record))
        req = dict(template_id=0, step=0, n_steps=steps, mask=mask, x=x0.clone())
        eng.run_batch([req], steps, load_stream=ls)
        torch.cuda.synchronize()
        used = eng.last_plan()[0]
        eng.close()
        return req["x"], used

    dense, _ = run(2, record=True)                    # the template run: fills the cache
    assert torch.isfinite(dense.float()).all()
    for policy, plan in ((3, [0] * 20 + [1] * 37), (1, None)):
        got, used = run(policy, plan)
        if plan:
            assert used == plan
        diff = (got.float() - dense.float()).abs().max().item()
        assert torch.equal(got.view(torch.int16), dense.view(torch.int16)), \
            f"plan {sum(used)} cached: max diff {diff}"
    cache.close()
