"""GPU parity of fps_run_batch (stack of N blocks, layer-ahead cache pipeline, step-level
continuous batching) against the oracle's masked_run, plus GPU-internal invariants."""
import numpy as np
import pytest
import torch

import synth
from oracle import sampler as SM
from oracle import stack as S
from gpu_util import TOL, check_close, stack_tol, to_dev, to_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as fps
    fps.require_gpu()
    return fps


def _setup(F, mode, dtype, plan_policy, plan=None, N=3, steps=3, H=256, heads=2, Fd=512,
           L_img=256, L_txt=16, n_req=3, slots=0, copy_method=0, seed=5000, location=0,
           kind="seq", cross_step=False, cost_model=(0.0, 0.0, 0.0, 0.0), sampler=0,
           copy_ctas=0):
    g = synth.rng(seed)
    W = synth.stack_weights(g, N, H, Fd, dtype, kind)
    mods = synth.mod_table(g, N, steps, H, dtype)
    deltas = synth.delta_table(steps)
    L = L_img + L_txt
    n_t = 2
    # template cache: random activations of the right shapes (both sides consume the same)
    cache_np = [[[{"K": synth.latent(g, L, H, dtype), "V": synth.latent(g, L, H, dtype),
                   "Y": synth.latent(g, L, H, dtype)} for _ in range(N)] for _ in range(steps)]
                for _ in range(n_t)]
    dt = F.DTYPE_CODE[dtype]
    m = F.MODE_CODE[mode]
    cache = F.Cache(m, dt, H, L_img, N, steps, n_templates=n_t, copy_method=copy_method,
                    location=location, copy_ctas=copy_ctas)
    for t in range(n_t):
        for s in range(steps):
            for l in range(N):
                e = cache_np[t][s][l]
                if mode == "kv":
                    cache.store(t, s, l, to_dev(np.concatenate([e["K"], e["V"]], 1), dtype))
                else:
                    cache.store(t, s, l, to_dev(e["Y"], dtype))
            if mode == "kv":
                cache.store(t, s, N, to_dev(cache_np[t][s][N - 1]["Y"], dtype))
    torch.cuda.synchronize()
    layers = [F.BlockWeights(w, heads, dt) for w in W]
    eng = F.Engine(layers, heads, m, dt, L_img, L_txt, max_batch=4, n_steps=steps, deltas=deltas,
                   cache=cache, mod_table=to_dev(mods, dtype), slots=slots,
                   plan_policy=plan_policy, plan=plan, cross_step=cross_step,
                   cost_model=cost_model, sampler=sampler,
                   sigmas=SM.flow_sigmas(steps, 3.0) if sampler else None)
    reqs = []
    ratios = [0.1, 0.45, 0.25, 0.6][:n_req]
    for i in range(n_req):
        mask = synth.token_mask(synth.mask_blobs(g, 16, 16, ratios[i]), L_txt)
        x0 = synth.latent(g, L, H, dtype)
        reqs.append(dict(template_id=i % n_t, step=i % 2, n_steps=steps, mask_np=mask, x0=x0,
                         mask=torch.as_tensor(mask).cuda(), x=to_dev(x0, dtype)))
        if sampler:      # flow-blend sampler (R29): the request's template latent and noise
            z, eps = synth.latent(g, L_img, H, dtype), synth.latent(g, L_img, H, dtype)
            reqs[-1].update(z_np=z, eps_np=eps, z=to_dev(z, dtype), noise=to_dev(eps, dtype))
    return W, mods, deltas, cache_np, eng, reqs


def _oracle(W, mods, deltas, cache_np, reqs, plan, mode, heads, steps_run):
    outs = []
    for r in reqs:
        s0 = r["step0"]
        n = min(steps_run, r["n_steps"] - s0)
        x = S.masked_run(r["x0"], r["mask_np"], W, mods, deltas, plan, mode,
                         cache_np[r["template_id"]], heads, n, step0=s0)
        outs.append(x)
    return outs


@pytest.mark.parametrize("mode,dtype,policy,plan", [
    ("kv", "bf16", 1, None), ("y", "bf16", 1, None), ("kv", "f32", 1, None),
    ("y", "f32", 3, [1, 0, 1]), ("kv", "bf16", 3, [0, 1, 1]), ("y", "bf16", 3, [0, 1, 0]),
    ("kv", "bf16", 2, None)])
def test_run_batch_matches_oracle(F, mode, dtype, policy, plan):
    W, mods, deltas, cache_np, eng, reqs = _setup(F, mode, dtype, policy, plan)
    for r in reqs:
        r["step0"] = r["step"]
    eng.run_batch(reqs, 2)
    torch.cuda.synchronize()
    used = eng.last_plan()[0]
    if policy == 1:
        assert used == [1, 1, 1]
    if policy == 3:
        assert used == plan
    ref = _oracle(W, mods, deltas, cache_np, reqs, used, mode, 2, 2)
    for r, x in zip(reqs, ref):
        check_close(to_np(r["x"]), x, stack_tol(dtype, 3), f"{mode} {dtype} plan={used}")
        assert r["step"] == min(r["step0"] + 2, r["n_steps"])


@pytest.mark.parametrize("mode,dtype,policy,plan", [
    ("kv", "bf16", 1, None), ("y", "bf16", 3, [1, 0, 1]), ("kv", "f32", 3, [0, 1, 1])])
def test_run_batch_parallel_blocks(F, mode, dtype, policy, plan):
    """A stack of parallel (Flux single-stream) blocks through fps_run_batch (NEXT-2, R23)."""
    W, mods, deltas, cache_np, eng, reqs = _setup(F, mode, dtype, policy, plan, kind="par")
    for r in reqs:
        r["step0"] = r["step"]
    eng.run_batch(reqs, 2)
    torch.cuda.synchronize()
    used = eng.last_plan()[0]
    ref = _oracle(W, mods, deltas, cache_np, reqs, used, mode, 2, 2)
    for r, x in zip(reqs, ref):
        check_close(to_np(r["x"]), x, stack_tol(dtype, 3), f"parallel {mode} {dtype} plan={used}")


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_degenerate_masks_in_one_batch(F, mode):
    """Continuous batch mixing an empty mask (no masked image token: only text rows active), a
    full mask (every row active: no cache rows), tiny and large masks, and requests at different
    steps -- one varlen launch per kernel."""
    g = synth.rng(5400)
    N, steps, H, heads, Fd, L_img, L_txt = 2, 3, 256, 2, 512, 256, 16
    L = L_img + L_txt
    W = synth.stack_weights(g, N, H, Fd, "bf16")
    mods = synth.mod_table(g, N, steps, H, "bf16")
    deltas = synth.delta_table(steps)
    cache_np = [[{"K": synth.latent(g, L, H, "bf16"), "V": synth.latent(g, L, H, "bf16"),
                  "Y": synth.latent(g, L, H, "bf16")} for _ in range(N)] for _ in range(steps)]
    m = F.MODE_CODE[mode]
    cache = F.Cache(m, F.FPS_BF16, H, L_img, N, steps, n_templates=1)
    for s in range(steps):
        for l in range(N):
            e = cache_np[s][l]
            cache.store(0, s, l, to_dev(np.concatenate([e["K"], e["V"]], 1) if mode == "kv"
                                        else e["Y"], "bf16"))
        if mode == "kv":
            cache.store(0, s, N, to_dev(cache_np[s][N - 1]["Y"], "bf16"))
    torch.cuda.synchronize()
    layers = [F.BlockWeights(w, heads, F.FPS_BF16) for w in W]
    eng = F.Engine(layers, heads, m, F.FPS_BF16, L_img, L_txt, 6, steps, deltas, cache,
                   mod_table=to_dev(mods, "bf16"), plan_policy=1)
    reqs = []
    for i, ratio in enumerate([0.0, 1.0, 1 / 256, 0.6, 0.3, 0.05]):
        mask = synth.token_mask(synth.mask_random(g, L_img, ratio), L_txt)
        x0 = synth.latent(g, L, H, "bf16")
        reqs.append(dict(template_id=0, step=i % 3 if i % 3 < 2 else 0, n_steps=steps,
                         mask_np=mask, x0=x0, mask=torch.as_tensor(mask).cuda(),
                         x=to_dev(x0, "bf16")))
    for r in reqs:
        r["step0"] = r["step"]
    eng.run_batch(reqs, 1)
    torch.cuda.synchronize()
    for r in reqs:
        ref = S.masked_run(r["x0"], r["mask_np"], W, mods, deltas, [1] * N, mode, cache_np, heads,
                           1, step0=r["step0"])
        check_close(to_np(r["x"]), ref, stack_tol("bf16", N), f"{mode} n={r['mask_np'].sum()}")


def test_requests_leave_at_step_boundary(F):
    """A request reaching its last step leaves; the others keep running (L237)."""
    W, mods, deltas, cache_np, eng, reqs = _setup(F, "kv", "bf16", 1, steps=3)
    for r in reqs:
        r["step0"] = r["step"]
    eng.run_batch(reqs, 3)
    torch.cuda.synchronize()
    assert [r["status"] for r in reqs] == [1, 1, 1]
    assert [r["step"] for r in reqs] == [3, 3, 3]
    ref = _oracle(W, mods, deltas, cache_np, reqs, [1, 1, 1], "kv", 2, 3)
    for r, x in zip(reqs, ref):
        check_close(to_np(r["x"]), x, stack_tol("bf16", 3), "leave")


@pytest.mark.parametrize("slots,method,location", [(1, 0, 0), (2, 1, 0), (0, 0, 0), (2, 0, 1),
                                                  (0, 2, 1), (1, 2, 1), (2, 2, 0), (0, 3, 0),
                                                  (1, 3, 0), (2, 3, 0)])
def test_pipeline_slots_and_copy_methods_bit_identical(F, slots, method, location):
    """The staging ring depth, the H2D method and the cache tier (pinned host / HBM) change
    timing only, never the bits."""
    outs = []
    for sl, me, lo in ((0, 0, 0), (slots, method, location)):
        _, _, _, _, eng, reqs = _setup(F, "kv", "bf16", 1, slots=sl, copy_method=me, seed=5100,
                                       location=lo)
        # the second run on its own load stream (method 3 then reserves its SMs)
        eng.run_batch(reqs, 2, load_stream=torch.cuda.Stream() if sl == slots else None)
        torch.cuda.synchronize()
        outs.append([r["x"].clone() for r in reqs])
    for a, b in zip(*outs):
        assert torch.equal(a.view(torch.int16), b.view(torch.int16))


@pytest.mark.parametrize("mode,slots", [("kv", 2), ("y", 2), ("kv", 1)])
def test_batched_run_dma_bit_identical(F, mode, slots):
    """copy_method 1 on a real load stream goes through one cudaMemcpyAsync per run of
    consecutive unmasked rows; with a shallow staging ring the slot reuse must still be ordered."""
    outs = []
    for me, use_ls in ((0, False), (1, True)):
        _, _, _, _, eng, reqs = _setup(F, mode, "bf16", 1, slots=slots if me else 0,
                                       copy_method=me, seed=5150)
        ls = torch.cuda.Stream() if use_ls else None
        eng.run_batch(reqs, 2, load_stream=ls)
        torch.cuda.synchronize()
        outs.append([r["x"].clone() for r in reqs])
    for a, b in zip(*outs):
        assert torch.equal(a.view(torch.int16), b.view(torch.int16))


@pytest.mark.parametrize("mode,method,location", [("y", 0, 0), ("kv", 0, 0), ("kv", 2, 1),
                                                  ("y", 2, 1), ("kv", 1, 0), ("y", 1, 0),
                                                  ("kv", 2, 0), ("y", 2, 0), ("kv", 3, 0),
                                                  ("y", 3, 0)])
def test_delayed_load_stream_bit_identical(F, mode, method, location):
    """Robustness of the event ordering: a busy load stream (a long spin queued before the
    prefetches) must not change the result -- in particular a late whole-entry DMA (method 2)
    must not land on fresh K/V rows."""
    _, _, _, _, eng, reqs = _setup(F, mode, "bf16", 1, seed=5200, copy_method=method,
                                   location=location)
    eng.run_batch(reqs, 2)
    torch.cuda.synchronize()
    ref = [r["x"].clone() for r in reqs]
    _, _, _, _, eng, reqs = _setup(F, mode, "bf16", 1, seed=5200, copy_method=method,
                                   location=location)
    ls = torch.cuda.Stream()
    with torch.cuda.stream(ls):
        torch.cuda._sleep(200_000_000)          # ~0.1 s of spinning on the load stream
    eng.run_batch(reqs, 2, load_stream=ls)
    torch.cuda.synchronize()
    for a, r in zip(ref, reqs):
        assert torch.equal(a.view(torch.int16), r["x"].view(torch.int16))


@pytest.mark.parametrize("mode,ctas,prio", [("kv", 8, -5), ("y", 8, -5), ("kv", 6, 0)])
def test_row_gather_wide_high_priority_bit_identical(F, mode, ctas, prio):
    """configs[3]'s H2D setting: the TMA row gather on 8 CTAs (8 reserved SMs, compute grids on
    the other 140) from a high-priority load stream, cross-step prefetch on, gives the bits of
    the SM row gather (method 0) without a load stream."""
    outs = []
    for me, ct, use_ls in ((0, 0, False), (3, ctas, True)):
        _, _, _, _, eng, reqs = _setup(F, mode, "bf16", 1, copy_method=me, seed=5250,
                                       copy_ctas=ct, cross_step=True)
        ls = torch.cuda.Stream(priority=prio) if use_ls else None
        eng.run_batch(reqs, 3, load_stream=ls)
        torch.cuda.synchronize()
        outs.append([r["x"].clone() for r in reqs])
    for a, b in zip(*outs):
        assert torch.equal(a.view(torch.int16), b.view(torch.int16))


def test_identical_input_cache_gpu_internal_invariant(F):
    """L144/L157 on the GPU: store the GPU's own dense-run activations as the cache; the masked
    run on the identical input reproduces the dense run's latents bit-for-bit (token-wise
    kernels have row-independent arithmetic, attention sees the same keys in the same order)."""
    g = synth.rng(5300)
    N, steps, H, heads, Fd, L_img, L_txt = 3, 1, 256, 2, 512, 256, 16
    L = L_img + L_txt
    W = synth.stack_weights(g, N, H, Fd, "bf16")
    mods = synth.mod_table(g, N, steps, H, "bf16")
    dt = F.FPS_BF16
    layers = [F.BlockWeights(w, heads, dt) for w in W]
    x0 = synth.latent(g, L, H, "bf16")
    mask = synth.token_mask(synth.mask_blobs(g, 16, 16, 0.3), L_txt)
    for mode in ("kv", "y"):
        m = F.MODE_CODE[mode]
        # dense template run on the GPU, one block at a time, capturing K|V and Y
        b = F.VarlenBatch([L], [L], mod=None)
        cache = F.Cache(m, dt, H, L_img, N, steps, n_templates=1)
        cur = to_dev(x0, "bf16")
        for l in range(N):
            bl = F.VarlenBatch([L], [L], mod=to_dev(mods[l, 0][None], "bf16"))
            y, kv = F.dense_block_forward(layers[l], bl, cur)
            cache.store(0, 0, l, kv if mode == "kv" else y)
            cur = y
        if mode == "kv":
            cache.store(0, 0, N, cur)
        torch.cuda.synchronize()
        outs = []
        for policy in (1, 2):          # all blocks cached vs all blocks dense (no cache)
            eng = F.Engine(layers, heads, m, dt, L_img, L_txt, 1, steps, synth.delta_table(steps),
                           cache, mod_table=to_dev(mods, "bf16"), plan_policy=policy)
            req = dict(template_id=0, step=0, n_steps=steps, mask=torch.as_tensor(mask).cuda(),
                       x=to_dev(x0, "bf16"))
            eng.run_batch([req], 1)
            torch.cuda.synchronize()
            outs.append(req["x"].clone())
        diff = (outs[0].float() - outs[1].float()).abs().max().item()
        assert torch.equal(outs[0].view(torch.int16), outs[1].view(torch.int16)), f"{mode}: {diff}"


def test_hbm_whole_entry_loads_with_dense_prefix_complete():
    """Regression: HBM-tier whole-entry loads under a plan with a dense prefix (C2B stack,
    21 dense + 39 cached blocks).  Issued as driver device-to-device memcpys next to the PDL
    compute chain this hung on the first step; the library copy kernel must complete.  Runs in
    a subprocess so a hang fails the test instead of stalling the suite."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    p = subprocess.run([sys.executable, os.path.join(root, "tools", "hang_probe.py"), "C2B", "kv",
                        "1", "2", "21", "3"], capture_output=True, text=True, timeout=180)
    assert p.returncode == 0 and "DONE" in p.stdout, p.stdout[-2000:] + p.stderr[-2000:]


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_full_scale_stack_identical_input_invariant(F, mode):
    """configs[2] at its full size (57 Flux-scale blocks, 4096 + 512 tokens, m = 0.2): with the
    cache taken from the GPU's own dense template run on the identical input, the mask-aware
    step (every block cached) reproduces the dense step bit-for-bit -- a property that holds at
    any size (L144/L157), checked where the fp64 oracle cannot run the whole stack.  So does
    the bench's plan shape (uncached prefix, cached suffix)."""
    H, heads, Fd, L_img, L_txt, N, steps = 3072, 24, 12288, 4096, 512, 57, 1
    L = L_img + L_txt
    dev = torch.device("cuda")
    gen = torch.Generator(device=dev).manual_seed(57)
    rnd = lambda *s, sc=1.0: (torch.randn(*s, generator=gen, device=dev) * sc).to(torch.bfloat16)
    dt = F.FPS_BF16
    layers = []
    for _ in range(N):
        t = {"w_qkv": rnd(3 * H, H, sc=H ** -0.5), "b_qkv": rnd(3 * H, sc=0.02),
             "w_o": rnd(H, H, sc=H ** -0.5), "b_o": rnd(H, sc=0.02),
             "w_up": rnd(Fd, H, sc=H ** -0.5), "b_up": rnd(Fd, sc=0.02),
             "w_down": rnd(H, Fd, sc=Fd ** -0.5), "b_down": rnd(H, sc=0.02)}
        bw = F.BlockWeights.__new__(F.BlockWeights)
        bw.t, bw.H, bw.F, bw.heads, bw.dtype, bw.kind = t, H, Fd, heads, dt, 0
        bw.c = F.fps_block_weights(H, heads, H // heads, Fd, dt,
                                   *[t[k].data_ptr() for k in ("w_qkv", "b_qkv", "w_o", "b_o",
                                                               "w_up", "b_up", "w_down", "b_down")], 0)
        layers.append(bw)
    mods = (0.02 * torch.randn(N, steps, 6, H, generator=gen, device=dev))
    mods[:, :, 2] += 1.0
    mods[:, :, 5] += 1.0
    mods = mods.reshape(N, steps, 6 * H).to(torch.bfloat16)
    x0 = torch.randn(L, H, generator=gen, device=dev).to(torch.bfloat16)
    mask = synth.token_mask(synth.mask_blobs(synth.rng(57), 64, 64, 0.2), L_txt)
    m = F.MODE_CODE[mode]
    cache = F.Cache(m, dt, H, L_img, N, steps, n_templates=1)
    cur = x0.clone()
    for l in range(N):
        bl = F.VarlenBatch([L], [L], mod=mods[l, 0][None].contiguous())
        y, kv = F.dense_block_forward(layers[l], bl, cur)
        cache.store(0, 0, l, kv if mode == "kv" else y)
        cur = y
    if mode == "kv":
        cache.store(0, 0, N, cur)
    torch.cuda.synchronize()
    outs = []
    # every block cached, a 15-block uncached prefix (the bench's C3 plan: in KV-mode its last
    # block is the transition block, R28), every block dense (the reference, last)
    prefix = [0] * 15 + [1] * (N - 15)
    for policy in (1, 3, 2):
        eng = F.Engine(layers, heads, m, dt, L_img, L_txt, 1, steps, synth.delta_table(steps),
                       cache, mod_table=mods, plan_policy=policy,
                       plan=prefix if policy == 3 else None)
        req = dict(template_id=0, step=0, n_steps=steps, mask=torch.as_tensor(mask).cuda(),
                   x=x0.clone())
        eng.run_batch([req], 1)
        torch.cuda.synchronize()
        outs.append(req["x"].clone())
        eng.close()
    cache.close()
    for o in outs[:2]:
        assert torch.isfinite(o.float()).all()
        assert torch.equal(o.view(torch.int16), outs[2].view(torch.int16)), \
            f"{mode}: max diff {(o.float() - outs[2].float()).abs().max().item()}"


@pytest.mark.parametrize("mode,plan,copy_method", [("kv", [0, 1, 1], 1), ("y", [1, 0, 1], 0),
                                                   ("kv", [1, 1, 1], 2), ("y", [1, 1, 1], 1),
                                                   ("kv", [0, 1, 1], 3), ("y", [1, 0, 1], 3)])
def test_cross_step_prefetch_matches_oracle_and_per_step_bits(F, mode, plan, copy_method):
    """Cross-step prefetch (R26) only moves loads earlier: over 2 steps the latents match the
    oracle and are bit-identical to the per-step pipeline's."""
    outs = []
    for cross in (False, True):
        W, mods, deltas, cache_np, eng, reqs = _setup(F, mode, "bf16", 3, plan, steps=4,
                                                      copy_method=copy_method, cross_step=cross)
        for r in reqs:
            r["step0"] = r["step"]
        eng.run_batch(reqs, 2, load_stream=torch.cuda.Stream())
        torch.cuda.synchronize()
        outs.append([r["x"].clone() for r in reqs])
        ref = _oracle(W, mods, deltas, cache_np, reqs, plan, mode, 2, 2)
        for r, x in zip(reqs, ref):
            check_close(to_np(r["x"]), x, stack_tol("bf16", 3),
                        f"cross={cross} {mode} plan={plan}")
    for a, b in zip(*outs):
        assert torch.equal(a, b)


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_admission_reuse_step_by_step(F, mode):
    """A serving loop advancing the batch one step per call (the same requests each call) reuses
    the first call's admission -- no mask-index launch, no host sync -- and produces bit-identical
    latents to one multi-step call; a changed request set is re-admitted."""
    import ctypes as C
    outs = []
    for per_call in (False, True):
        W, mods, deltas, cache_np, eng, reqs = _setup(F, mode, "bf16", 1, None, steps=4,
                                                      cross_step=True)
        for r in reqs:
            r["step"] = 0
        if per_call:
            F.fps_profile_enable(1)
            for _ in range(3):
                eng.run_batch(reqs, 1)
            torch.cuda.synchronize()
            cnt = np.zeros(7, dtype=np.int64)
            F.fps_profile_read(None, None, None, cnt.ctypes.data_as(C.POINTER(C.c_int64)))
            F.fps_profile_enable(0)
            assert cnt[6] == 1, f"mask index launched {cnt[6]} times for one batch"
        else:
            eng.run_batch(reqs, 3)
        torch.cuda.synchronize()
        outs.append([r["x"].clone() for r in reqs])
    for a, b in zip(*outs):
        assert torch.equal(a, b)
    # a different request set (one request dropped) is admitted again and still matches the oracle
    sub = reqs[:2]
    for r in sub:
        r["step0"] = r["step"]
    F.fps_profile_enable(1)
    eng.run_batch(sub, 1)
    torch.cuda.synchronize()
    cnt = np.zeros(7, dtype=np.int64)
    F.fps_profile_read(None, None, None, cnt.ctypes.data_as(C.POINTER(C.c_int64)))
    F.fps_profile_enable(0)
    assert cnt[6] == 1


@pytest.mark.parametrize("kind", ["seq", "par"])
@pytest.mark.parametrize("plan", [[0, 0, 1, 1], [0, 1, 1, 1]])
def test_kv_transition_block_matches_oracle_and_dense_run(F, kind, plan):
    """KV-mode transition block (R28): the last uncached block before the cached suffix runs as
    a masked block over the fresh full input.  With it on (default) and off (dense), the latents
    match the oracle's plan (whose uncached blocks are dense over all rows) and each other."""
    outs = []
    for on in (1, 0):
        W, mods, deltas, cache_np, eng, reqs = _setup(F, "kv", "bf16", 3, plan, N=4, kind=kind)
        F.fps_engine_set_kv_transition(eng.h, on)
        for r in reqs:
            r["step0"] = r["step"]
        eng.run_batch(reqs, 2)
        torch.cuda.synchronize()
        assert eng.last_plan()[0] == plan
        ref = _oracle(W, mods, deltas, cache_np, reqs, plan, "kv", 2, 2)
        for r, x in zip(reqs, ref):
            check_close(to_np(r["x"]), x, stack_tol("bf16", 4), f"transition={on} {kind} {plan}")
        outs.append([to_np(r["x"]) for r in reqs])
    for a, b in zip(*outs):
        check_close(a, b, stack_tol("bf16", 4), "transition on vs off")


@pytest.mark.parametrize("cross", [False, True])
def test_kv_transition_planner_prices_each_suffix(F, cross):
    """With the transition block (R28) the engine's KV-mode planner prices every suffix plan
    with its prefix's last block at the transition cost (Y-mode FLOPs over the fresh input):
    its plan and latency are the argmin of the library's pipeline model over the N+1 suffixes
    with those cost vectors; off, it is the library planner's."""
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched as Sd
    N, H, Fd, L_img, L_txt = 6, 256, 512, 256, 16
    L = L_img + L_txt
    cm = (1.0e-9, 0.01, 1.3e-6, 0.01)      # ms / FLOP, ms, ms / byte, ms: a dense-prefix optimum
    for on in (1, 0):
        W, mods, deltas, cache_np, eng, reqs = _setup(F, "kv", "bf16", 0, None, N=N,
                                                      cross_step=cross, cost_model=cm)
        F.fps_engine_set_kv_transition(eng.h, on)
        eng.run_batch(reqs, 1)
        torch.cuda.synchronize()
        plan, lat = eng.last_plan()
        nq = [int(r["mask_np"].sum()) for r in reqs]
        Cw = [cm[0] * sum(Sd.block_flops("kv", n, L, H, Fd) for n in nq) + cm[1]] * N
        Cwo = [cm[0] * sum(Sd.block_flops("dense", n, L, H, Fd) for n in nq) + cm[1]] * N
        Ct = cm[0] * sum(Sd.block_flops("y", n, L, H, Fd) for n in nq) + cm[1]
        nu = sum(L - n for n in nq)
        Lm = [cm[2] * nu * 2 * H * 2 + cm[3]] * N
        fin = cm[2] * nu * H * 2 + cm[3]
        best = None
        for kc in range(N + 1):               # k cached blocks; ties -> fewer cached
            k = N - kc
            use = [0] * k + [1] * (N - k)
            C2 = list(Cwo)
            if on and 0 < k < N:
                C2[k - 1] = Ct
            t = F.pipeline_latency(use, Cw, C2, Lm, F.FPS_MODE_KV, fin, cross_step=cross)
            if best is None or t < best[0] - 1e-12 * max(1.0, abs(best[0])):
                best = (t, use)
        if not on:
            ref_plan, ref_lat = F.plan_pipeline(Cw, Cwo, Lm, F.FPS_MODE_KV, fin, cross_step=cross)
            assert list(ref_plan) == best[1] and ref_lat == pytest.approx(best[0], rel=1e-9)
        if on:
            lib_plan, lib_lat = F.plan_pipeline_kv_transition(Cw, Cwo, [Ct] * N, Lm, fin,
                                                              cross_step=cross)
            assert lib_plan == best[1] and lib_lat == pytest.approx(best[0], rel=1e-9)
        assert plan == best[1], (on, plan, best)
        assert 0 < sum(plan) < N, plan
        assert lat == pytest.approx(best[0], rel=1e-9)


@pytest.mark.parametrize("mode,dtype,policy,plan", [
    ("kv", "bf16", 1, None), ("y", "bf16", 3, [1, 0, 1]), ("kv", "f32", 3, [0, 1, 1]),
    ("y", "f32", 1, None)])
def test_flow_blend_sampler_matches_oracle(F, mode, dtype, policy, plan):
    """NEXT-4 / R29: the flow-matching Euler sampler with inpainting blend after the stack --
    masked image rows x += (sigma_{s+1} - sigma_s) y, unmasked image rows reset to the template
    latent re-noised to sigma_{s+1}, text rows kept -- each request at its own step, over two
    steps of a continuous batch, against the oracle's masked_run with the same sampler."""
    W, mods, deltas, cache_np, eng, reqs = _setup(F, mode, dtype, policy, plan, sampler=1)
    for r in reqs:
        r["step0"] = r["step"]
    eng.run_batch(reqs, 2, load_stream=torch.cuda.Stream())
    torch.cuda.synchronize()
    used = eng.last_plan()[0]
    sig = SM.flow_sigmas(3, 3.0)
    for r in reqs:
        s0 = r["step0"]
        n = min(2, r["n_steps"] - s0)
        ref = S.masked_run(r["x0"], r["mask_np"], W, mods, deltas, used, mode,
                           cache_np[r["template_id"]], 2, n, step0=s0, L_txt=16,
                           sampler={"sigmas": sig, "z": r["z_np"], "eps": r["eps_np"]})
        got = to_np(r["x"])
        check_close(got, ref, stack_tol(dtype, 3), f"flow-blend {mode} {dtype} plan={used}")
        # after the schedule's last step the unmasked image rows ARE the template latent
        if s0 + n == r["n_steps"]:
            U = np.flatnonzero(r["mask_np"][:256] == 0)
            assert np.array_equal(got[U], to_np(r["z"])[U])


def test_flow_blend_sampler_needs_template_latent(F):
    W, mods, deltas, cache_np, eng, reqs = _setup(F, "kv", "bf16", 1, None, sampler=1)
    del reqs[0]["noise"]
    with pytest.raises(F.FlashPSError):
        eng.run_batch(reqs, 1)


@pytest.mark.parametrize("mode", ["kv", "y"])
def test_record_cache_is_the_template_run(F, mode):
    """fps_engine_set_record: a dense engine run stores each block's K|V (KV-mode) or output
    (Y-mode) rows -- and KV-mode's final Y -- as the template's cache entries of that step;
    they match the oracle's template run, and a masked run of the same request against them
    reproduces the dense run bit for bit (L130 / L203: the cache is the template's prior full
    inference)."""
    g = synth.rng(5600)
    N, steps, Hh, heads, Fd, L_img, L_txt = 3, 2, 256, 2, 512, 256, 16
    L = L_img + L_txt
    W = synth.stack_weights(g, N, Hh, Fd, "bf16")
    mods = synth.mod_table(g, N, steps, Hh, "bf16")
    deltas = synth.delta_table(steps)
    m = F.MODE_CODE[mode]
    cache = F.Cache(m, F.FPS_BF16, Hh, L_img, N, steps, n_templates=1)
    layers = [F.BlockWeights(w, heads, F.FPS_BF16) for w in W]
    x0 = synth.latent(g, L, Hh, "bf16")
    mask = synth.token_mask(synth.mask_blobs(g, 16, 16, 0.3), L_txt)
    outs = []
    for policy, record in ((2, 1), (1, 0)):
        eng = F.Engine(layers, heads, m, F.FPS_BF16, L_img, L_txt, 1, steps, deltas, cache,
                       mod_table=to_dev(mods, "bf16"), plan_policy=policy, cross_step=True)
        F.fps_engine_set_record(eng.h, record)
        req = dict(template_id=0, step=0, n_steps=steps, mask=torch.as_tensor(mask).cuda(),
                   x=to_dev(x0, "bf16"))
        eng.run_batch([req], steps, load_stream=torch.cuda.Stream())
        torch.cuda.synchronize()
        outs.append(req["x"].clone())
        eng.close()
    assert torch.equal(outs[0].view(torch.int16), outs[1].view(torch.int16))
    ref_cache, _ = S.template_run(x0, W, mods, deltas, heads, steps)
    for s in range(steps):
        for l in range(N + (1 if mode == "kv" else 0)):
            e = cache.entry_numpy(0, s, l)
            got = torch.as_tensor(e.view(np.int16)).view(torch.bfloat16).float().numpy()
            if l == N:
                ref = ref_cache[s][N - 1]["Y"][:L_img]
            elif mode == "kv":
                ref = np.concatenate([ref_cache[s][l]["K"], ref_cache[s][l]["V"]], 1)[:L_img]
            else:
                ref = ref_cache[s][l]["Y"][:L_img]
            check_close(got, ref, stack_tol("bf16", (l + 1) + s * N), f"{mode} entry ({s},{l})")
    cache.close()
