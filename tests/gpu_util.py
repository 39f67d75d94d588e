"""Helpers for the GPU parity tests (test infrastructure)."""
import numpy as np
import torch

import synth

TOL = {"bf16": 2e-2, "f32": 1e-5}          # BASELINE.json north_star tolerances (block outputs)


def stack_tol(dtype, n_blocks):
    """Tolerance for a latent after a chain of n_blocks blocks: the
    per-block bound grows like sqrt(n) because each block adds an independent rounding error to
    the bf16 residual stream; the fp32 path keeps 1e-5 per block, i.e. 1e-5 * n."""
    import math
    return TOL[dtype] * (math.sqrt(n_blocks) if dtype == "bf16" else n_blocks)


def to_dev(a, dtype):
    td = torch.bfloat16 if dtype == "bf16" else torch.float32
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.float32)).to("cuda").to(td)


def to_np(t):
    return t.detach().float().cpu().numpy().astype(np.float64)


def check_close(got, ref, tol, what=""):
    """Pass iff |g - r| <= tol * max(1, |r|) elementwise (reading R20)."""
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    assert got.shape == ref.shape, (what, got.shape, ref.shape)
    err = np.abs(got - ref) / np.maximum(1.0, np.abs(ref))
    worst = float(err.max()) if err.size else 0.0
    assert np.all(np.isfinite(got)), f"{what}: non-finite output"
    assert worst <= tol, (f"{what}: max scaled err {worst:.3e} > {tol} "
                          f"(max abs {np.abs(got - ref).max():.3e})")
    return worst


def bits(t):
    return t.detach().contiguous().view(torch.int16 if t.element_size() == 2 else torch.int32).cpu()
