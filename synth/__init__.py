"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the FlashPS method: it only draws random numbers (numpy
PCG64), rounds them to the storage precision, and shapes them like the paper's workloads
(DESIGN.md "Input recipe"). Both sides of every parity test consume exactly these arrays; the
oracle (`oracle/`) and the CUDA path (`paper_conf_eurosys_jianglyfdlzllyl26_b200/`) never
import each other.

Shapes follow SURVEY.md §8(d):
  * weights ~ N(0, 1/fan_in), biases ~ N(0, 0.02^2), bf16-rounded when dtype == "bf16";
  * adaLN vectors per (layer, step): shift, scale ~ N(0, 0.02^2), gate ~ 1 + N(0, 0.02^2);
  * latents x ~ N(0, 1);
  * masks: exact-count uniform-random, or "blobs" (a smooth random field thresholded at the
    exact count), "no assumption of the shape of masks";
  * mask ratios for serving sweeps ~ Beta(2, 8.5) (mean 0.19, public trace).
Text tokens (Flux joint attention) are appended AFTER the image tokens and are always active
(reading R9).
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

__all__ = [
    "rng", "bf16_round", "BlockDims", "CONFIGS", "block_weights", "stack_weights", "mod_table",
    "delta_table", "latent", "context", "mask_random", "mask_blobs", "token_mask", "n_masked_for",
    "sample_mask_ratios",
]


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def bf16_round(a) -> np.ndarray:
    """Round float32 values to the nearest bf16 (ties to even); returned as float32."""
    a = np.ascontiguousarray(np.asarray(a, dtype=np.float32))
    u = a.view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) >> 16 << 16
    return u.astype(np.uint32).view(np.float32).reshape(a.shape)


def _store(a: np.ndarray, dtype: str) -> np.ndarray:
    a = a.astype(np.float32)
    return bf16_round(a) if dtype == "bf16" else a


@dataclasses.dataclass(frozen=True)
class BlockDims:
    """One transformer block: hidden H, `heads` x `head_dim`, MLP width F, tokens L_img + L_txt."""
    H: int
    heads: int
    F: int
    L_img: int
    L_txt: int = 0
    grid_h: int = 0          # image token grid (for blob masks); 0 -> sqrt(L_img)
    grid_w: int = 0

    @property
    def head_dim(self) -> int:
        return self.H // self.heads

    @property
    def L(self) -> int:
        return self.L_img + self.L_txt

    def grid(self):
        if self.grid_h:
            return self.grid_h, self.grid_w
        g = int(round(math.sqrt(self.L_img)))
        assert g * g == self.L_img
        return g, g


# BASELINE.json "configs" (C1..C5), SURVEY.md §8(d) table.
CONFIGS = {
    "C1": dict(dims=BlockDims(H=64, heads=2, F=256, L_img=256), m=0.25, batch=1, dtype="f32",
               layers=1, steps=1, seed=1001),
    "C2A": dict(dims=BlockDims(H=640, heads=10, F=2560, L_img=4096), m=(0.1, 0.3, 0.5), batch=4,
                dtype="bf16", layers=10, steps=50, seed=1002),
    "C2B": dict(dims=BlockDims(H=1280, heads=20, F=5120, L_img=1024), m=(0.1, 0.3, 0.5), batch=4,
                dtype="bf16", layers=60, steps=50, seed=1002),
    "C3": dict(dims=BlockDims(H=3072, heads=24, F=12288, L_img=4096, L_txt=512), m=0.2, batch=1,
               dtype="bf16", layers=57, steps=28, seed=1003),
    "C4": dict(dims=BlockDims(H=3072, heads=24, F=12288, L_img=4096, L_txt=512), m=(0.05, 0.60),
               batch=16, dtype="bf16", layers=57, steps=28, seed=1004),
}


def block_weights(g: np.random.Generator, H: int, F: int, dtype: str = "bf16",
                  kind: str = "seq", D_ctx: int = 2048) -> dict:
    """nn.Linear layout: W[out, in]. Q/K/V stacked as rows [0,H), [H,2H), [2H,3H) of w_qkv.

    kind="par" (parallel block, NEXT-2): w_1 [3H+F, H] stacks Q, K, V and the MLP input rows;
    w_2 [H, H+F] maps the concatenation [attention | GELU(MLP)] back to H.

    kind="sdxl" (SDXL UNet transformer block, NEXT-2): bias-free Q/K/V projections (w_qkv, and
    w_q2 / w_kv2 [2H, D_ctx] for the cross-attention, K rows then V rows), biased output
    projections w_o / w_o2, GEGLU input w_up [2F, H] (first F rows the value half, last F the
    gate half), w_down [H, F], and three affine LayerNorms ln{1,2,3}_w ~ 1 + N(0, 0.02^2),
    ln{1,2,3}_b ~ N(0, 0.02^2)."""
    if kind == "double":     # Flux double-stream block: one sequential set per stream (R25)
        return {"kind": "double", "img": block_weights(g, H, F, dtype),
                "txt": block_weights(g, H, F, dtype)}
    if kind == "sdxl":
        n = lambda *shape: g.standard_normal(shape, dtype=np.float32)
        w = {
            "w_qkv": n(3 * H, H) / math.sqrt(H),
            "w_o": n(H, H) / math.sqrt(H), "b_o": 0.02 * n(H),
            "w_q2": n(H, H) / math.sqrt(H),
            "w_kv2": n(2 * H, D_ctx) / math.sqrt(D_ctx),
            "w_o2": n(H, H) / math.sqrt(H), "b_o2": 0.02 * n(H),
            "w_up": n(2 * F, H) / math.sqrt(H), "b_up": 0.02 * n(2 * F),
            "w_down": n(H, F) / math.sqrt(F), "b_down": 0.02 * n(H),
        }
        for i in (1, 2, 3):
            w[f"ln{i}_w"] = 1.0 + 0.02 * n(H)
            w[f"ln{i}_b"] = 0.02 * n(H)
        out = {k: _store(v, dtype) for k, v in w.items()}
        out["kind"] = "sdxl"
        return out
    if kind == "par":
        w = {
            "w_1": g.standard_normal((3 * H + F, H), dtype=np.float32) / math.sqrt(H),
            "b_1": 0.02 * g.standard_normal(3 * H + F, dtype=np.float32),
            "w_2": g.standard_normal((H, H + F), dtype=np.float32) / math.sqrt(H + F),
            "b_2": 0.02 * g.standard_normal(H, dtype=np.float32),
        }
        out = {k: _store(v, dtype) for k, v in w.items()}
        out["kind"] = "par"
        return out
    w = {
        "w_qkv": g.standard_normal((3 * H, H), dtype=np.float32) / math.sqrt(H),
        "b_qkv": 0.02 * g.standard_normal(3 * H, dtype=np.float32),
        "w_o": g.standard_normal((H, H), dtype=np.float32) / math.sqrt(H),
        "b_o": 0.02 * g.standard_normal(H, dtype=np.float32),
        "w_up": g.standard_normal((F, H), dtype=np.float32) / math.sqrt(H),
        "b_up": 0.02 * g.standard_normal(F, dtype=np.float32),
        "w_down": g.standard_normal((H, F), dtype=np.float32) / math.sqrt(F),
        "b_down": 0.02 * g.standard_normal(H, dtype=np.float32),
    }
    return {k: _store(v, dtype) for k, v in w.items()}


def stack_weights(g: np.random.Generator, layers: int, H: int, F: int, dtype: str = "bf16",
                  kind: str = "seq", D_ctx: int = 2048):
    return [block_weights(g, H, F, dtype, kind, D_ctx) for _ in range(layers)]


def context(g: np.random.Generator, L_ctx: int = 77, D_ctx: int = 2048,
            dtype: str = "bf16") -> np.ndarray:
    """A request's prompt encoding for the SDXL cross-attention (77 tokens x 2048 channels in
    SDXL), ~ N(0, 1)."""
    return _store(g.standard_normal((L_ctx, D_ctx), dtype=np.float32), dtype)


def mod_table(g: np.random.Generator, layers: int, steps: int, H: int, dtype: str = "bf16",
              enabled: bool = True, streams: int = 1) -> np.ndarray:
    """adaLN vectors [layers, steps, 6H] = (shift1, scale1, gate1, shift2, scale2, gate2);
    streams=2 (double-stream blocks): [layers, steps, 12H], the image stream's 6H then the text
    stream's.

    enabled=False gives the identity modulation (shift 0, scale 0, gate 1): plain LN + residual.
    """
    t = np.zeros((layers, steps, streams, 6, H), dtype=np.float32)
    if enabled:
        t[:] = 0.02 * g.standard_normal(t.shape, dtype=np.float32)
    t[:, :, :, 2] += 1.0
    t[:, :, :, 5] += 1.0
    return _store(t.reshape(layers, steps, streams * 6 * H), dtype)


def delta_table(steps: int) -> np.ndarray:
    """Per-step Euler coefficient of the synthetic sampler update x <- x + delta_s * y."""
    return np.full(steps, -1.0 / max(steps, 1), dtype=np.float32)


def latent(g: np.random.Generator, L: int, H: int, dtype: str = "bf16") -> np.ndarray:
    return _store(g.standard_normal((L, H), dtype=np.float32), dtype)


def n_masked_for(m: float, L_img: int) -> int:
    """Exact-count masks: n_img = floor(m * L_img + 0.5) (reading R18)."""
    return int(math.floor(m * L_img + 0.5))


def mask_random(g: np.random.Generator, L_img: int, m: float) -> np.ndarray:
    n = n_masked_for(m, L_img)
    mask = np.zeros(L_img, dtype=np.uint8)
    mask[g.permutation(L_img)[:n]] = 1
    return mask


def mask_blobs(g: np.random.Generator, gh: int, gw: int, m: float, n_blobs: int = 3) -> np.ndarray:
    """Irregular blob mask with an exact token count: a sum of random anisotropic Gaussian
    bumps on the token grid, thresholded at the n-th largest value (ties by token order)."""
    n = n_masked_for(m, gh * gw)
    yy, xx = np.meshgrid(np.arange(gh), np.arange(gw), indexing="ij")
    field = np.zeros((gh, gw), dtype=np.float64)
    for _ in range(n_blobs):
        cy, cx = g.uniform(0, gh), g.uniform(0, gw)
        sy, sx = g.uniform(0.08, 0.3) * gh, g.uniform(0.08, 0.3) * gw
        th = g.uniform(0, math.pi)
        dy, dx = yy - cy, xx - cx
        u = (dy * math.cos(th) + dx * math.sin(th)) / sy
        v = (-dy * math.sin(th) + dx * math.cos(th)) / sx
        field += g.uniform(0.5, 1.0) * np.exp(-0.5 * (u * u + v * v))
    flat = field.reshape(-1)
    order = np.lexsort((np.arange(flat.size), -flat))   # descending value, then token id
    mask = np.zeros(flat.size, dtype=np.uint8)
    mask[order[:n]] = 1
    return mask


def token_mask(img_mask: np.ndarray, L_txt: int) -> np.ndarray:
    """Full token mask [L_img + L_txt]: text tokens (appended last) always active."""
    return np.concatenate([img_mask.astype(np.uint8), np.ones(L_txt, dtype=np.uint8)])


def sample_mask_ratios(g: np.random.Generator, n: int, a: float = 2.0, b: float = 8.5,
                       lo: float = 0.05, hi: float = 0.60) -> np.ndarray:
    return np.clip(g.beta(a, b, size=n), lo, hi)
