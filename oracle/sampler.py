"""The sampler update after the block stack (a9), oracle side (test infrastructure only).

PAPER.md L73-L79 (§2.1, Fig. 2): the template image and the mask are encoded into a latent, "a
diffusion model then uses the latent for N steps of denoising computation, producing a final
latent that is decoded into the output image"; L157 (§3.1): only the masked region is computed,
the unmasked region keeps the template's content ("image editing only modifies the masked
regions of image templates, while preserving the original content in the unmasked areas",
L9).  The paper never writes the sampler (reading R29):

  * Flow-matching Euler, the scheduler of the Flux model the paper serves (L305): noise levels
    sigma_0 = 1 > sigma_1 > ... > sigma_S = 0, the stack's output y is the velocity, and
        x_{s+1} = x_s + (sigma_{s+1} - sigma_s) * y_s
  * Inpainting blend (the image-editing form of that sampler): after each step the unmasked
    image rows are reset to the template latent z re-noised to the next level with the
    request's noise eps,
        x_{s+1}[u] = (1 - sigma_{s+1}) * z[u] + sigma_{s+1} * eps[u]      u unmasked image row
    so at the last step (sigma_S = 0) the unmasked region IS the template latent.
  * Text rows (Flux's prompt tokens, always active, R9) are the prompt encoding, re-fed
    unchanged every step.
  * Schedule: Flux's shifted schedule, t_i = 1 - i/S (i < S), sigma_i = shift t_i / (1 + (shift-1)
    t_i), sigma_S = 0; shift = exp(1.15) for 4096 image tokens (Flux's resolution-dependent shift
    at its maximum sequence length), 1 = the plain linear schedule.

The synthetic update of reading R21 (x <- x + delta_s * y over the whole latent) stays the
default of the parity tests (stack.euler_update).
"""
from __future__ import annotations

import math

import numpy as np

from .block import f64

FLUX_SHIFT = math.exp(1.15)


def flow_sigmas(steps: int, shift: float = 1.0) -> np.ndarray:
    """sigma_0 .. sigma_S of the shifted flow-matching schedule (R29); float64, S + 1 values."""
    t = 1.0 - np.arange(steps, dtype=np.float64) / steps
    sig = shift * t / (1.0 + (shift - 1.0) * t)
    return np.concatenate([sig, [0.0]])


def flow_init(z, eps, sigma0, L_txt_rows=None):
    """Starting latent of an inpainting request: the template latent noised to sigma_0
    ((1 - sigma_0) z + sigma_0 eps; pure noise at sigma_0 = 1), text rows appended as given."""
    x = (1.0 - sigma0) * f64(z) + sigma0 * f64(eps)
    if L_txt_rows is not None:
        x = np.concatenate([x, f64(L_txt_rows)], axis=0)
    return x


def flow_blend_update(x, y, mask, z, eps, sigma_s, sigma_next, L_img):
    """One step of the flow-matching Euler sampler with inpainting blend (R29).

    x, y: [L, H] latent entering the step and the stack's output; mask: [L] token mask (nonzero =
    active); z, eps: [L_img, H] template latent and noise; rows >= L_img are text rows."""
    x = f64(x).copy()
    y = f64(y)
    m = np.asarray(mask)[:L_img] != 0
    img = x[:L_img]
    img[m] = img[m] + (float(sigma_next) - float(sigma_s)) * y[:L_img][m]
    img[~m] = (1.0 - float(sigma_next)) * f64(z)[~m] + float(sigma_next) * f64(eps)[~m]
    return x
