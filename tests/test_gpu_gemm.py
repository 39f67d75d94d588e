"""GPU parity of the projection GEMMs (fps_linear: tcgen05 for bf16) against fp64 matmul of the
same bf16 inputs; shapes of the block's GEMMs at configs[1..3] plus ragged edges."""
import numpy as np
import pytest
import torch

import synth
from oracle.block import gelu_tanh, linear
from gpu_util import TOL, check_close, to_dev, to_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as fps
    fps.require_gpu()
    return fps


@pytest.mark.parametrize("M,N,K", [(128, 256, 64), (1, 8, 64), (130, 136, 128), (1331, 9216, 3072),
                                   (1331, 3072, 12288), (409, 1920, 640), (2048, 2560, 1280),
                                   (300, 640, 2560), (4608, 3072, 3072)])
@pytest.mark.parametrize("act", [0, 1])
@pytest.mark.parametrize("kernel", ["auto", "1sm", "1sm_epi4", "pair", "pair_epi4", "swap"])
def test_linear_bf16(F, M, N, K, act, kernel):
    g = synth.rng(M * 7 + N + K + act)
    a = synth.latent(g, M, K, "bf16")
    w = synth.bf16_round(g.standard_normal((N, K), dtype=np.float32) / np.sqrt(K))
    b = synth.bf16_round(0.1 * g.standard_normal(N, dtype=np.float32))
    F.fps_set_disable_tc({"auto": 0, "1sm": 4, "1sm_epi4": 4 | 2048, "pair": 8, "pair_epi4": 8 | 2048, "swap": 12}[kernel])
    try:
        out = F.linear(to_dev(a, "bf16"), to_dev(w, "bf16"), to_dev(b, "bf16"), act=act)
        torch.cuda.synchronize()
    finally:
        F.fps_set_disable_tc(0)
    ref = linear(a, w, b)
    if act:
        ref = gelu_tanh(ref)
    rows = np.arange(M) if M * N <= 4_000_000 else synth.rng(1).choice(M, 256, replace=False)
    check_close(to_np(out)[rows], ref[rows], TOL["bf16"], f"linear {M}x{N}x{K}")


def test_linear_deterministic(F):
    g = synth.rng(9)
    a = to_dev(synth.latent(g, 1000, 1024, "bf16"), "bf16")
    w = to_dev(synth.latent(g, 768, 1024, "bf16"), "bf16")
    o1, o2 = F.linear(a, w), F.linear(a, w)
    torch.cuda.synchronize()
    assert torch.equal(o1.view(torch.int16), o2.view(torch.int16))
