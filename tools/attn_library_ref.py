"""Library attention on the same box, for context: torch SDPA (cuDNN and flash backends) at
the C3 shapes (24 heads x 128, L = 4608 keys; 1331 or 4608 queries), bf16, TFLOP/s."""
import torch
import torch.nn.functional as Fn
from torch.nn.attention import SDPBackend, sdpa_kernel


def bench(q, k, v, backend, iters=20):
    with sdpa_kernel(backend):
        for _ in range(3):
            Fn.scaled_dot_product_attention(q, k, v)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(iters):
            Fn.scaled_dot_product_attention(q, k, v)
        e1.record()
        torch.cuda.synchronize()
    return e0.elapsed_time(e1) / iters


for n in (1331, 4608):
    L, h, d = 4608, 24, 128
    q = torch.randn(1, h, n, d, device="cuda", dtype=torch.bfloat16)
    k = torch.randn(1, h, L, d, device="cuda", dtype=torch.bfloat16)
    v = torch.randn(1, h, L, d, device="cuda", dtype=torch.bfloat16)
    for be in (SDPBackend.CUDNN_ATTENTION, SDPBackend.FLASH_ATTENTION, SDPBackend.EFFICIENT_ATTENTION):
        try:
            ms = bench(q, k, v, be)
            print(f"n={n} L={L} {be.name}: {ms * 1e3:.1f} us  {4 * n * L * h * d / (ms * 1e-3) / 1e12:.0f} TF/s")
        except Exception as ex:
            print(f"n={n} {be.name}: unavailable ({str(ex)[:80]})")
