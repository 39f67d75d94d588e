"""Library attention on the same box, for context: torch SDPA (cuDNN and flash backends) at
the C3 shapes (24 heads x 128, L = 4608 keys; 1331 or 4608 queries) and, with `sdxl`, the C2A
shapes (10 heads x 64, L = 4096 keys, batch 4; 1229 or 4096 queries), bf16, TFLOP/s.

  python tools/attn_library_ref.py [sdxl]"""
import sys
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


sdxl = len(sys.argv) > 1 and sys.argv[1] == "sdxl"
for n in ((1229, 4096) if sdxl else (1331, 4608)):
    L, h, d, B = (4096, 10, 64, 4) if sdxl else (4608, 24, 128, 1)
    q = torch.randn(B, h, n, d, device="cuda", dtype=torch.bfloat16)
    k = torch.randn(B, h, L, d, device="cuda", dtype=torch.bfloat16)
    v = torch.randn(B, h, L, d, device="cuda", dtype=torch.bfloat16)
    for be in (SDPBackend.CUDNN_ATTENTION, SDPBackend.FLASH_ATTENTION, SDPBackend.EFFICIENT_ATTENTION):
        try:
            ms = bench(q, k, v, be)
            print(f"n={n} L={L} {be.name}: {ms * 1e3:.1f} us  {4 * B * n * L * h * d / (ms * 1e-3) / 1e12:.0f} TF/s")
        except Exception as ex:
            print(f"n={n} {be.name}: unavailable ({str(ex)[:80]})")
