"""Quick per-kernel timing (CUDA events on the launching stream, inputs > L2 not required here:
weights and activations are re-read each rep, this is a development probe, not the bench)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F

def t_ms(fn, reps=20, warm=5):
    for _ in range(warm): fn()
    s = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record(s)
    for _ in range(reps): fn()
    e1.record(s); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps

res = {}
for (M, N, K) in [(1331, 9216, 3072), (1331, 3072, 3072), (1331, 12288, 3072), (1331, 3072, 12288),
                  (4608, 9216, 3072), (8192, 8192, 8192), (29491, 9216, 3072)]:
    a = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    w = (torch.randn(N, K, device="cuda") / K ** 0.5).to(torch.bfloat16)
    out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    ms = t_ms(lambda: F.linear(a, w, out=out))
    ms_cublas = t_ms(lambda: torch.matmul(a, w.t(), out=out))
    tf = 2 * M * N * K / ms / 1e9
    res[f"{M}x{N}x{K}"] = dict(ms=ms, tflops=tf, cublas_ms=ms_cublas, cublas_tflops=2*M*N*K/ms_cublas/1e9)
    print(f"{M}x{N}x{K}: ours {ms:.4f} ms {tf:.0f} TF/s | cuBLAS {ms_cublas:.4f} ms {2*M*N*K/ms_cublas/1e9:.0f} TF/s", flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/bench_kernels.json", "w"), indent=1)
