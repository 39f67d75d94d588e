"""Per-CTA timeline of one 1-SM tcgen05 GEMM launch (developer build libflashps_gtrace.so,
`make VARIANT=gtrace EXTRA=-DFPS_GEMM_TRACE`): %globaltimer stamps at entry, setup done, PDL
wait done, first stage landed, last MMA of the first tile issued, its accumulator ready in the
epilogue, its epilogue done, exit.  Prints the median phase durations over the CTAs (us) and
the launch span.

  FPS_LIB=.../libflashps_gtrace.so python tools/gemm_trace.py M N K [force]
"""
import ctypes as C
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
from paper_conf_eurosys_jianglyfdlzllyl26_b200 import _lib

M, N, K = (int(v) for v in sys.argv[1:4])
force = int(sys.argv[4]) if len(sys.argv) > 4 else 4
F.fps_set_disable_tc(force)
a = torch.randn(M, K, device="cuda").to(torch.bfloat16)
w = (torch.randn(N, K, device="cuda") / K ** 0.5).to(torch.bfloat16)
out = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
for _ in range(5):
    F.linear(a, w, out=out)
torch.cuda.synchronize()
F.linear(a, w, out=out)
torch.cuda.synchronize()
lib = C.CDLL(_lib.LIB_PATH)
buf = (C.c_ulonglong * (160 * 8))()
assert lib.fps_debug_gemm_trace(buf) == 0
t = np.frombuffer(buf, dtype=np.uint64).reshape(160, 8).astype(np.float64)
t = t[t[:, 0] > 0]
t0 = t[:, 0].min()
rel = (t - t0) / 1e3
names = ["entry", "setup", "pdl_wait", "first_stage", "last_mma_issued", "acc_ready",
         "epilogue_done", "exit"]
print(f"{M}x{N}x{K} force={force}: {len(t)} CTAs, launch span {rel[:, 7].max():.2f} us, "
      f"CTA start spread {rel[:, 0].max():.2f} us")
for i in range(1, 7):
    d = rel[:, i] - rel[:, i - 1]
    print(f"  {names[i - 1]:>15} -> {names[i]:<15} median {np.median(d):6.2f} us  max {d.max():6.2f}")
