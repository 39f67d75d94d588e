import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np
import synth
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
g = synth.rng(3)
H, heads, Fd, L = 3072, 24, 12288, 4608
w = synth.block_weights(g, H, Fd, "bf16")
bw = F.BlockWeights(w, heads, F.FPS_BF16)
x = torch.randn(L, H, device="cuda").to(torch.bfloat16)
outs = {}
for flags in (256, 512, 0):
    F.fps_set_disable_tc(flags)
    F.fps_profile_enable(1)
    b = F.VarlenBatch([L], [L])
    y, _ = F.dense_block_forward(bw, b, x)
    torch.cuda.synchronize()
    cnt = np.zeros(7, dtype=np.int64)
    import ctypes as C
    F.fps_profile_read(None, None, None, cnt.ctypes.data_as(C.POINTER(C.c_int64)))
    F.fps_profile_enable(0)
    outs[flags] = y.clone()
    print(flags, "launch counts", cnt.tolist(), "launches total", F.fps_launch_count())
F.fps_set_disable_tc(0)
print("S=1 vs S=2 bit-equal:", torch.equal(outs[256], outs[512]), "auto == S=2:", torch.equal(outs[0], outs[512]),
      "max diff", (outs[256].float() - outs[512].float()).abs().max().item())
