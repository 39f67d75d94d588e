import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch, synth
import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
from oracle.index import build_mask_index
g = synth.rng(102)
H, L_img, L_txt, N, S = 256, 1024, 64, 3, 2
for mode in ("kv", "y"):
  for method in (0, 1):
    m = F.MODE_CODE[mode]
    c = F.Cache(m, F.FPS_BF16, H, L_img, N, S, n_templates=2, copy_method=method)
    W = 2 * H if mode == "kv" else H
    layers = N + (1 if mode == "kv" else 0)
    ents = {}
    for t in range(2):
        for s in range(S):
            for l in range(layers):
                w = H if (mode == "kv" and l == N) else W
                e = synth.latent(g, L_img + L_txt, w, "bf16")
                ents[(t, s, l)] = e
                c.store(t, s, l, torch.as_tensor(e).cuda().to(torch.bfloat16))
    torch.cuda.synchronize()
    masks = [synth.mask_random(g, L_img, 0.2), synth.mask_blobs(g, 32, 32, 0.4)]
    ids = [build_mask_index(mk)[1] for mk in masks]
    s = 1
    for layer in ([2, N] if mode == "kv" else [2]):
        w = H if (mode == "kv" and layer == N) else W
        dst = torch.zeros(2 * (L_img + L_txt), w, dtype=torch.bfloat16, device="cuda")
        d_ids = [torch.as_tensor(u).cuda() for u in ids]
        items = [F.fps_prefetch_item(t, s, layer, len(ids[r]), d_ids[r].data_ptr(), ids[r].ctypes.data,
                                     dst[r * (L_img + L_txt)].data_ptr(), w * 2) for r, t in enumerate((1, 0))]
        ls = torch.cuda.Stream(); ls.wait_stream(torch.cuda.current_stream())
        ev = torch.cuda.Event()
        c.prefetch(items, ls, ev); ev.synchronize()
        got = dst.float().cpu().numpy()
        for r, t in enumerate((1, 0)):
            base = r * (L_img + L_txt)
            exp = np.zeros(((L_img + L_txt), w), np.float32)
            exp[ids[r]] = ents[(t, s, layer)][ids[r]]
            bad = np.argwhere(got[base:base + L_img + L_txt] != exp)
            print(mode, method, "layer", layer, "req", r, "bad", len(bad), bad[:5].tolist(),
                  "rows", np.unique(bad[:, 0])[:10].tolist() if len(bad) else [])
            if len(bad):
                rr = bad[0][0]
                print("  got", got[base + rr, :4], "exp", exp[rr, :4], "in U", rr in set(ids[r].tolist()))
                # which entry does it match?
                for k, e in ents.items():
                    if np.array_equal(got[base + rr], e[rr]): print("  matches entry", k)
    c.close()
