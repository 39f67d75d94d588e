"""NEXT-1's peer tier (the hierarchical activation store, one level up):
a template arena in one GPU worker's HBM, exported as a CUDA IPC handle and opened by another
worker process (cache location 4), whose prefetches read it over NVLink / NVSwitch.  On a
one-GPU lease both processes share the device -- the same IPC mapping and code path, over the
device's own memory instead of the links.  Checked: the rows U land byte for byte (row gather
and whole-entry copy), and a mask-aware engine step over the peer arena is bit-identical to
the same step over a local copy of the entries."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, port, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    from oracle.index import build_mask_index
    from gpu_util import to_dev
    torch.cuda.set_device(0)
    H, L_img, L_txt, N, S, heads = 256, 256, 16, 3, 2, 2
    g = synth.rng(91)
    ents = {(s, l): synth.latent(g, L_img, 2 * H if l < N else H, "bf16") for s in range(S)
            for l in range(N + 1)}
    desc = dict(mode=F.FPS_MODE_KV, dtype=F.FPS_BF16, H=H, L_img=L_img, n_layers=N, n_steps=S)
    ok = True
    if rank == 0:
        owner = F.Cache(desc["mode"], desc["dtype"], H, L_img, N, S, location=1)
        for (s, l), e in ents.items():
            owner.store(0, s, l, to_dev(e, "bf16"))
        torch.cuda.synchronize()
        obj = [owner.export_ipc()]
    else:
        obj = [None]
    dist.broadcast_object_list(obj, src=0)
    if rank == 1:
        W = synth.stack_weights(g, N, H, 512, "bf16")
        mods = synth.mod_table(g, N, S, H, "bf16")
        layers = [F.BlockWeights(w, heads, F.FPS_BF16) for w in W]
        mask = synth.token_mask(synth.mask_blobs(g, 16, 16, 0.3), L_txt)
        U = build_mask_index(mask)[1]
        U = U[U < L_img]
        Ud = torch.as_tensor(U).cuda()
        for method in (0, 2, 3):
            peer = F.Cache(desc["mode"], desc["dtype"], H, L_img, N, S, location=4,
                           copy_method=method, peer_handle=obj[0])
            for (s, l), e in ents.items():
                w = 2 * H if l < N else H
                dst = torch.zeros(L_img, w, dtype=torch.bfloat16, device="cuda")
                it = F.fps_prefetch_item(0, s, l, len(U), Ud.data_ptr(), U.ctypes.data,
                                         dst.data_ptr(), w * 2)
                ls = torch.cuda.Stream()
                ls.wait_stream(torch.cuda.current_stream())
                ev = torch.cuda.Event()
                peer.prefetch([it], ls, ev)
                ev.synchronize()
                exp = np.zeros((L_img, w), np.float32)
                rows = np.arange(L_img) if method == 2 else U
                exp[rows] = e[rows]
                ok &= bool(np.array_equal(dst.float().cpu().numpy(), exp))
            # an engine step over the peer arena vs over a local copy of the entries
            local = F.Cache(desc["mode"], desc["dtype"], H, L_img, N, S, location=1, copy_method=method)
            for (s, l), e in ents.items():
                local.store(0, s, l, to_dev(e, "bf16"))
            torch.cuda.synchronize()
            outs = []
            x0 = synth.latent(synth.rng(5), L_img + L_txt, H, "bf16")
            for c in (peer, local):
                eng = F.Engine(layers, heads, F.FPS_MODE_KV, F.FPS_BF16, L_img, L_txt, 1, S,
                               synth.delta_table(S), c, mod_table=to_dev(mods, "bf16"),
                               plan_policy=1, cross_step=True)
                req = dict(template_id=0, step=0, n_steps=S, mask=torch.as_tensor(mask).cuda(),
                           x=to_dev(x0, "bf16"))
                eng.run_batch([req], S, load_stream=torch.cuda.Stream())
                torch.cuda.synchronize()
                outs.append(req["x"].clone())
                eng.close()
            ok &= bool(torch.equal(outs[0].view(torch.int16), outs[1].view(torch.int16)))
            local.close()
            peer.close()
    np.save(os.path.join(out_dir, f"p{rank}.npy"), np.array([ok]))
    dist.barrier()                     # the owner keeps its arena until the importer is done
    if rank == 0:
        owner.close()
    dist.destroy_process_group()


def test_peer_tier_ipc_arena():
    import tempfile
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    F.require_gpu()
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_worker, args=(_free_port(), d), nprocs=2, join=True)
        assert all(bool(np.load(os.path.join(d, f"p{r}.npy"))[0]) for r in range(2))
