"""One pinned template arena shared by the worker processes of a box (SURVEY §8(e) "shared
resource"; PAPER.md L203 the host-DRAM activation store, L222 one store serving the workers):
cache location 3 maps the same file (a memfd here) MAP_SHARED and page-locks it in each
process.  Rank 0 stores the template's entries; rank 1 prefetches rows U of them into its own
HBM, byte for byte -- the entries exist once in host memory for all GPUs."""
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


def _worker(rank, world, port, path, out_dir, method):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    from oracle.index import build_mask_index
    torch.cuda.set_device(0)
    H, L_img, N, S = 256, 1024, 2, 2
    c = F.Cache(F.FPS_MODE_KV, F.FPS_BF16, H, L_img, N, S, n_templates=1, copy_method=method,
                location=3, shm_path=path)
    g = synth.rng(77)
    ents = {(s, l): synth.latent(g, L_img, 2 * H if l < N else H, "bf16") for s in range(S)
            for l in range(N + 1)}
    if rank == 0:
        for (s, l), e in ents.items():
            c.store(0, s, l, torch.as_tensor(e).cuda().to(torch.bfloat16))
        torch.cuda.synchronize()
    dist.barrier()                      # rank 0's stores are in the shared pages
    ok = True
    U = build_mask_index(synth.token_mask(synth.mask_blobs(g, 32, 32, 0.3), 0))[1]
    Ud = torch.as_tensor(U).cuda()
    for (s, l), e in ents.items():
        w = 2 * H if l < N else H
        dst = torch.zeros(L_img, w, dtype=torch.bfloat16, device="cuda")
        it = F.fps_prefetch_item(0, s, l, len(U), Ud.data_ptr(), U.ctypes.data, dst.data_ptr(), w * 2)
        ls = torch.cuda.Stream()
        ls.wait_stream(torch.cuda.current_stream())
        ev = torch.cuda.Event()
        c.prefetch([it], ls, ev)
        ev.synchronize()
        exp = np.zeros((L_img, w), np.float32)
        rows = np.arange(L_img) if method == 2 else U
        exp[rows] = e[rows]
        ok &= bool(np.array_equal(dst.float().cpu().numpy(), exp))
    np.save(os.path.join(out_dir, f"s{rank}.npy"), np.array([ok]))
    dist.barrier()
    c.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("method", [2, 3])
def test_shared_arena_two_processes(tmp_path, method):
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as F
    F.require_gpu()
    fd = os.memfd_create("flashps_test_arena")
    try:
        path = f"/proc/{os.getpid()}/fd/{fd}"
        port = _free_port()
        mp.spawn(_worker, args=(2, port, path, str(tmp_path), method), nprocs=2, join=True)
        assert all(bool(np.load(tmp_path / f"s{r}.npy")[0]) for r in range(2))
        # one copy of the arena for both processes: the file holds the entries
        assert os.fstat(fd).st_size >= 2 * 3 * 1024 * 2 * 256 * 2
    finally:
        os.close(fd)
