"""GPU parity, bit-exact: a1 mask index, a2/a9 gather/scatter, a3 cache store/prefetch."""
import numpy as np
import pytest
import torch

import synth
from oracle.index import build_mask_index, gather_rows, scatter_rows

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def F():
    import paper_conf_eurosys_jianglyfdlzllyl26_b200 as fps
    fps.require_gpu()
    return fps


def _masks(g):
    out = []
    for L_img, L_txt, m, kind in [(256, 0, 0.25, "r"), (4096, 512, 0.2, "b"), (1024, 0, 0.1, "r"),
                                  (4096, 0, 0.0, "r"), (100, 7, 1.0, "r"), (33, 0, 0.5, "r"),
                                  (1, 0, 1.0, "r"), (2048, 77, 0.6, "r"), (4096, 512, 0.05, "b"),
                                  (3000, 0, 0.3, "r")]:
        if kind == "b":
            gh = int(np.sqrt(L_img))
            im = synth.mask_blobs(g, gh, L_img // gh, m)
        else:
            im = synth.mask_random(g, L_img, m)
        out.append(synth.token_mask(im, L_txt))
    return out


def test_mask_index_bit_exact(F):
    g = synth.rng(100)
    masks = _masks(g)
    mids, uids, nm, off = F.build_mask_index([torch.as_tensor(m).cuda() for m in masks])
    torch.cuda.synchronize()
    mids, uids, nm, off = (t.cpu().numpy() for t in (mids, uids, nm, off))
    for r, m in enumerate(masks):
        M, U = build_mask_index(m)
        o = off[r]
        assert nm[r] == len(M)
        assert np.array_equal(mids[o:o + len(M)], M)
        assert np.array_equal(uids[o:o + len(U)], U)


@pytest.mark.parametrize("dtype,H", [("bf16", 8), ("bf16", 640), ("bf16", 3072), ("f32", 64),
                                     ("f32", 4), ("bf16", 6144)])
def test_gather_scatter_bit_exact(F, dtype, H):
    g = synth.rng(101)
    L = 1000
    x = synth.latent(g, L, H, dtype)
    mask = synth.mask_random(g, L, 0.3)
    M, U = build_mask_index(mask)
    td = torch.bfloat16 if dtype == "bf16" else torch.float32
    xd = torch.as_tensor(x).cuda().to(td)
    Md, Ud = torch.as_tensor(M).cuda(), torch.as_tensor(U).cuda()
    xm = F.gather_rows(xd, Md)
    xu = F.gather_rows(xd, Ud)
    out = torch.full_like(xd, float("nan"))
    F.scatter_rows(xm, Md, out)
    F.scatter_rows(xu, Ud, out)
    torch.cuda.synchronize()
    assert torch.equal(xm.float().cpu(), torch.as_tensor(gather_rows(x, M)))
    assert torch.equal(out.view(torch.int16 if dtype == "bf16" else torch.int32),
                       xd.view(torch.int16 if dtype == "bf16" else torch.int32))
    ref = scatter_rows(gather_rows(x, M), M, np.zeros_like(x))
    got = torch.zeros_like(xd)
    F.scatter_rows(xm, Md, got)
    assert torch.equal(got.float().cpu(), torch.as_tensor(ref))


def test_empty_gather_is_noop(F):
    x = torch.randn(4, 8, device="cuda")
    ids = torch.empty(0, dtype=torch.int32, device="cuda")
    out = F.gather_rows(x, ids)
    assert out.shape == (0, 8)


@pytest.mark.parametrize("mode,method,location,H,ctas", [
    ("kv", 0, 0, 256, 0), ("y", 0, 0, 256, 0), ("kv", 1, 0, 256, 0), ("y", 1, 0, 256, 0),
    ("kv", 0, 1, 256, 0), ("y", 0, 1, 256, 0), ("kv", 1, 1, 256, 0),
    ("kv", 2, 0, 256, 0), ("y", 2, 0, 256, 0), ("kv", 2, 1, 256, 0),
    ("kv", 3, 0, 256, 0), ("y", 3, 0, 256, 0), ("kv", 3, 0, 3072, 0), ("y", 3, 0, 3072, 0),
    ("kv", 3, 0, 1280, 6), ("kv", 3, 1, 640, 2), ("y", 3, 0, 4096, 1),
    ("kv", 3, 0, 3072, 8)])                             # configs[3]'s KV-mode setting
def test_cache_store_prefetch_bytes_equal(F, mode, method, location, H, ctas):
    """a3: the prefetched rows are the stored entry's rows, byte for byte, at their token rows.
    Exact-row methods (0, 1, 3) leave every other row untouched; the whole-entry DMA (2) lands
    all L_img image rows of the entry (text rows untouched).  Method 3 (TMA bulk row gather)
    also at Flux / SDXL row widths (one-row chunks, odd row sizes) and odd CTA counts."""
    g = synth.rng(102)
    L_img, L_txt, N, S = 1024, 64, 3, 2
    m = F.MODE_CODE[mode]
    c = F.Cache(m, F.FPS_BF16, H, L_img, N, S, n_templates=2, copy_method=method,
                location=location, copy_ctas=ctas)
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
    # host arena == stored rows (bit-exact); the HBM tier is checked through the prefetch below
    for (t, s, l), e in (ents.items() if location == 0 else []):
        host = c.entry_numpy(t, s, l)
        ref = torch.as_tensor(e[:L_img]).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
        assert np.array_equal(host, ref)
    # prefetch rows U of two requests into their regions of a batch buffer
    masks = [synth.mask_random(g, L_img, 0.2), synth.mask_blobs(g, 32, 32, 0.4)]
    ids = [build_mask_index(mk)[1] for mk in masks]
    s, l = 1, 2
    for layer in ([l, N] if mode == "kv" else [l]):
        w = H if (mode == "kv" and layer == N) else W
        dst = torch.zeros(2 * (L_img + L_txt), w, dtype=torch.bfloat16, device="cuda")
        d_ids = [torch.as_tensor(u).cuda() for u in ids]
        items = []
        for r, t in enumerate((1, 0)):
            items.append(F.fps_prefetch_item(t, s, layer, len(ids[r]), d_ids[r].data_ptr(),
                                             ids[r].ctypes.data, dst[r * (L_img + L_txt)].data_ptr(),
                                             w * 2))
        ls = torch.cuda.Stream()
        ls.wait_stream(torch.cuda.current_stream())     # dst zero-fill and ids upload first
        ev = torch.cuda.Event()
        c.prefetch(items, ls, ev)
        ev.synchronize()
        got = dst.float().cpu().numpy()
        for r, t in enumerate((1, 0)):
            base = r * (L_img + L_txt)
            exp = np.zeros(((L_img + L_txt), w), np.float32)
            rows = np.arange(L_img) if method == 2 else ids[r]
            exp[rows] = ents[(t, s, layer)][rows]
            assert np.array_equal(got[base:base + L_img + L_txt], exp)
    c.close()


@pytest.mark.parametrize("Hp,Wp,f,L_txt,n_req,p", [(1024, 1024, 16, 512, 2, 0.0005),
                                                  (1024, 1024, 32, 0, 3, 0.0002),
                                                  (30, 45, 3, 5, 2, 0.02), (64, 48, 16, 0, 1, 0.0),
                                                  (64, 64, 16, 3, 1, 1.0), (8, 8, 1, 0, 1, 0.3),
                                                  (96, 80, 8, 1, 4, 0.01)])
def test_mask_to_tokens_bit_exact(F, Hp, Wp, f, L_txt, n_req, p):
    from oracle.index import pixel_to_token_mask
    g = synth.rng(Hp + Wp + f)
    pix = (g.random((n_req, Hp, Wp)) < p).astype(np.uint8)
    if Hp >= 64:                                    # plus an irregular blob region
        yy, xx = np.mgrid[:Hp, :Wp]
        pix[0] |= (((yy - Hp / 3) / (Hp / 6)) ** 2 + ((xx - Wp / 2) / (Wp / 5)) ** 2 < 1).astype(np.uint8)
    tok = F.mask_to_tokens(torch.as_tensor(pix).cuda(), f, L_txt)
    torch.cuda.synchronize()
    got = tok.cpu().numpy()
    for r in range(n_req):
        assert got[r].tolist() == pixel_to_token_mask(pix[r], f, L_txt).tolist()


def test_mask_to_tokens_rejects_bad_geometry(F):
    pix = torch.zeros(1, 30, 40, dtype=torch.uint8, device="cuda")
    with pytest.raises(F.FlashPSError):
        F.mask_to_tokens(pix, 16)
