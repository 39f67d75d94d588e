"""B200-native FlashPS hot path: the mask-aware transformer-block forward (§3.1),
its layer-ahead cache pipeline with the Alg. 1 planner (§4.2) and step-level continuous
batching (§4.3), as the C-ABI library libflashps.so (include/flashps.h) plus this thin binding.

`fps_*` are the C entry points (ctypes, argument marshalling only). The small classes below wrap
torch tensors (device memory) into the C descriptor structs. Nothing here computes the method:
every step runs in the library's CUDA kernels; there is no CPU fallback.
"""
from __future__ import annotations

import ctypes as C

import numpy as np
import torch

from . import _lib
from ._lib import *  # noqa: F401,F403  (the fps_* C entry points and struct types)
from ._lib import (FPS_BF16, FPS_F32, FPS_MODE_KV, FPS_MODE_Y, FlashPSError, fps_block_weights,
                   fps_cache_desc, fps_engine_desc, fps_prefetch_item, fps_request,
                   fps_varlen_batch)

TORCH_DTYPE = {FPS_BF16: torch.bfloat16, FPS_F32: torch.float32}
DTYPE_CODE = {"bf16": FPS_BF16, "f32": FPS_F32}
MODE_CODE = {"kv": FPS_MODE_KV, "y": FPS_MODE_Y}


def ptr(t):
    """Device/host address of a tensor as an int (None for None)."""
    return None if t is None else t.data_ptr()


def stream_ptr(s=None):
    s = s if s is not None else torch.cuda.current_stream()
    return s.cuda_stream


def require_gpu():
    if not torch.cuda.is_available() or not _lib.fps_device_ok():
        raise FlashPSError("require_gpu", _lib.FPS_ECUDA, "no usable sm_100 (B200) device")


# ---------------------------------------------------------------------------------------
def mask_to_tokens(pix, f, L_txt=0, stream=None):
    """NEXT-4 on the GPU: pixel masks (uint8 cuda tensor [n_req, Hp, Wp] or [Hp, Wp]) -> token
    masks [n_req, (Hp/f)*(Wp/f) + L_txt] (uint8, text tokens active)."""
    p = pix.reshape((-1,) + tuple(pix.shape[-2:])).contiguous().to(torch.uint8)
    n, Hp, Wp = p.shape
    tok = torch.empty(n, (Hp // f) * (Wp // f) + L_txt, dtype=torch.uint8, device=pix.device)
    _lib.fps_mask_to_tokens(ptr(p), n, Hp, Wp, f, L_txt, ptr(tok), stream_ptr(stream))
    return tok


def build_mask_index(masks, stream=None):
    """a1 on the GPU. masks: list of uint8 cuda tensors (one per request, text rows set).
    Returns (masked_ids, unmasked_ids, n_masked, offsets) as cuda int32 tensors; request r's
    ids live at [off[r], off[r] + n) / [off[r], off[r] + L_r - n)."""
    dev = masks[0].device
    lens = [int(m.numel()) for m in masks]
    off = torch.tensor(np.concatenate([[0], np.cumsum(lens)]), dtype=torch.int32, device=dev)
    flat = torch.cat([m.reshape(-1) for m in masks]).to(torch.uint8)
    total = int(off[-1])
    mids = torch.empty(max(total, 1), dtype=torch.int32, device=dev)
    uids = torch.empty(max(total, 1), dtype=torch.int32, device=dev)
    nm = torch.empty(len(masks), dtype=torch.int32, device=dev)
    _lib.fps_build_mask_index(ptr(flat), ptr(off), len(masks), max(lens), ptr(mids), ptr(uids),
                              ptr(nm), stream_ptr(stream))
    return mids, uids, nm, off


def gather_rows(src, ids, out=None, stream=None):
    n = int(ids.numel())
    out = out if out is not None else torch.empty((n,) + tuple(src.shape[1:]), dtype=src.dtype,
                                                  device=src.device)
    rb = src[0].numel() * src.element_size()
    _lib.fps_gather_rows(ptr(src), ptr(ids), n, rb, ptr(out), stream_ptr(stream))
    return out


def scatter_rows(src, ids, out, stream=None):
    rb = out[0].numel() * out.element_size()
    _lib.fps_scatter_rows(ptr(src), ptr(ids), int(ids.numel()), rb, ptr(out), stream_ptr(stream))
    return out


_KIND = {"seq": _lib.FPS_BLOCK_SEQ, "par": _lib.FPS_BLOCK_PAR, "sdxl": _lib.FPS_BLOCK_SDXL,
         "double": _lib.FPS_BLOCK_DOUBLE}
_SEQ_KEYS = ("w_qkv", "b_qkv", "w_o", "b_o", "w_up", "b_up", "w_down", "b_down")
_SDXL_KEYS = ("ln1_w", "ln1_b", "ln2_w", "ln2_b", "ln3_w", "ln3_b", "w_q2", "b_q2", "w_kv2",
              "b_kv2", "w_o2", "b_o2")


class BlockWeights:
    """Holds one block's device weights (nn.Linear layout) and its C descriptor."""

    def __init__(self, w: dict, heads: int, dtype: int, device="cuda", stream=None):
        """w: the sequential block's w_qkv, b_qkv, w_o, b_o, w_up, b_up, w_down, b_down, or with
        w["kind"] == "par" the parallel block's w_1 [3H+F, H], b_1, w_2 [H, H+F], b_2, or with
        w["kind"] == "sdxl" the SDXL block's weights (synth.block_weights names); its GEGLU input
        projection w_up [2F, H] is repacked on the device by fps_geglu_pack."""
        td = TORCH_DTYPE[dtype]
        self.kind = _KIND[w.get("kind", "seq")]
        alias = {"w_1": "w_qkv", "b_1": "b_qkv", "w_2": "w_down", "b_2": "b_down"}
        if self.kind == _lib.FPS_BLOCK_DOUBLE:     # image stream = the primary fields
            w = dict(w["img"], **{"t" + k[1:] if k.startswith("w_") else "tb" + k[1:]: v
                                  for k, v in w["txt"].items()})
        self.t = {alias.get(k, k): torch.as_tensor(np.ascontiguousarray(v)).to(device=device, dtype=td)
                  for k, v in w.items() if k != "kind" and v is not None}
        H = self.t["w_down"].shape[0]
        if self.kind == _lib.FPS_BLOCK_PAR:
            F = self.t["w_qkv"].shape[0] - 3 * H
        elif self.kind == _lib.FPS_BLOCK_SDXL:
            F = self.t["w_up"].shape[0] // 2
            K = self.t["w_up"].shape[1]
            wp = torch.empty_like(self.t["w_up"])
            bp = torch.empty_like(self.t["b_up"]) if "b_up" in self.t else None
            _lib.fps_geglu_pack(dtype, ptr(self.t["w_up"]), ptr(self.t.get("b_up")), F, K,
                                ptr(wp), ptr(bp), stream_ptr(stream))
            self.t["w_up"], self.t["b_up"] = wp, bp
        else:
            F = self.t["w_up"].shape[0]
        self.H, self.F, self.heads, self.dtype = H, F, heads, dtype
        self.D_ctx = self.t["w_kv2"].shape[1] if "w_kv2" in self.t else 0
        self.c = fps_block_weights(H, heads, H // heads, F, dtype,
                                   *[ptr(self.t.get(k)) for k in
                                     ("w_qkv", "b_qkv", "w_o", "b_o", "w_up", "b_up", "w_down",
                                      "b_down")], self.kind, self.D_ctx,
                                   *[ptr(self.t.get(k)) for k in _SDXL_KEYS],
                                   *[ptr(self.t.get("t" + k[1:] if k.startswith("w_") else
                                                    "tb" + k[1:])) for k in _SEQ_KEYS])

    def context_kv(self, ctx, out=None, stream=None):
        """SDXL block: the cross-attention K|V rows [n, 2H] of prompt encodings ctx [n, D_ctx]."""
        out = out if out is not None else torch.empty(ctx.shape[0], 2 * self.H, dtype=ctx.dtype,
                                                      device=ctx.device)
        _lib.fps_context_kv(C.byref(self.c), ptr(ctx), ctx.shape[0], ptr(out), stream_ptr(stream))
        return out


class VarlenBatch:
    """Descriptor of one varlen launch over a batch of requests (host bookkeeping + upload).

    n_active[r], L[r]: rows; q_row: global merged row of every active row (None = dense);
    u_row / u_src: Y-mode cached rows. mod: [n_req, 6H] device tensor or None."""

    def __init__(self, n_active, L, q_row=None, mod=None, mode=FPS_MODE_KV, u_row=None,
                 u_src=None, n_unmasked=None, device="cuda", ctx_kv=None, n_ctx=None,
                 act_ids=None, L_img=None, mod_stride=0, stream_inverse=True):
        self.n_active = list(map(int, n_active))
        self.L = list(map(int, L))
        cu_q = np.concatenate([[0], np.cumsum(self.n_active)]).astype(np.int32)
        cu_k = np.concatenate([[0], np.cumsum(self.L)]).astype(np.int32)
        self.h_cu_q, self.h_cu_k = cu_q, cu_k
        self.cu_q = torch.tensor(cu_q, device=device)
        self.cu_k = torch.tensor(cu_k, device=device)
        self.q_row = q_row
        self.mod = mod
        self.u_row, self.u_src = u_row, u_src
        nu = n_unmasked if n_unmasked is not None else [0] * len(self.L)
        cu_u = np.concatenate([[0], np.cumsum(nu)]).astype(np.int32)
        self.cu_u = torch.tensor(cu_u, device=device)
        self.c = fps_varlen_batch(
            len(self.L), int(cu_q[-1]), int(cu_k[-1]), max(self.n_active, default=0),
            max(self.L, default=0), ptr(self.cu_q), ptr(self.cu_k),
            self.h_cu_q.ctypes.data_as(C.c_void_p), self.h_cu_k.ctypes.data_as(C.c_void_p),
            ptr(q_row), ptr(mod), mode, int(cu_u[-1]), ptr(self.cu_u), ptr(u_src), ptr(u_row))
        self.c.mod_stride = mod_stride
        if act_ids is not None:      # double-stream blocks: stream-major order of the rows
            # act_ids[r]: ascending token ids of request r's active rows (all rows if dense)
            perm, kvr, ni, nt = [], [], [], []
            for st in (0, 1):
                for r, ids in enumerate(act_ids):
                    ids = np.asarray(ids)
                    sel = np.flatnonzero((ids >= L_img) if st else (ids < L_img))
                    perm.append(cu_q[r] + sel)
                    kvr.append(cu_k[r] + ids[sel])
                    (nt if st else ni).append(len(sel))
            pm = np.concatenate(perm)
            inv = np.empty_like(pm)
            inv[pm] = np.arange(len(pm))
            arrs = (pm, np.concatenate(kvr), np.concatenate([[0], np.cumsum(ni)]),
                    np.concatenate([[0], np.cumsum(nt)]), inv)
            self.sm = [torch.as_tensor(a.astype(np.int32), device=device) for a in arrs]
            self.c.total_q_img = int(sum(ni))
            (self.c.d_sm_perm, self.c.d_sm_kvrow, self.c.d_cu_img, self.c.d_cu_txt,
             self.c.d_sm_inv) = (ptr(t) for t in self.sm)
            if not stream_inverse:
                self.c.d_sm_inv = None
        if ctx_kv is not None:       # SDXL blocks: request r's prompt K|V rows (n_ctx[r] each)
            cu_c = np.concatenate([[0], np.cumsum(n_ctx)]).astype(np.int32)
            self.h_cu_ctx, self.cu_ctx, self.ctx_kv = cu_c, torch.tensor(cu_c, device=device), ctx_kv
            self.c.d_ctx_kv = ptr(ctx_kv)
            self.c.d_cu_ctx = ptr(self.cu_ctx)
            self.c.h_cu_ctx = self.h_cu_ctx.ctypes.data_as(C.c_void_p)

    @property
    def total_q(self):
        return int(self.h_cu_q[-1])

    @property
    def total_k(self):
        return int(self.h_cu_k[-1])


def workspace(H, F, dtype, max_q, max_u, device="cuda"):
    n = _lib.fps_block_workspace_bytes(H, F, dtype, max_q, max_u)
    return torch.empty(max(n, 256), dtype=torch.uint8, device=device)


def masked_block_forward(w: BlockWeights, b: VarlenBatch, x_act, kv, xu=None, kv_ready=None,
                         y_act=None, ws=None, stream=None):
    y_act = y_act if y_act is not None else torch.empty_like(x_act)
    ws = ws if ws is not None else workspace(w.H, w.F, w.dtype, b.total_q, b.c.total_u)
    ev = kv_ready.cuda_event if kv_ready is not None else None
    _lib.fps_masked_block_forward(C.byref(w.c), C.byref(b.c), ptr(x_act), ptr(y_act), ptr(kv),
                                  ptr(xu), ev, ptr(ws), ws.numel(), stream_ptr(stream))
    return y_act


def dense_block_forward(w: BlockWeights, b: VarlenBatch, x, kv=None, y=None, ws=None,
                        stream=None):
    y = y if y is not None else torch.empty_like(x)
    kv = kv if kv is not None else torch.empty((x.shape[0], 2 * w.H), dtype=x.dtype,
                                               device=x.device)
    ws = ws if ws is not None else workspace(w.H, w.F, w.dtype, b.total_q, 0)
    _lib.fps_dense_block_forward(C.byref(w.c), C.byref(b.c), ptr(x), ptr(y), ptr(kv), ptr(ws),
                                 ws.numel(), stream_ptr(stream))
    return y, kv


def masked_attention(q, kv, n_active, L, heads, out=None, stream=None):
    """a6 through fps_masked_attention: q [sum n, H], kv [sum L, 2H] (K|V rows)."""
    H = q.shape[1]
    cu_q = np.concatenate([[0], np.cumsum(n_active)]).astype(np.int32)
    cu_k = np.concatenate([[0], np.cumsum(L)]).astype(np.int32)
    d_cu_q = torch.tensor(cu_q, device=q.device)
    d_cu_k = torch.tensor(cu_k, device=q.device)
    out = out if out is not None else torch.empty_like(q)
    dt = FPS_BF16 if q.dtype == torch.bfloat16 else FPS_F32
    _lib.fps_masked_attention(dt, ptr(q), ptr(kv), ptr(out), heads, H // heads, ptr(d_cu_q),
                              ptr(d_cu_k), cu_q.ctypes.data, cu_k.ctypes.data, len(n_active),
                              stream_ptr(stream))
    out._fps_keep = (d_cu_q, d_cu_k, cu_q, cu_k)          # keep the index arrays alive
    return out


def linear(a, w, bias=None, act=0, out=None, stream=None):
    """out = act(a w^T + bias) through fps_linear (tcgen05 GEMM for bf16)."""
    M, K = a.shape
    N = w.shape[0]
    out = out if out is not None else torch.empty(M, N, dtype=a.dtype, device=a.device)
    dt = FPS_BF16 if a.dtype == torch.bfloat16 else FPS_F32
    _lib.fps_linear(dt, ptr(a), ptr(w), ptr(bias), M, N, K, act, ptr(out), stream_ptr(stream))
    return out


# ---------------------------------------------------------------------------------------
def plan_pipeline(c_cached, c_dense, load, mode, final_load=0.0, cross_step=False):
    """Alg. 1 (host, in the library). Returns (use_cache list, latency).  cross_step: the
    cross-step prefetch planner (R26)."""
    N = len(c_cached)
    arr = lambda v: (C.c_double * N)(*map(float, v))
    use = (C.c_uint8 * max(N, 1))()
    lat = C.c_double()
    f = _lib.fps_plan_pipeline_cross if cross_step else _lib.fps_plan_pipeline
    f(arr(c_cached), arr(c_dense), arr(load), N, mode, float(final_load), use, C.byref(lat))
    return [int(use[i]) for i in range(N)], lat.value


def plan_pipeline_kv_transition(c_cached, c_dense, c_transition, load, final_load=0.0,
                                cross_step=False):
    """KV-mode Alg. 1 with the transition block (R28). Returns (use_cache list, latency)."""
    N = len(c_cached)
    arr = lambda v: (C.c_double * max(N, 1))(*map(float, v))
    use = (C.c_uint8 * max(N, 1))()
    lat = C.c_double()
    _lib.fps_plan_pipeline_kv_transition(arr(c_cached), arr(c_dense), arr(c_transition), arr(load),
                                         N, float(final_load), int(bool(cross_step)), use,
                                         C.byref(lat))
    return [int(use[i]) for i in range(N)], lat.value


def pipeline_latency(use, c_cached, c_dense, load, mode, final_load=0.0, cross_step=False):
    N = len(use)
    arr = lambda v: (C.c_double * N)(*map(float, v))
    f = _lib.fps_pipeline_latency_cross if cross_step else _lib.fps_pipeline_latency
    return f((C.c_uint8 * max(N, 1))(*use), arr(c_cached), arr(c_dense), arr(load), N, mode,
             float(final_load))


class Cache:
    """fps_cache_t: pinned host arena of template activations (L203)."""

    def __init__(self, mode, dtype, H, L_img, n_layers, n_steps, n_templates=1, n_entries=0,
                 copy_method=0, copy_ctas=0, location=0, shm_path=None, peer_handle=None):
        self._shm = shm_path.encode() if shm_path else None
        self._peer = (C.c_uint8 * 64).from_buffer_copy(peer_handle) if peer_handle else None
        self.desc = fps_cache_desc(mode, dtype, H, L_img, n_layers, n_steps, n_templates,
                                   n_entries, copy_method, copy_ctas, location, self._shm,
                                   C.cast(self._peer, C.c_void_p) if self._peer is not None else None)
        h = C.c_void_p()
        _lib.fps_cache_create(C.byref(self.desc), C.byref(h))
        self.h = h
        self.mode, self.dtype, self.H, self.L_img = mode, dtype, H, L_img

    def close(self):
        if self.h:
            _lib.fps_cache_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def export_ipc(self):
        """64-byte CUDA IPC handle of an HBM-tier arena (NEXT-1 peer tier)."""
        h = (C.c_uint8 * 64)()
        _lib.fps_cache_export_ipc(self.h, h)
        return bytes(h)

    def entry_numpy(self, template_id, step, layer):
        """Host view of an entry as raw uint16 (bf16) / float32 numpy array [L_img, width]."""
        p = _lib.fps_cache_entry_host_ptr(self.h, template_id, step, layer)
        nb = _lib.fps_cache_entry_bytes(self.h, layer)
        buf = (C.c_uint8 * nb).from_address(p)
        a = np.frombuffer(buf, dtype=np.uint16 if self.dtype == FPS_BF16 else np.float32)
        return a.reshape(self.L_img, -1)

    def store(self, template_id, step, layer, src, stream=None):
        _lib.fps_cache_store(self.h, template_id, step, layer, ptr(src),
                             src[0].numel() * src.element_size(), stream_ptr(stream))

    def prefetch(self, items, load_stream=None, ready_event=None):
        arr = (fps_prefetch_item * max(len(items), 1))(*items)
        _lib.fps_cache_prefetch(self.h, arr, len(items), stream_ptr(load_stream), None)
        if ready_event is not None:       # torch creates its events lazily: record it here
            ready_event.record(load_stream if load_stream is not None
                               else torch.cuda.current_stream())


class Engine:
    """fps_engine_t: N-block stack with step-level continuous batching (fps_run_batch)."""

    def __init__(self, layers, heads, mode, dtype, L_img, L_txt, max_batch, n_steps, deltas,
                 cache: Cache, mod_table=None, slots=0, plan_policy=0, plan=None,
                 cost_model=(0.0, 0.0, 0.0, 0.0), L_ctx=0, mod_width=0, cross_step=False,
                 sampler=0, sigmas=None, layer_comp=None):
        self.layers = layers                      # list[BlockWeights] (keeps tensors alive)
        self._w = (fps_block_weights * len(layers))(*[l.c for l in layers])
        self._deltas = (C.c_float * n_steps)(*map(float, deltas))
        self._plan = (C.c_uint8 * len(layers))(*(plan or [0] * len(layers)))
        self._sigmas = (C.c_float * (n_steps + 1))(*map(float, sigmas)) if sigmas is not None else None
        self._layer_comp = ((C.c_double * (2 * len(layers)))(*[float(v) for ab in layer_comp for v in ab])
                            if layer_comp is not None else None)
        self.mod_table = mod_table
        self.cache = cache
        H, F = layers[0].H, layers[0].F
        d = fps_engine_desc(H, heads, F, len(layers), dtype, mode, L_img, L_txt, max_batch,
                            n_steps, C.cast(self._w, C.c_void_p), ptr(mod_table),
                            C.cast(self._deltas, C.c_void_p), cache.h, slots, plan_policy,
                            C.cast(self._plan, C.c_void_p), (C.c_double * 4)(*cost_model),
                            L_ctx, max((getattr(l, "D_ctx", 0) for l in layers), default=0),
                            mod_width, int(cross_step), int(sampler),
                            C.cast(self._sigmas, C.c_void_p) if self._sigmas is not None else None,
                            C.cast(self._layer_comp, C.c_void_p) if self._layer_comp is not None else None)
        self.desc = d
        h = C.c_void_p()
        _lib.fps_engine_create(C.byref(d), C.byref(h))
        self.h = h
        self.n_layers = len(layers)

    def close(self):
        if self.h:
            _lib.fps_engine_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def run_batch(self, reqs, n_steps, stream=None, load_stream=None):
        """reqs: list of dicts with template_id, step, n_steps, mask (cuda uint8), x (cuda),
        and ctx (cuda [L_ctx, D_ctx]) for SDXL blocks. Updates each dict's step/status in place."""
        arr = (fps_request * max(len(reqs), 1))()
        for i, r in enumerate(reqs):
            arr[i] = fps_request(r["template_id"], r["step"], r["n_steps"], ptr(r["mask"]),
                                 ptr(r["x"]), 0, ptr(r.get("ctx")), ptr(r.get("z")),
                                 ptr(r.get("noise")))
        ls = stream_ptr(load_stream) if load_stream is not None else None
        _lib.fps_run_batch(self.h, arr, len(reqs), n_steps, stream_ptr(stream), ls)
        for i, r in enumerate(reqs):
            r["step"], r["status"] = arr[i].step, arr[i].status
        return reqs

    def last_plan(self):
        use = (C.c_uint8 * self.n_layers)()
        lat = C.c_double()
        _lib.fps_engine_last_plan(self.h, use, C.byref(lat))
        return [int(u) for u in use], lat.value

    def last_launches(self):
        return int(_lib.fps_engine_last_launches(self.h))
