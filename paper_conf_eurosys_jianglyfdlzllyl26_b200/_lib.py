"""ctypes binding of libflashps.so (include/flashps.h). Argument marshalling only.

Every function here has the C name and forwards plain pointers/sizes; torch supplies device
memory and streams.  There is no fallback: importing this module on a machine where the library
is missing raises, and device calls fail with FlashPSError when no sm_100 GPU is usable.
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# FPS_LIB selects another in-tree build of the same library (used by tools/ for A/B timing)
LIB_PATH = os.environ.get("FPS_LIB") or os.path.join(_HERE, "libflashps.so")

FPS_OK, FPS_EINVAL, FPS_ECUDA, FPS_ENOMEM, FPS_EUNSUPPORTED, FPS_ESTATE = 0, -1, -2, -3, -4, -5
FPS_F32, FPS_BF16 = 0, 1
FPS_MODE_KV, FPS_MODE_Y = 0, 1
FPS_BLOCK_SEQ, FPS_BLOCK_PAR, FPS_BLOCK_SDXL, FPS_BLOCK_DOUBLE = 0, 1, 2, 3
FPS_SAMPLER_EULER, FPS_SAMPLER_FLOW_BLEND = 0, 1

vp, i32, u32, i64, sz, dbl = C.c_void_p, C.c_int32, C.c_uint32, C.c_int64, C.c_size_t, C.c_double
P_i32, P_u8, P_dbl, P_f32 = C.POINTER(C.c_int32), C.POINTER(C.c_uint8), C.POINTER(C.c_double), C.POINTER(C.c_float)


class FlashPSError(RuntimeError):
    def __init__(self, fn, code, msg):
        super().__init__(f"{fn} -> {code}: {msg}")
        self.code = code


class fps_cache_desc(C.Structure):
    _fields_ = [("mode", i32), ("dtype", i32), ("H", i32), ("L_img", i32), ("n_layers", i32),
                ("n_steps", i32), ("n_templates", i32), ("n_entries", i32),
                ("copy_method", i32), ("copy_ctas", i32), ("location", i32),
                ("shm_path", C.c_char_p), ("peer_ipc_handle", vp)]


class fps_prefetch_item(C.Structure):
    _fields_ = [("template_id", u32), ("step", i32), ("layer", i32), ("n_rows", i32),
                ("d_rows", vp), ("h_rows", vp), ("d_dst", vp), ("dst_row_bytes", i32)]


class fps_block_weights(C.Structure):
    _fields_ = [("H", i32), ("heads", i32), ("head_dim", i32), ("F", i32), ("dtype", i32),
                ("w_qkv", vp), ("b_qkv", vp), ("w_o", vp), ("b_o", vp), ("w_up", vp),
                ("b_up", vp), ("w_down", vp), ("b_down", vp), ("kind", i32), ("D_ctx", i32),
                ("ln1_w", vp), ("ln1_b", vp), ("ln2_w", vp), ("ln2_b", vp), ("ln3_w", vp),
                ("ln3_b", vp), ("w_q2", vp), ("b_q2", vp), ("w_kv2", vp), ("b_kv2", vp),
                ("w_o2", vp), ("b_o2", vp), ("t_qkv", vp), ("tb_qkv", vp), ("t_o", vp),
                ("tb_o", vp), ("t_up", vp), ("tb_up", vp), ("t_down", vp), ("tb_down", vp)]


class fps_varlen_batch(C.Structure):
    _fields_ = [("n_req", i32), ("total_q", i32), ("total_k", i32), ("max_q", i32),
                ("max_k", i32), ("d_cu_q", vp), ("d_cu_k", vp), ("h_cu_q", vp), ("h_cu_k", vp),
                ("d_q_row", vp), ("d_mod", vp), ("mode", i32), ("total_u", i32),
                ("d_cu_u", vp), ("d_u_src", vp), ("d_u_row", vp), ("d_ctx_kv", vp),
                ("d_cu_ctx", vp), ("h_cu_ctx", vp), ("mod_stride", i32), ("total_q_img", i32),
                ("d_sm_perm", vp), ("d_sm_kvrow", vp), ("d_cu_img", vp), ("d_cu_txt", vp),
                ("d_sm_inv", vp), ("x_full_rows", i32)]


class fps_engine_desc(C.Structure):
    _fields_ = [("H", i32), ("heads", i32), ("F", i32), ("n_layers", i32), ("dtype", i32),
                ("mode", i32), ("L_img", i32), ("L_txt", i32), ("max_batch", i32),
                ("n_steps", i32), ("layers", vp), ("d_mod_table", vp), ("h_deltas", vp),
                ("cache", vp), ("slots", i32), ("plan_policy", i32), ("h_plan", vp),
                ("cost_model", dbl * 4), ("L_ctx", i32), ("D_ctx", i32), ("mod_width", i32),
                ("cross_step", i32), ("sampler", i32), ("h_sigmas", vp), ("h_layer_comp", vp)]


class fps_request(C.Structure):
    _fields_ = [("template_id", u32), ("step", i32), ("n_steps", i32), ("d_mask", vp),
                ("d_x", vp), ("status", i32), ("d_ctx", vp), ("d_z", vp), ("d_noise", vp)]


# (name, restype, argtypes, checked)
_SIGS = [
    ("fps_last_error", C.c_char_p, [], False),
    ("fps_abi_version", i32, [], False),
    ("fps_device_ok", i32, [], False),
    ("fps_launch_count", i64, [], False),
    ("fps_set_disable_tc", None, [i32], False),
    ("fps_profile_enable", None, [i32], False),
    ("fps_profile_read", i32, [P_dbl, P_dbl, P_dbl, C.POINTER(C.c_int64)], False),
    ("fps_profile_trace", i64, [P_dbl, P_dbl, C.POINTER(C.c_int32), C.POINTER(C.c_int64), i64], False),
    ("fps_mask_to_tokens", C.c_int, [vp, i32, i32, i32, i32, i32, vp, vp], True),
    ("fps_build_mask_index", C.c_int, [vp, vp, i32, i32, vp, vp, vp, vp], True),
    ("fps_gather_rows", C.c_int, [vp, vp, i32, i32, vp, vp], True),
    ("fps_scatter_rows", C.c_int, [vp, vp, i32, i32, vp, vp], True),
    ("fps_copy_rows", C.c_int, [vp, vp, vp, i32, i32, vp, vp], True),
    ("fps_cache_create", C.c_int, [C.POINTER(fps_cache_desc), C.POINTER(vp)], True),
    ("fps_cache_destroy", C.c_int, [vp], True),
    ("fps_cache_entry_host_ptr", vp, [vp, u32, i32, i32], False),
    ("fps_cache_entry_ptr", vp, [vp, u32, i32, i32], False),
    ("fps_cache_entry_bytes", sz, [vp, i32], False),
    ("fps_cache_export_ipc", C.c_int, [vp, vp], True),
    ("fps_cache_store", C.c_int, [vp, u32, i32, i32, vp, i32, vp], True),
    ("fps_cache_prefetch", C.c_int, [vp, C.POINTER(fps_prefetch_item), i32, vp, vp], True),
    ("fps_geglu_pack", C.c_int, [i32, vp, vp, i32, i32, vp, vp, vp], True),
    ("fps_context_kv", C.c_int, [C.POINTER(fps_block_weights), vp, i32, vp, vp], True),
    ("fps_block_workspace_bytes", sz, [i32, i32, i32, i32, i32], False),
    ("fps_masked_block_forward", C.c_int,
     [C.POINTER(fps_block_weights), C.POINTER(fps_varlen_batch), vp, vp, vp, vp, vp, vp, sz, vp],
     True),
    ("fps_linear", C.c_int, [i32, vp, vp, vp, i32, i32, i32, i32, vp, vp], True),
    ("fps_masked_attention", C.c_int, [i32, vp, vp, vp, i32, i32, vp, vp, vp, vp, i32, vp], True),
    ("fps_dense_block_forward", C.c_int,
     [C.POINTER(fps_block_weights), C.POINTER(fps_varlen_batch), vp, vp, vp, vp, sz, vp], True),
    ("fps_plan_pipeline", C.c_int, [P_dbl, P_dbl, P_dbl, i32, i32, dbl, P_u8, P_dbl], True),
    ("fps_pipeline_latency", dbl, [P_u8, P_dbl, P_dbl, P_dbl, i32, i32, dbl], False),
    ("fps_plan_pipeline_cross", C.c_int, [P_dbl, P_dbl, P_dbl, i32, i32, dbl, P_u8, P_dbl], True),
    ("fps_pipeline_latency_cross", dbl, [P_u8, P_dbl, P_dbl, P_dbl, i32, i32, dbl], False),
    ("fps_plan_pipeline_kv_transition", C.c_int, [P_dbl, P_dbl, P_dbl, P_dbl, i32, dbl, i32, P_u8, P_dbl], True),
    ("fps_engine_create", C.c_int, [C.POINTER(fps_engine_desc), C.POINTER(vp)], True),
    ("fps_engine_destroy", C.c_int, [vp], True),
    ("fps_run_batch", C.c_int, [vp, C.POINTER(fps_request), i32, i32, vp, vp], True),
    ("fps_engine_last_plan", C.c_int, [vp, P_u8, P_dbl], True),
    ("fps_engine_last_launches", i64, [vp], False),
    ("fps_engine_set_admission_reuse", None, [vp, i32], False),
    ("fps_engine_set_kv_transition", None, [vp, i32], False),
    ("fps_engine_set_skip_loads", None, [vp, i32], False),
    ("fps_engine_set_record", None, [vp, i32], False),
]

EXPORTED = [s[0] for s in _SIGS]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"libflashps.so not built at {LIB_PATH}: run __graft_entry__.build() "
                          "(no CPU fallback exists)")
    lib = C.CDLL(LIB_PATH)
    for name, res, args, _ in _SIGS:
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


lib = _load()


def _checked(name):
    f = getattr(lib, name)

    def call(*args):
        rc = f(*args)
        if rc != FPS_OK:
            raise FlashPSError(name, rc, lib.fps_last_error().decode(errors="replace"))
        return rc

    call.__name__ = name
    return call


for _name, _res, _args, _chk in _SIGS:
    globals()[_name] = _checked(_name) if _chk else getattr(lib, _name)
