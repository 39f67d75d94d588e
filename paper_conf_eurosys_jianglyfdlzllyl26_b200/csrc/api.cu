// C ABI entry points of libflashps: validation, dispatch, and the block-forward composition
// (PAPER.md L146 block; L157 mask-aware Y-mode; L161 KV-mode).  See include/flashps.h.
#include <cstring>
#include <mutex>
#include <vector>

#include "kernels.h"

namespace fps {

static thread_local std::string g_err;
thread_local long long g_launches = 0;
int g_disable_tc = 0;
int g_sm_reserved = 0;
int g_pdl = 1;
int g_y_grouped = 1;   // Y-mode parallel block: one grouped launch for W1(M) + K|V(U) (bit 15 off)
thread_local PdlFence g_pdl_fence;

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
}

fps_status fail(fps_status code, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

static int elt_size(int dtype) { return dtype == FPS_BF16 ? 2 : 4; }

// ---- profiling ------------------------------------------------------------------------------
namespace prof {
struct Rec {
  cudaEvent_t a, b;
  int kind;
  double flops, bytes;
  cudaStream_t s;
};
static bool g_on = false;
static std::vector<Rec> g_recs;
static std::vector<cudaEvent_t> g_pool;
static size_t g_used = 0;
static cudaEvent_t g_pending = nullptr;

static cudaEvent_t take() {
  if (g_used == g_pool.size()) {
    cudaEvent_t e;
    if (cudaEventCreate(&e) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    g_pool.push_back(e);
  }
  return g_pool[g_used++];
}
bool enabled() { return g_on; }
void begin(cudaStream_t s) {
  if (!g_on) return;
  g_pending = take();
  if (g_pending) cudaEventRecord(g_pending, s);
}
void end(cudaStream_t s, int kind, double flops, double bytes) {
  if (!g_on || !g_pending) return;
  cudaEvent_t b = take();
  if (!b) return;
  cudaEventRecord(b, s);
  g_recs.push_back(Rec{g_pending, b, kind, flops, bytes, s});
  g_pending = nullptr;
}
}  // namespace prof

static fps_status launch_gemm_impl(int dtype, const void* A, const void* B, int M, int N, int K,
                                   const Epilogue& ep, cudaStream_t s) {
  if (!(g_disable_tc & 1) && gemm_tc_supported(dtype, M, N, K))
    return launch_gemm_tc(A, B, M, N, K, ep, s);
  return launch_gemm_simt(dtype, A, B, M, N, K, ep, s);
}

fps_status launch_gemm(int dtype, const void* A, const void* B, int M, int N, int K,
                       const Epilogue& ep, cudaStream_t s) {
  if (M <= 0 || N <= 0) return FPS_OK;
  prof::begin(s);
  fps_status st = launch_gemm_impl(dtype, A, B, M, N, K, ep, s);
  const double e = elt_size(dtype);
  prof::end(s, prof::GEMM, 2.0 * M * N * K, e * ((double)M * K + (double)N * K + (double)M * N));
  return st;
}

fps_status launch_gemm_grouped(int dtype, const void* A, const void* B0, const void* B1, int M0,
                               int M1, int N, int K, const Epilogue& ep0, const Epilogue& ep1,
                               cudaStream_t s, int N1) {
  if (N1 <= 0) N1 = N;
  if (M1 <= 0) return launch_gemm(dtype, A, B0, M0, N, K, ep0, s);
  if (M0 <= 0) return launch_gemm(dtype, (const char*)A + (size_t)M0 * K * elt_size(dtype), B1, M1,
                                  N1, K, ep1, s);
  if ((g_disable_tc & 1) || !gemm_tc_supported(dtype, M0 + M1, N, K) ||
      !gemm_tc_supported(dtype, M0 + M1, N1, K)) {
    FPS_TRY(launch_gemm(dtype, A, B0, M0, N, K, ep0, s));
    return launch_gemm(dtype, (const char*)A + (size_t)M0 * K * elt_size(dtype), B1, M1, N1, K,
                       ep1, s);
  }
  prof::begin(s);
  fps_status st = launch_gemm_tc_grouped(A, B0, B1, M0, M1, N, K, ep0, ep1, s, N1);
  const double e = elt_size(dtype), M = (double)M0 + M1;
  const double MN = (double)M0 * N + (double)M1 * N1;
  prof::end(s, prof::GEMM, 2.0 * MN * K, e * (M * K + (double)(N + N1) * K + MN));
  return st;
}

fps_status launch_attention(int dtype, const void* q, const void* kv, void* o, int heads,
                            int head_dim, const int32_t* d_cu_q, const int32_t* d_cu_k,
                            const int32_t* h_cu_q, const int32_t* h_cu_k, int n_req, int total_q,
                            int max_q, int max_k, cudaStream_t s, int ldo,
                            const AttnScratch* sc, const int32_t* o_map) {
  (void)max_k;
  if (total_q <= 0) return FPS_OK;
  prof::begin(s);
  fps_status st;
  if (!(g_disable_tc & 2) && attention_tc_supported(dtype, head_dim) && h_cu_q && h_cu_k)
    st = launch_attention_tc(q, kv, o, heads, head_dim, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s,
                             ldo, sc, o_map);
  else
    st = launch_attention_simt(dtype, q, kv, o, heads, head_dim, d_cu_q, d_cu_k, n_req, total_q, s,
                               ldo, o_map);
  if (prof::enabled() && h_cu_q && h_cu_k) {
    // algorithmic work: QK^T and PV, 4 n_r L_r H FLOPs; bytes: Q, O once + K|V once per request
    double fl = 0, by = 0;
    const double H = (double)heads * head_dim, e = elt_size(dtype);
    for (int r = 0; r < n_req; ++r) {
      const double n = h_cu_q[r + 1] - h_cu_q[r], L = h_cu_k[r + 1] - h_cu_k[r];
      fl += 4.0 * n * L * H;
      by += e * (2.0 * n * H + 2.0 * L * H);
    }
    prof::end(s, prof::ATTN, fl, by);
  }
  return st;
}

struct BlockWs {
  char *h, *q, *ao, *x1, *h2, *u, *hu, *x2;
};

static size_t align256(size_t v) { return (v + 255) & ~size_t(255); }

static size_t ws_layout(int H, int F, int dtype, int max_q, int max_u, char* base, BlockWs* ws) {
  const size_t e = elt_size(dtype);
  size_t off = 0;
  auto take = [&](size_t bytes) {
    char* p = base ? base + off : nullptr;
    off += align256(bytes);
    return p;
  };
  char* h = take((size_t)max_q * H * e);
  char* q = take((size_t)max_q * H * e);
  char* ao = take((size_t)max_q * H * e);
  char* x1 = take((size_t)max_q * H * 4);              // fp32 for the SDXL block's residual stream
  char* h2 = take((size_t)max_q * H * e);
  char* u = take((size_t)max_q * F * e);
  // Y-mode: LN of all rows in token order; max_q rows of headroom in front, where the
  // sequential / SDXL block puts the compact rows M right before it (one A operand for the
  // grouped Q + K|V launch)
  char* hu = take((size_t)(2 * max_q + max_u) * H * e) + (base ? (size_t)max_q * H * e : 0);
  char* x2 = take((size_t)max_q * H * 4);              // SDXL block: after cross-attention (fp32)
  if (ws) *ws = BlockWs{h, q, ao, x1, h2, u, hu, x2};
  return off;
}

// Split-KV attention scratch inside the block workspace: buffers that are dead while the
// attention runs -- the LN output h (consumed by the QKV GEMM) for the statistics, and the MLP
// hidden u (written after the attention) or, for the parallel block whose u holds GELU(Z)
// already, the x1 buffer for the partial outputs.
static AttnScratch attn_scratch(const BlockWs& ws, int H, int F, int dtype, int max_q, bool par) {
  const size_t e = elt_size(dtype);
  AttnScratch sc{};
  sc.ml = ws.h;
  sc.ml_bytes = (size_t)max_q * H * e;
  sc.part = par ? ws.x1 : ws.u;
  sc.part_bytes = par ? (size_t)max_q * H * 4 : (size_t)max_q * F * e;
  return sc;
}

static fps_status check_weights(const fps_block_weights* w) {
  FPS_CHECK_ARG(w, "weights is NULL");
  FPS_CHECK_ARG(w->dtype == FPS_BF16 || w->dtype == FPS_F32, "dtype %d", w->dtype);
  FPS_CHECK_ARG(w->H > 0 && w->heads > 0 && w->head_dim > 0 && w->heads * w->head_dim == w->H,
                "H=%d heads=%d head_dim=%d", w->H, w->heads, w->head_dim);
  FPS_CHECK_ARG(w->F > 0, "F=%d", w->F);
  FPS_CHECK_ARG(w->kind >= FPS_BLOCK_SEQ && w->kind <= FPS_BLOCK_DOUBLE, "kind %d", w->kind);
  if (w->kind == FPS_BLOCK_DOUBLE)
    FPS_CHECK_ARG(w->w_qkv && w->w_o && w->w_up && w->w_down && w->t_qkv && w->t_o && w->t_up &&
                  w->t_down, "double-stream block: image or text weight pointer is NULL");
  if (w->kind == FPS_BLOCK_SDXL) {
    FPS_CHECK_ARG(w->w_qkv && w->w_o && w->w_up && w->w_down && w->w_q2 && w->w_kv2 && w->w_o2,
                  "SDXL block: weight pointer is NULL");
    FPS_CHECK_ARG(w->ln1_w && w->ln1_b && w->ln2_w && w->ln2_b && w->ln3_w && w->ln3_b,
                  "SDXL block: LayerNorm gamma / beta is NULL");
    FPS_CHECK_ARG(w->D_ctx > 0, "SDXL block: D_ctx=%d", w->D_ctx);
    if (w->dtype != FPS_BF16 || (g_disable_tc & 1) || w->H % 64 || w->F % 64 || w->D_ctx % 64)
      return fail(FPS_EUNSUPPORTED,
                  "SDXL block: bf16 tcgen05 path only (H=%d, F=%d, D_ctx=%d multiples of 64)",
                  w->H, w->F, w->D_ctx);
  } else if (w->kind == FPS_BLOCK_DOUBLE) {
  } else if (w->kind == FPS_BLOCK_PAR)
    FPS_CHECK_ARG(w->w_qkv && w->w_down && !w->w_o && !w->b_o && !w->w_up && !w->b_up,
                  "parallel block: w_qkv (W1) and w_down (W2) set, w_o/b_o/w_up/b_up NULL");
  else
    FPS_CHECK_ARG(w->w_qkv && w->w_o && w->w_up && w->w_down, "weight pointer is NULL");
  const int vec = 16 / elt_size(w->dtype);
  FPS_CHECK_ARG(w->H % vec == 0 && w->F % vec == 0, "H and F must be multiples of %d", vec);
  return FPS_OK;
}

static fps_status check_batch(const fps_varlen_batch* b) {
  FPS_CHECK_ARG(b, "batch is NULL");
  FPS_CHECK_ARG(b->n_req >= 0 && b->total_q >= 0 && b->total_k >= 0, "negative sizes");
  FPS_CHECK_ARG(b->n_req == 0 || (b->d_cu_q && b->d_cu_k), "cu arrays are NULL");
  FPS_CHECK_ARG(b->mode == FPS_MODE_KV || b->mode == FPS_MODE_Y, "mode %d", b->mode);
  if (b->mode == FPS_MODE_Y && b->total_u > 0) {
    FPS_CHECK_ARG(b->d_cu_u && b->d_u_src && b->d_u_row, "Y-mode needs cu_u/u_src/u_row");
    FPS_CHECK_ARG(b->total_q + b->total_u == b->total_k,
                  "Y-mode: every merged row must be active or cached (%d + %d != %d)", b->total_q,
                  b->total_u, b->total_k);
  }
  return FPS_OK;
}

static fps_status check_streams(const fps_block_weights* w, const fps_varlen_batch* b) {
  if (w->kind != FPS_BLOCK_DOUBLE || b->n_req == 0 || b->total_q == 0) return FPS_OK;
  FPS_CHECK_ARG(b->d_sm_perm && b->d_sm_kvrow && b->d_cu_img && b->d_cu_txt,
                "double-stream block: stream-major order (d_sm_perm, d_sm_kvrow, d_cu_img, "
                "d_cu_txt) required");
  FPS_CHECK_ARG(b->total_q_img >= 0 && b->total_q_img <= b->total_q, "total_q_img %d",
                b->total_q_img);
  return FPS_OK;
}

static fps_status check_ctx(const fps_block_weights* w, const fps_varlen_batch* b) {
  if (w->kind != FPS_BLOCK_SDXL || b->n_req == 0 || b->total_q == 0) return FPS_OK;
  FPS_CHECK_ARG(b->d_ctx_kv && b->d_cu_ctx && b->h_cu_ctx && b->h_cu_q,
                "SDXL block: d_ctx_kv / cu_ctx (device and host) / h_cu_q required");
  for (int r = 0; r < b->n_req; ++r)
    FPS_CHECK_ARG(b->h_cu_ctx[r + 1] > b->h_cu_ctx[r],
                  "SDXL block: request %d has an empty prompt context", r);
  return FPS_OK;
}

// Double-stream (Flux MM-DiT) block, reading R25.  The active rows are processed in
// stream-major order (all image rows, then all text rows) so each stream's projections are
// one GEMM over contiguous rows with that stream's weights; Q is scattered back to the
// request-major order the varlen attention reads, its output gathered to stream-major again,
// and the final epilogue writes y in request-major order.
static fps_status double_block_forward(const fps_block_weights* w, const fps_varlen_batch* b,
                                       const void* x_act, void* y_act, void* kv, const void* xu,
                                       cudaEvent_t kv_ready, void* d_ws, size_t ws_bytes,
                                       cudaStream_t s) {
  const int H = w->H, F = w->F, dt = w->dtype, tq = b->total_q;
  const int tu = (b->mode == FPS_MODE_Y) ? b->total_u : 0;
  const int ti = b->total_q_img, tt = tq - ti;
  const size_t e = elt_size(dt), rowb = (size_t)H * e;
  BlockWs ws;
  const size_t need = ws_layout(H, F, dt, tq, tu, (char*)d_ws, &ws);
  FPS_CHECK_ARG(ws_bytes >= need, "workspace %zu < %zu bytes", ws_bytes, need);
  const int MS = b->mod_stride > 0 ? b->mod_stride : 12 * H;
  const char* mod = (const char*)b->d_mod;
  auto modp = [&](int stream, int off) -> const void* {
    return mod ? mod + ((size_t)stream * 6 * H + (size_t)off * H) * e : nullptr;
  };
  const int32_t* perm = b->d_sm_perm;
  const int32_t* kvrow = b->d_sm_kvrow;
  // a2 fused into the consumers: x_act may be the full merged buffer, read at the active rows'
  // merged rows (stream-major order -> d_sm_kvrow) instead of a compact gathered copy
  const int32_t* xperm = b->x_full_rows ? kvrow : perm;
  const int32_t* cu[2] = {b->d_cu_img, b->d_cu_txt};
  const int rows0[2] = {0, ti}, nrows[2] = {ti, tt};
  const void* Wqkv[2] = {w->w_qkv, w->t_qkv};
  const void* Bqkv[2] = {w->b_qkv, w->tb_qkv};
  const void* Wo[2] = {w->w_o, w->t_o};
  const void* Bo[2] = {w->b_o, w->tb_o};
  const void* Wup[2] = {w->w_up, w->t_up};
  const void* Bup[2] = {w->b_up, w->tb_up};
  const void* Wdn[2] = {w->w_down, w->t_down};
  const void* Bdn[2] = {w->b_down, w->tb_down};
  char* x_sm = ws.x2;      // x in stream-major order (the fp32-sized buffer is free here)
  char* ao_sm = ws.h2;     // attention output, stream-major (h2 is written only after its use)
  auto at = [&](char* base, int st, size_t width = 0) {
    return base + (size_t)rows0[st] * (width ? width : rowb);
  };
  // Without reordering copies: the norms read x through the stream-major order, the O
  // projection reads its residual through it, and the attention writes its output rows
  // straight to their stream-major positions (d_sm_inv).  The copy path remains for the
  // attention kernels forced by tests.
  const bool direct = b->d_sm_inv != nullptr && (g_attn_force == 0 || g_attn_force == 3);
  if (tq > 0) {
    if (!direct) FPS_TRY(launch_copy_rows(x_act, xperm, nullptr, tq, (int)rowb, x_sm, s));
    // a4 per stream; a5 for both streams in one grouped launch: Q -> request-major rows,
    // K|V -> merged key rows
    // both streams' norms in one launch (rows >= ti: the text stream's vectors)
    FPS_TRY(launch_ln_mod2(dt, direct ? x_act : x_sm, direct ? xperm : nullptr, tq, H, ws.h, cu[0],
                           cu[1], ti, b->n_req, mod, 0, 6 * H, s, MS));
    Epilogue ep[2] = {};
    for (int st = 0; st < 2; ++st) {
      ep[st].bias = Bqkv[st];
      ep[st].out0 = ws.q; ep[st].ld0 = H; ep[st].map0 = perm + rows0[st];
      ep[st].out1 = kv; ep[st].ld1 = 2 * H; ep[st].map1 = kvrow + rows0[st];
      ep[st].split = H;
    }
    FPS_TRY(launch_gemm_grouped(dt, ws.h, Wqkv[0], Wqkv[1], ti, tt, 3 * H, H, ep[0], ep[1], s));
  }
  if (tu > 0) {
    // Y-mode: cached input rows U (image rows, R9) -> image-stream LN -> K|V projection
    if (kv_ready) FPS_CUDA_TRY(stream_wait(s, kv_ready, 0));
    kv_ready = nullptr;
    FPS_TRY(launch_ln_mod(dt, xu, b->d_u_src, tu, H, ws.hu, b->d_cu_u, b->n_req, mod, 0, s,
                          nullptr, MS));
    Epilogue ep{};
    ep.bias = w->b_qkv ? (const char*)w->b_qkv + (size_t)H * e : nullptr;
    ep.out0 = kv; ep.ld0 = 2 * H; ep.map0 = b->d_u_row;
    ep.split = 2 * H;
    FPS_TRY(launch_gemm(dt, ws.hu, (const char*)w->w_qkv + (size_t)H * H * e, tu, 2 * H, H, ep, s));
  }
  if (tq == 0) return FPS_OK;
  // a6: joint attention of both streams' queries over the merged keys
  if (kv_ready) FPS_CUDA_TRY(stream_wait(s, kv_ready, 0));
  const AttnScratch sc = attn_scratch(ws, H, F, dt, tq, false);
  if (direct) {
    FPS_TRY(launch_attention(dt, ws.q, kv, ao_sm, w->heads, w->head_dim, b->d_cu_q, b->d_cu_k,
                             b->h_cu_q, b->h_cu_k, b->n_req, tq, b->max_q, b->max_k, s, 0, &sc,
                             b->d_sm_inv));
  } else {
    FPS_TRY(launch_attention(dt, ws.q, kv, ws.ao, w->heads, w->head_dim, b->d_cu_q, b->d_cu_k,
                             b->h_cu_q, b->h_cu_k, b->n_req, tq, b->max_q, b->max_k, s, 0, &sc));
    FPS_TRY(launch_copy_rows(ws.ao, perm, nullptr, tq, (int)rowb, ao_sm, s));
  }
  // a7, a8: each projection one grouped launch over both streams (their own weights, adaLN
  // gates and request offsets); y written back in request-major order
  Epilogue eo[2] = {}, eu[2] = {}, ed[2] = {};
  for (int st = 0; st < 2; ++st) {   // x1 = x + gate1 (A Wo^T + bo)
    eo[st].bias = Bo[st];
    if (direct) {
      eo[st].resid = x_act; eo[st].resid_map = xperm + rows0[st];
    } else {
      eo[st].resid = at(x_sm, st);
    }
    eo[st].ld_resid = H;
    eo[st].gate = modp(st, 2); eo[st].gate_stride = MS; eo[st].cu = cu[st]; eo[st].n_req = b->n_req;
    eo[st].out0 = at(ws.x1, st); eo[st].ld0 = H; eo[st].split = H;
  }
  FPS_TRY(launch_gemm_grouped(dt, ao_sm, Wo[0], Wo[1], ti, tt, H, H, eo[0], eo[1], s));
  FPS_TRY(launch_ln_mod2(dt, ws.x1, nullptr, tq, H, ws.h2, cu[0], cu[1], ti, b->n_req, mod,
                         3 * H, 6 * H, s, MS));
  for (int st = 0; st < 2; ++st) {
    eu[st].bias = Bup[st]; eu[st].act = 1;
    eu[st].out0 = at(ws.u, st, (size_t)F * e); eu[st].ld0 = F; eu[st].split = F;
    ed[st].bias = Bdn[st];
    ed[st].resid = at(ws.x1, st); ed[st].ld_resid = H;
    ed[st].gate = modp(st, 5); ed[st].gate_stride = MS; ed[st].cu = cu[st]; ed[st].n_req = b->n_req;
    ed[st].out0 = y_act; ed[st].ld0 = H; ed[st].map0 = perm + rows0[st]; ed[st].split = H;
  }
  FPS_TRY(launch_gemm_grouped(dt, ws.h2, Wup[0], Wup[1], ti, tt, F, H, eu[0], eu[1], s));
  return launch_gemm_grouped(dt, ws.u, Wdn[0], Wdn[1], ti, tt, H, F, ed[0], ed[1], s);
}

static fps_status block_forward(const fps_block_weights* w, const fps_varlen_batch* b,
                                const void* x_act, void* y_act, void* kv, const void* xu,
                                cudaEvent_t kv_ready, void* d_ws, size_t ws_bytes,
                                cudaStream_t s) {
  const int H = w->H, F = w->F, dt = w->dtype, tq = b->total_q;
  const int tu = (b->mode == FPS_MODE_Y) ? b->total_u : 0;
  const size_t e = elt_size(dt);
  BlockWs ws;
  const size_t need = ws_layout(H, F, dt, tq, tu, (char*)d_ws, &ws);
  FPS_CHECK_ARG(ws_bytes >= need, "workspace %zu < %zu bytes", ws_bytes, need);
  if (w->kind == FPS_BLOCK_DOUBLE)
    return double_block_forward(w, b, x_act, y_act, kv, xu, kv_ready, d_ws, ws_bytes, s);
  const bool sdxl = w->kind == FPS_BLOCK_SDXL;
  const int MS = b->mod_stride > 0 ? b->mod_stride : 6 * H;
  const char* mod = sdxl ? nullptr : (const char*)b->d_mod;
  auto modp = [&](int off) -> const void* { return mod ? mod + (size_t)off * H * e : nullptr; };
  // a2 fused into the consumers: with x_full_rows the block reads its active input rows
  // straight out of the full merged buffer at d_q_row (first norm + residual), no gathered copy
  const int32_t* xr = b->x_full_rows ? b->d_q_row : nullptr;
  // a4, the first norm: adaLN-modulated LN, or the SDXL block's affine LN (reading R24)
  auto ln1 = [&](const void* x, const int32_t* rows, int n, void* out, const int32_t* cu,
                 const int32_t* out_rows) -> fps_status {
    if (sdxl) return launch_ln_affine(dt, x, rows, n, H, out, w->ln1_w, w->ln1_b, s, out_rows);
    return launch_ln_mod(dt, x, rows, n, H, out, cu, b->n_req, mod, 0, s, out_rows, MS);
  };

  // Y-mode, sequential block: Q over the active rows, K|V in ONE GEMM over all rows of the
  // merged buffer (fresh rows M and cached input rows U, normalised into token order) -- the same
  // FLOPs as the QKV GEMM on M plus a K|V GEMM on U, in fewer waves with no 256-row padding at
  // the M/U split (C3: 6 + 1 waves instead of 3 + 5)
  const bool y_split = tu > 0 && tq > 0 && w->kind != FPS_BLOCK_PAR;
  if (y_split) {
    // one norm launch for both row sets (after the load of x[U]): rows M -> ws.h (compact, the Q
    // GEMM's A) and ws.hu at their token rows; cached rows U -> ws.hu at theirs
    if (kv_ready) FPS_CUDA_TRY(stream_wait(s, kv_ready, 0));
    kv_ready = nullptr;
    // the compact rows M sit right before ws.hu (its headroom), so Q over rows M and K|V over
    // all rows are ONE grouped launch on one A operand (per-problem N: H and 2H); bit-identical
    // to two launches (flag bit 15 selects those)
    char* hq = g_y_grouped ? ws.hu - (size_t)tq * H * e : ws.h;
    FPS_TRY(launch_ln_ysplit(dt, x_act, xr, tq, xu, b->d_u_src, tu, H, hq, ws.hu, b->d_q_row,
                             b->d_u_row, b->d_cu_q, b->d_cu_u, b->n_req, mod, 0, MS,
                             sdxl ? w->ln1_w : nullptr, sdxl ? w->ln1_b : nullptr, s));
    Epilogue eq{};
    eq.bias = w->b_qkv;
    eq.out0 = ws.q; eq.ld0 = H; eq.split = H;
    Epilogue ek{};
    ek.bias = w->b_qkv ? (const char*)w->b_qkv + (size_t)H * e : nullptr;
    ek.out0 = kv; ek.ld0 = 2 * H; ek.split = 2 * H;
    if (g_y_grouped) {
      FPS_TRY(launch_gemm_grouped(dt, hq, w->w_qkv, (const char*)w->w_qkv + (size_t)H * H * e, tq,
                                  b->total_k, H, H, eq, ek, s, 2 * H));
    } else {
      FPS_TRY(launch_gemm(dt, hq, w->w_qkv, tq, H, H, eq, s));
      FPS_TRY(launch_gemm(dt, ws.hu, (const char*)w->w_qkv + (size_t)H * H * e, b->total_k, 2 * H,
                          H, ek, s));
    }
  }
  // Y-mode parallel block: the W1 GEMM of rows M ([Q|K|V|Z]) and the K|V GEMM of the cached
  // rows U in ONE grouped launch (A = both rows' LN outputs, stacked in ws.hu): the persistent
  // grid runs both problems' tiles back to back, so the K|V problem's partial last wave is
  // filled (C3: 504 + 312 pair tiles = 11.03 waves in one launch vs 7 + 5 in two).  Per element
  // the arithmetic is unchanged (same K order and epilogue), so outputs are bit-identical.
  const bool par_group = w->kind == FPS_BLOCK_PAR && tq > 0 && tu > 0 && g_y_grouped;
  if (tq > 0 && !y_split) {
    // a4: h1 = LN(x)(1+scale1)+shift1 on active rows (Y-mode parallel block: and on the cached
    // rows U in the same launch, rows [tq, tq + tu) of ws.hu -- after the load of x[U])
    if (par_group) {
      if (kv_ready) FPS_CUDA_TRY(stream_wait(s, kv_ready, 0));
      kv_ready = nullptr;
      FPS_TRY(launch_ln_mod_2src(dt, x_act, xr, tq, xu, b->d_u_src, tu, H, ws.hu, b->d_cu_q,
                                 b->d_cu_u, b->n_req, mod, 0, s, MS));
    } else {
      FPS_TRY(ln1(x_act, xr, tq, ws.h, b->d_cu_q, nullptr));
    }
    // a5: [tq,H] x [3H,H]^T; Q -> compact, K|V -> merged key rows at original positions
    Epilogue ep{};
    ep.bias = w->b_qkv;
    ep.out0 = ws.q; ep.ld0 = H; ep.map0 = nullptr;
    ep.out1 = kv; ep.ld1 = 2 * H; ep.map1 = b->d_q_row;
    ep.split = H;
    int n_out = 3 * H;
    if (w->kind == FPS_BLOCK_PAR) {     // + MLP input rows: GELU(Z) -> cat[:, H:H+F]
      ep.out2 = (char*)ws.ao + (size_t)H * e; ep.ld2 = H + F; ep.split2 = 3 * H;
      ep.act = 1; ep.act_from = 3 * H;
      n_out += F;
    }
    if (par_group) {
      // Y-mode: K|V of the cached block-input rows U (normalised above)
      Epilogue ek{};
      ek.bias = w->b_qkv ? (const char*)w->b_qkv + (size_t)H * e : nullptr;
      ek.out0 = kv; ek.ld0 = 2 * H; ek.map0 = b->d_u_row;
      ek.split = 2 * H;
      FPS_TRY(launch_gemm_grouped(dt, ws.hu, w->w_qkv, (const char*)w->w_qkv + (size_t)H * H * e,
                                  tq, tu, n_out, H, ep, ek, s, 2 * H));
    } else {
      FPS_TRY(launch_gemm(dt, ws.h, w->w_qkv, tq, n_out, H, ep, s));
    }
  }
  if (tu > 0 && !y_split && !par_group) {
    // Y-mode: cached block-input rows U -> LN -> K|V projection (Fig. 5-Bottom, reading R5)
    if (kv_ready) FPS_CUDA_TRY(stream_wait(s, kv_ready, 0));
    kv_ready = nullptr;
    FPS_TRY(ln1(xu, b->d_u_src, tu, ws.hu, b->d_cu_u, nullptr));
    Epilogue ep{};
    ep.bias = w->b_qkv ? (const char*)w->b_qkv + (size_t)H * e : nullptr;
    ep.out0 = kv; ep.ld0 = 2 * H; ep.map0 = b->d_u_row;
    ep.split = 2 * H;
    FPS_TRY(launch_gemm(dt, ws.hu, (const char*)w->w_qkv + (size_t)H * H * e, tu, 2 * H, H, ep, s));
  }
  if (tq == 0) return FPS_OK;
  if (w->kind == FPS_BLOCK_PAR) {
    // parallel block (reading R23): ws.ao..ws.u hold cat = [A | GELU(Z)], [tq, H+F]
    char* cat = ws.ao;
    if (kv_ready) FPS_CUDA_TRY(stream_wait(s, kv_ready, 0));
    const AttnScratch sc = attn_scratch(ws, H, F, dt, tq, true);
    FPS_TRY(launch_attention(dt, ws.q, kv, cat, w->heads, w->head_dim, b->d_cu_q, b->d_cu_k,
                             b->h_cu_q, b->h_cu_k, b->n_req, tq, b->max_q, b->max_k, s, H + F,
                             &sc));
    Epilogue ep{};
    ep.bias = w->b_down;
    ep.resid = x_act; ep.ld_resid = H; ep.resid_map = xr;
    ep.gate = modp(2); ep.gate_stride = MS; ep.cu = b->d_cu_q; ep.n_req = b->n_req;
    ep.out0 = y_act; ep.ld0 = H; ep.split = H;
    return launch_gemm(dt, cat, w->w_down, tq, H, H + F, ep, s);
  }
  // a6: queries from active rows only, keys = merged fresh + cached rows (L159)
  if (kv_ready) FPS_CUDA_TRY(stream_wait(s, kv_ready, 0));
  const AttnScratch sc = attn_scratch(ws, H, F, dt, tq, false);
  FPS_TRY(launch_attention(dt, ws.q, kv, ws.ao, w->heads, w->head_dim, b->d_cu_q, b->d_cu_k,
                           b->h_cu_q, b->h_cu_k, b->n_req, tq, b->max_q, b->max_k, s, 0, &sc));
  {  // a7: x1 = x + gate1 (A Wo^T + bo)
    Epilogue ep{};
    ep.bias = w->b_o;
    ep.resid = x_act; ep.ld_resid = H; ep.resid_map = xr;
    ep.gate = modp(2); ep.gate_stride = MS; ep.cu = b->d_cu_q; ep.n_req = b->n_req;
    ep.out0 = ws.x1; ep.ld0 = H; ep.split = H;
    ep.out0_f32 = sdxl;          // SDXL: keep the residual stream x1, x2 in fp32 (R24)
    FPS_TRY(launch_gemm(dt, ws.ao, w->w_o, tq, H, H, ep, s));
  }
  if (sdxl) {
    // SDXL block (reading R24): cross-attention of the active rows to the request's prompt
    // K|V (token-wise in the latent, so rows M only), then the GEGLU feed-forward
    FPS_TRY(launch_ln_affine_f32in((const float*)ws.x1, tq, H, ws.h2, w->ln2_w, w->ln2_b, s));
    {
      Epilogue ep{};
      ep.bias = w->b_q2;
      ep.out0 = ws.q; ep.ld0 = H; ep.split = H;
      FPS_TRY(launch_gemm(dt, ws.h2, w->w_q2, tq, H, H, ep, s));
    }
    int max_c = 0;
    for (int r = 0; r < b->n_req; ++r) max_c = std::max(max_c, b->h_cu_ctx[r + 1] - b->h_cu_ctx[r]);
    FPS_TRY(launch_attention(dt, ws.q, b->d_ctx_kv, ws.ao, w->heads, w->head_dim, b->d_cu_q,
                             b->d_cu_ctx, b->h_cu_q, b->h_cu_ctx, b->n_req, tq, b->max_q, max_c, s,
                             0, &sc));
    {
      Epilogue ep{};
      ep.bias = w->b_o2;
      ep.resid = ws.x1; ep.ld_resid = H; ep.resid_f32 = 1;
      ep.out0 = ws.x2; ep.ld0 = H; ep.split = H; ep.out0_f32 = 1;
      FPS_TRY(launch_gemm(dt, ws.ao, w->w_o2, tq, H, H, ep, s));
    }
    FPS_TRY(launch_ln_affine_f32in((const float*)ws.x2, tq, H, ws.h2, w->ln3_w, w->ln3_b, s));
    {
      Epilogue ep{};
      ep.bias = w->b_up; ep.act = 2;
      ep.out0 = ws.u; ep.ld0 = F; ep.split = 2 * F;
      FPS_TRY(launch_gemm(dt, ws.h2, w->w_up, tq, 2 * F, H, ep, s));
    }
    Epilogue ep{};
    ep.bias = w->b_down;
    ep.resid = ws.x2; ep.ld_resid = H; ep.resid_f32 = 1;
    ep.out0 = y_act; ep.ld0 = H; ep.split = H;
    return launch_gemm(dt, ws.u, w->w_down, tq, H, F, ep, s);
  }
  // a8: y = x1 + gate2 (GELU(LN(x1)(1+scale2)+shift2 W1^T + b1) W2^T + b2)
  FPS_TRY(launch_ln_mod(dt, ws.x1, nullptr, tq, H, ws.h2, b->d_cu_q, b->n_req, b->d_mod, 3 * H, s,
                        nullptr, MS));
  {
    Epilogue ep{};
    ep.bias = w->b_up; ep.act = 1;
    ep.out0 = ws.u; ep.ld0 = F; ep.split = F;
    FPS_TRY(launch_gemm(dt, ws.h2, w->w_up, tq, F, H, ep, s));
  }
  {
    Epilogue ep{};
    ep.bias = w->b_down;
    ep.resid = ws.x1; ep.ld_resid = H;
    ep.gate = modp(5); ep.gate_stride = MS; ep.cu = b->d_cu_q; ep.n_req = b->n_req;
    ep.out0 = y_act; ep.ld0 = H; ep.split = H;
    FPS_TRY(launch_gemm(dt, ws.u, w->w_down, tq, H, F, ep, s));
  }
  return FPS_OK;
}

}  // namespace fps

using namespace fps;

extern "C" {

const char* fps_last_error(void) { return fps::g_err.c_str(); }
int32_t fps_abi_version(void) { return FPS_ABI_VERSION; }

int32_t fps_device_ok(void) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  cudaDeviceProp p;
  if (cudaGetDeviceProperties(&p, dev) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return p.major == 10 && p.minor == 0 ? 1 : 0;
}

int64_t fps_launch_count(void) { return fps::g_launches; }

void fps_profile_enable(int32_t on) {
  fps::prof::g_on = on != 0;
  fps::prof::g_recs.clear();
  fps::prof::g_used = 0;
  fps::prof::g_pending = nullptr;
}

int32_t fps_profile_read(double* ms, double* flops, double* bytes, int64_t* count) {
  using namespace fps::prof;
  for (int k = 0; k < NKIND; ++k) {
    if (ms) ms[k] = 0;
    if (flops) flops[k] = 0;
    if (bytes) bytes[k] = 0;
    if (count) count[k] = 0;
  }
  for (const Rec& r : g_recs) {
    float t = 0.f;
    if (cudaEventSynchronize(r.b) != cudaSuccess || cudaEventElapsedTime(&t, r.a, r.b) != cudaSuccess) {
      cudaGetLastError();
      return FPS_ECUDA;
    }
    if (ms) ms[r.kind] += t;
    if (flops) flops[r.kind] += r.flops;
    if (bytes) bytes[r.kind] += r.bytes;
    if (count) count[r.kind] += 1;
  }
  return NKIND;
}
int64_t fps_profile_trace(double* start_ms, double* end_ms, int32_t* kind, int64_t* stream,
                          int64_t max_n) {
  using namespace fps::prof;
  if (g_recs.empty()) return 0;
  const int64_t n = std::min<int64_t>(max_n, (int64_t)g_recs.size());
  const cudaEvent_t t0 = g_recs[0].a;
  for (int64_t i = 0; i < n; ++i) {
    const Rec& r = g_recs[i];
    float a = 0.f, b = 0.f;
    if (cudaEventSynchronize(r.b) != cudaSuccess || cudaEventElapsedTime(&a, t0, r.a) != cudaSuccess ||
        cudaEventElapsedTime(&b, t0, r.b) != cudaSuccess) {
      cudaGetLastError();
      return FPS_ECUDA;
    }
    if (start_ms) start_ms[i] = a;
    if (end_ms) end_ms[i] = b;
    if (kind) kind[i] = r.kind;
    if (stream) stream[i] = (int64_t)(uintptr_t)r.s;
  }
  return n;
}

void fps_set_disable_tc(int32_t flags) {
  fps::g_disable_tc = flags & 3;
  fps::g_gemm_force = (flags >> 2) & 3;
  fps::g_attn_force = (flags >> 4) & 3;
  fps::g_pdl = (flags & 64) ? 0 : 1;
  fps::g_d2d_kernel = (flags & 128) ? 0 : 1;
  fps::g_attn_split = (flags >> 8) & 7;
  fps::g_gemm_epi4 = (flags >> 11) & 1;
  fps::g_attn_pair = (flags >> 12) & 1;
  fps::g_gemm_bn = (flags >> 13) & 3;
  fps::g_y_grouped = (flags >> 15) & 1 ? 0 : 1;
  fps::g_attn_rot = (flags >> 16) & 1 ? 0 : 1;
}

fps_status fps_build_mask_index(const uint8_t* d_masks, const int32_t* d_offsets, int32_t n_req,
                                int32_t max_len, int32_t* d_masked_ids, int32_t* d_unmasked_ids,
                                int32_t* d_n_masked, void* stream) {
  FPS_CHECK_ARG(n_req >= 0, "n_req < 0");
  if (n_req == 0) return FPS_OK;
  FPS_CHECK_ARG(d_masks && d_offsets && d_masked_ids && d_unmasked_ids && d_n_masked,
                "NULL pointer");
  return launch_mask_index(d_masks, d_offsets, n_req, max_len, d_masked_ids, d_unmasked_ids,
                           d_n_masked, as_stream(stream));
}

fps_status fps_mask_to_tokens(const uint8_t* d_pix, int32_t n_req, int32_t Hp, int32_t Wp,
                              int32_t f, int32_t L_txt, uint8_t* d_tok, void* stream) {
  FPS_CHECK_ARG(n_req >= 0 && Hp >= 0 && Wp >= 0 && L_txt >= 0, "negative size");
  FPS_CHECK_ARG(f > 0 && Hp % f == 0 && Wp % f == 0, "f=%d must divide Hp=%d and Wp=%d", f, Hp, Wp);
  if (n_req == 0 || (Hp * Wp == 0 && L_txt == 0)) return FPS_OK;
  FPS_CHECK_ARG(d_tok && (d_pix || Hp * Wp == 0), "NULL pointer");
  return launch_mask_pool(d_pix, n_req, Hp, Wp, f, L_txt, d_tok, as_stream(stream));
}

static fps_status check_rows(const void* src, const void* dst, int32_t n, int32_t row_bytes) {
  FPS_CHECK_ARG(n >= 0, "n < 0");
  FPS_CHECK_ARG(row_bytes > 0 && row_bytes % 16 == 0, "row_bytes %d not a positive multiple of 16",
                row_bytes);
  if (n == 0) return FPS_OK;
  FPS_CHECK_ARG(src && dst, "NULL pointer");
  FPS_CHECK_ARG(aligned16(src) && aligned16(dst), "pointers must be 16-byte aligned");
  return FPS_OK;
}

fps_status fps_gather_rows(const void* d_src, const int32_t* d_ids, int32_t n, int32_t row_bytes,
                           void* d_dst, void* stream) {
  FPS_TRY(check_rows(d_src, d_dst, n, row_bytes));
  FPS_CHECK_ARG(n == 0 || d_ids, "ids is NULL");
  return launch_copy_rows(d_src, d_ids, nullptr, n, row_bytes, d_dst, as_stream(stream));
}

fps_status fps_scatter_rows(const void* d_src, const int32_t* d_ids, int32_t n, int32_t row_bytes,
                            void* d_dst, void* stream) {
  FPS_TRY(check_rows(d_src, d_dst, n, row_bytes));
  FPS_CHECK_ARG(n == 0 || d_ids, "ids is NULL");
  return launch_copy_rows(d_src, nullptr, d_ids, n, row_bytes, d_dst, as_stream(stream));
}

fps_status fps_copy_rows(const void* d_src, const int32_t* d_src_ids, const int32_t* d_dst_ids,
                         int32_t n, int32_t row_bytes, void* d_dst, void* stream) {
  FPS_TRY(check_rows(d_src, d_dst, n, row_bytes));
  return launch_copy_rows(d_src, d_src_ids, d_dst_ids, n, row_bytes, d_dst, as_stream(stream));
}

size_t fps_block_workspace_bytes(int32_t H, int32_t F, int32_t dtype, int32_t max_q,
                                 int32_t max_u) {
  return ws_layout(H, F, dtype, max_q, max_u, nullptr, nullptr);
}

fps_status fps_masked_block_forward(const fps_block_weights* w, const fps_varlen_batch* b,
                                    const void* d_x_act, void* d_y_act, void* d_kv,
                                    const void* d_xu, void* kv_ready, void* d_ws, size_t ws_bytes,
                                    void* stream) {
  FPS_TRY(check_weights(w));
  FPS_TRY(check_batch(b));
  if (b->total_q > 0) FPS_CHECK_ARG(d_x_act && d_y_act && d_kv && d_ws, "NULL buffer");
  if (b->mode == FPS_MODE_Y && b->total_u > 0) FPS_CHECK_ARG(d_xu && d_kv, "Y-mode needs d_xu");
  if (b->total_q > 0 && b->d_q_row == nullptr)
    FPS_CHECK_ARG(b->total_q == b->total_k, "d_q_row NULL requires total_q == total_k");
  if (b->x_full_rows && b->total_q > 0)
    FPS_CHECK_ARG(b->d_q_row && (w->kind != FPS_BLOCK_DOUBLE || b->d_sm_kvrow),
                  "x_full_rows needs d_q_row (and d_sm_kvrow for double-stream blocks)");
  FPS_CHECK_ARG(w->heads * w->head_dim == w->H, "heads*head_dim != H");
  FPS_TRY(check_ctx(w, b));
  FPS_TRY(check_streams(w, b));
  return block_forward(w, b, d_x_act, d_y_act, d_kv, d_xu, (cudaEvent_t)kv_ready, d_ws, ws_bytes,
                       as_stream(stream));
}

fps_status fps_geglu_pack(int32_t dtype, const void* d_w, const void* d_b, int32_t F, int32_t K,
                          void* d_w_out, void* d_b_out, void* stream) {
  FPS_CHECK_ARG(dtype == FPS_BF16 || dtype == FPS_F32, "dtype %d", dtype);
  FPS_CHECK_ARG(F > 0 && F % 32 == 0 && K > 0 && (K * elt_size(dtype)) % 16 == 0,
                "F=%d must be a positive multiple of 32, K*elt a multiple of 16 (K=%d)", F, K);
  FPS_CHECK_ARG(d_w && d_w_out && (!d_b || d_b_out), "NULL pointer");
  FPS_CHECK_ARG(d_w != d_w_out && (!d_b || d_b != d_b_out), "outputs must not alias inputs");
  FPS_CHECK_ARG(aligned16(d_w) && aligned16(d_w_out), "weights must be 16-byte aligned");
  return launch_geglu_pack(dtype, d_w, d_b, F, K, d_w_out, d_b ? d_b_out : nullptr,
                           as_stream(stream));
}

fps_status fps_context_kv(const fps_block_weights* w, const void* d_ctx, int32_t n_rows,
                          void* d_ctx_kv, void* stream) {
  FPS_TRY(check_weights(w));
  FPS_CHECK_ARG(w->kind == FPS_BLOCK_SDXL, "fps_context_kv: SDXL block weights required");
  FPS_CHECK_ARG(n_rows >= 0, "n_rows < 0");
  if (n_rows == 0) return FPS_OK;
  FPS_CHECK_ARG(d_ctx && d_ctx_kv, "NULL pointer");
  Epilogue ep{};
  ep.bias = w->b_kv2;
  ep.out0 = d_ctx_kv; ep.ld0 = 2 * w->H; ep.split = 2 * w->H;
  return launch_gemm(w->dtype, d_ctx, w->w_kv2, n_rows, 2 * w->H, w->D_ctx, ep, as_stream(stream));
}

fps_status fps_linear(int32_t dtype, const void* d_a, const void* d_w, const void* d_bias,
                      int32_t M, int32_t N, int32_t K, int32_t act, void* d_out, void* stream) {
  FPS_CHECK_ARG(dtype == FPS_BF16 || dtype == FPS_F32, "dtype %d", dtype);
  FPS_CHECK_ARG(M >= 0 && N > 0 && K > 0 && (act == 0 || act == 1), "bad sizes / act");
  FPS_CHECK_ARG(M == 0 || (d_a && d_w && d_out), "NULL pointer");
  FPS_CHECK_ARG(N % 8 == 0, "N %% 8 != 0");
  Epilogue ep{};
  ep.bias = d_bias;
  ep.act = act;
  ep.out0 = d_out;
  ep.ld0 = N;
  ep.split = N;
  return launch_gemm(dtype, d_a, d_w, M, N, K, ep, as_stream(stream));
}

fps_status fps_masked_attention(int32_t dtype, const void* d_q, const void* d_kv, void* d_o,
                                int32_t heads, int32_t head_dim, const int32_t* d_cu_q,
                                const int32_t* d_cu_k, const int32_t* h_cu_q,
                                const int32_t* h_cu_k, int32_t n_req, void* stream) {
  FPS_CHECK_ARG(dtype == FPS_BF16 || dtype == FPS_F32, "dtype %d", dtype);
  FPS_CHECK_ARG(heads > 0 && head_dim > 0 && n_req >= 0, "bad sizes");
  if (n_req == 0) return FPS_OK;
  FPS_CHECK_ARG(d_q && d_kv && d_o && d_cu_q && d_cu_k && h_cu_q && h_cu_k, "NULL pointer");
  const int total_q = h_cu_q[n_req];
  int max_q = 0, max_k = 0;
  for (int r = 0; r < n_req; ++r) {
    max_q = std::max(max_q, h_cu_q[r + 1] - h_cu_q[r]);
    max_k = std::max(max_k, h_cu_k[r + 1] - h_cu_k[r]);
  }
  return launch_attention(dtype, d_q, d_kv, d_o, heads, head_dim, d_cu_q, d_cu_k, h_cu_q, h_cu_k,
                          n_req, total_q, max_q, max_k, as_stream(stream));
}

fps_status fps_dense_block_forward(const fps_block_weights* w, const fps_varlen_batch* b,
                                   const void* d_x, void* d_y, void* d_kv, void* d_ws,
                                   size_t ws_bytes, void* stream) {
  FPS_TRY(check_weights(w));
  FPS_TRY(check_batch(b));
  FPS_CHECK_ARG(b->d_q_row == nullptr && b->total_q == b->total_k,
                "dense block: d_q_row must be NULL and total_q == total_k");
  FPS_TRY(check_ctx(w, b));
  FPS_TRY(check_streams(w, b));
  fps_varlen_batch bb = *b;
  bb.mode = FPS_MODE_KV;
  bb.total_u = 0;
  if (bb.total_q > 0) FPS_CHECK_ARG(d_x && d_y && d_kv && d_ws, "NULL buffer");
  return block_forward(w, &bb, d_x, d_y, d_kv, nullptr, nullptr, d_ws, ws_bytes,
                       as_stream(stream));
}

}  // extern "C"
