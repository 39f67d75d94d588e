// fps_run_batch: step-level continuous batching over a stack of N mask-aware blocks with the
// layer-ahead cache pipeline (§4.2 Fig. 9, L237 §4.3).
//
// One call = admission (mask index of every request, one host sync to size the varlen batch),
// then denoising steps.  Per step:
//   plan     Alg. 1 (planner.cpp) over per-layer costs of this batch (cost model {a,b,c,e});
//   load     stream: for every cached block, in block order, the unmasked rows of each request's
//            entry (template, step_r, block) are copied into a ring of `slots` staging buffers;
//            load j reuses a slot only after the compute stream has consumed load j - slots;
//   compute  stream: cached blocks run fps_masked_block_forward (waiting for their load only
//            right before the first kernel that reads cached rows); uncached blocks run the dense
//            block on all tokens (L211); transitions gather / rebuild rows;
//   replenish: y[M] from the last block, y[U] from the cache (L157); Euler x += delta_s y (R21).
#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include "kernels.h"

namespace fps {
struct Batch {
  int n = 0;                       // requests in the running batch
  std::vector<int> idx;            // index into the caller's reqs[]
  std::vector<int> nq, nu;         // active / unmasked rows per request
  int tq = 0, tu = 0, tk = 0, max_q = 0;
  int32_t *cu_q, *cu_k, *cu_u, *q_row, *u_row, *mod_ids;      // device (inside d_meta)
  int32_t *h_cu_q, *h_cu_k, *h_cu_u;                          // host (inside h_meta)
  // double-stream blocks: [0] masked batch, [1] dense batch (device, inside e->d_sm)
  int ti[2] = {0, 0};
  int32_t *sm_perm[2] = {nullptr, nullptr}, *sm_kvrow[2] = {nullptr, nullptr};
  int32_t *cu_img[2] = {nullptr, nullptr}, *cu_txt[2] = {nullptr, nullptr};
  int32_t* sm_inv[2] = {nullptr, nullptr};
};
}  // namespace fps

struct fps_engine {
  fps_engine_desc d{};
  std::vector<fps_block_weights> layers;
  std::vector<float> deltas;
  std::vector<float> sigmas;          // flow-blend sampler (R29): sigma_0 .. sigma_S
  std::vector<double> layer_comp;     // per-block compute model (a_l, b_l), or empty
  std::vector<uint8_t> fixed_plan;
  int L = 0, elt = 2, W = 0, D = 0;
  size_t row_h = 0, row_w = 0;  // bytes of an H row / a W row
  int maxR = 0;                 // max_batch * L rows
  // device buffers
  char *x_full = nullptr, *full[2] = {nullptr, nullptr}, *y_full = nullptr, *act[2] = {nullptr, nullptr};
  char *kv_scratch = nullptr, *final_slot = nullptr, *ws = nullptr, *mod_batch = nullptr;
  std::vector<char*> slots;
  size_t ws_bytes = 0;
  uint8_t* d_masks = nullptr;
  int32_t *d_off = nullptr, *d_mids = nullptr, *d_uids = nullptr, *d_nm = nullptr;
  int32_t *d_meta = nullptr;   // cu_q | cu_k | cu_u | q_row | u_row | mod_ids
  // SDXL blocks: batch prompt encodings and their per-block cross-attention K|V
  int n_sdxl = 0;
  std::vector<int> sdxl_slot;  // per layer: index into ctx_kv, or -1
  char *ctx_in = nullptr, *ctx_kv = nullptr;
  int32_t *d_cu_ctx = nullptr, *h_cu_ctx = nullptr;
  // double-stream blocks: stream-major order of the masked and the dense batch
  // (perm | kvrow | cu_img | cu_txt, masked then dense)
  bool has_double = false;
  int MW = 0;                   // modulation elements per request and block
  int32_t *d_sm = nullptr, *h_sm = nullptr;
  // cross-step prefetch (R26): loads of the previous step of the same batch, and the event
  // after which the final-Y slot is free again
  bool cross = false;
  int prev_ring = 0;
  cudaEvent_t final_consumed = nullptr;
  // admission reuse: the last admitted batch and the identity of its live requests
  fps::Batch last_B;
  std::vector<const void*> last_key;
  bool last_valid = false;
  float* d_delta = nullptr;
  // pinned host staging
  int32_t* h_meta = nullptr;
  int32_t *h_mids = nullptr, *h_uids = nullptr, *h_nm = nullptr, *h_off = nullptr;
  float* h_delta = nullptr;
  // per-step host staging (modulation row ids, Euler coefficients): a small ring of pinned
  // slots, each reused only after its previous H2D copy has executed -- the host may run
  // several steps ahead of the device, and an async copy reads its pinned source when it runs
  static constexpr int kStageRing = 4;
  int32_t* h_stage = nullptr;
  size_t stage_ints = 0;
  cudaEvent_t stage_ev[kStageRing] = {};
  long long stage_ctr = 0;
  bool no_reuse = false;   // experiments: admit every call
  bool no_transition = false;   // experiments: run a KV-mode plan's last dense block densely
  bool skip_loads = false;      // measurement: no cache loads, slots keep their last contents
  int sm_reserve_call = 0;      // SMs the call keeps for the TMA row gather (method 3)
  bool record = false;          // template run: store the K|V / Y rows of every dense block
  // flow-blend sampler: per-request (template latent, noise) pointers and step coefficients
  void** h_zeps = nullptr;
  void** d_zeps = nullptr;
  float* d_coef = nullptr;
  bool call_start = false; // first step of a fps_run_batch call
  std::vector<cudaEvent_t> ready, consumed;
  cudaEvent_t step_start = nullptr, admit_done = nullptr;
  std::vector<uint8_t> last_plan;
  double last_latency = 0.0;
  long long last_launches = 0;
};

namespace fps {

static void free_engine(fps_engine* e) {
  if (!e) return;
  char* bufs[] = {e->x_full, e->full[0], e->full[1], e->y_full, e->act[0], e->act[1],
                  e->kv_scratch, e->final_slot, e->ws, e->mod_batch};
  for (char* p : bufs) if (p) cudaFree(p);
  for (char* p : e->slots) if (p) cudaFree(p);
  if (e->d_sm) cudaFree(e->d_sm);
  if (e->h_sm) cudaFreeHost(e->h_sm);
  if (e->ctx_in) cudaFree(e->ctx_in);
  if (e->ctx_kv) cudaFree(e->ctx_kv);
  if (e->d_cu_ctx) cudaFree(e->d_cu_ctx);
  if (e->h_cu_ctx) cudaFreeHost(e->h_cu_ctx);
  if (e->d_masks) cudaFree(e->d_masks);
  int32_t* ib[] = {e->d_off, e->d_mids, e->d_uids, e->d_nm, e->d_meta};
  for (int32_t* p : ib) if (p) cudaFree(p);
  if (e->d_delta) cudaFree(e->d_delta);
  if (e->d_coef) cudaFree(e->d_coef);
  if (e->d_zeps) cudaFree(e->d_zeps);
  if (e->h_zeps) cudaFreeHost(e->h_zeps);
  void* hb[] = {e->h_meta, e->h_mids, e->h_uids, e->h_nm, e->h_off, e->h_delta, e->h_stage};
  for (auto ev : e->stage_ev) if (ev) cudaEventDestroy(ev);
  for (void* p : hb) if (p) cudaFreeHost(p);
  for (auto ev : e->ready) if (ev) cudaEventDestroy(ev);
  for (auto ev : e->consumed) if (ev) cudaEventDestroy(ev);
  if (e->step_start) cudaEventDestroy(e->step_start);
  if (e->final_consumed) cudaEventDestroy(e->final_consumed);
  if (e->admit_done) cudaEventDestroy(e->admit_done);
  delete e;
}

// Per-block FLOPs of one request (Table 1, exact per mode; oracle/counters.py restated).
// SDXL blocks (R24) add, per active row, the cross-attention Q / O projections (4 H^2), its
// attention over Lc prompt tokens (4 Lc H) and the GEGLU's doubled up-projection (2 H F).
static double flops_block(int mode, double n, double L, double H, double F, int kind = 0,
                          double Lc = 0) {
  const double attn = 4.0 * n * L * H;
  const double extra = kind == FPS_BLOCK_SDXL ? n * (4.0 * H * H + 4.0 * Lc * H + 2.0 * H * F) : 0.0;
  if (mode == FPS_MODE_KV) return 8.0 * n * H * H + 4.0 * n * H * F + attn + extra;
  return 4.0 * n * H * H + 4.0 * L * H * H + 4.0 * n * H * F + attn + extra;
}

}  // namespace fps

// SMs kept for the cache's TMA row gather; FPS_SM_RESERVE=n overrides (experiments)
static int reserved_sms(const fps_cache* c) {
  using fps::bulk_ctas;
  static const int forced = [] {
    const char* v = getenv("FPS_SM_RESERVE");
    return v ? atoi(v) : -1;
  }();
  const int n = bulk_ctas(c);
  return n > 0 && forced >= 0 ? forced : n;
}

using namespace fps;

extern "C" {

fps_status fps_engine_create(const fps_engine_desc* desc, fps_engine_t* out) {
  FPS_CHECK_ARG(desc && out, "NULL argument");
  const fps_engine_desc& d = *desc;
  FPS_CHECK_ARG(d.H > 0 && d.heads > 0 && d.H % d.heads == 0 && d.F > 0 && d.n_layers > 0,
                "bad dims");
  FPS_CHECK_ARG(d.dtype == FPS_BF16 || d.dtype == FPS_F32, "dtype");
  FPS_CHECK_ARG(d.mode == FPS_MODE_KV || d.mode == FPS_MODE_Y, "mode");
  FPS_CHECK_ARG(d.L_img > 0 && d.L_txt >= 0 && d.max_batch > 0 && d.n_steps > 0, "bad sizes");
  FPS_CHECK_ARG(d.layers && d.h_deltas && d.cache, "layers, h_deltas and cache are required");
  FPS_CHECK_ARG(d.plan_policy >= 0 && d.plan_policy <= 3, "plan_policy");
  FPS_CHECK_ARG(d.sampler == FPS_SAMPLER_EULER || d.sampler == FPS_SAMPLER_FLOW_BLEND, "sampler %d",
                d.sampler);
  FPS_CHECK_ARG(d.sampler != FPS_SAMPLER_FLOW_BLEND || d.h_sigmas, "flow-blend sampler needs h_sigmas");
  FPS_CHECK_ARG(d.plan_policy != 3 || d.h_plan, "plan_policy 3 needs h_plan");
  if (d.plan_policy == 3 && d.mode == FPS_MODE_KV) {
    bool seen = false;
    for (int l = 0; l < d.n_layers; ++l) {
      if (d.h_plan[l]) seen = true;
      else FPS_CHECK_ARG(!seen, "KV-mode plan must be monotone (reading R11)");
    }
  }
  for (int l = 0; l < d.n_layers; ++l) {
    FPS_CHECK_ARG(d.layers[l].H == d.H && d.layers[l].F == d.F && d.layers[l].dtype == d.dtype,
                  "layer %d: H / F / dtype differ from the engine's", l);
    if (d.layers[l].kind == FPS_BLOCK_SDXL)
      FPS_CHECK_ARG(d.L_ctx > 0 && d.layers[l].D_ctx == d.D_ctx,
                    "layer %d: SDXL block needs L_ctx > 0 and D_ctx == the engine's", l);
  }
  bool any_double = false;
  for (int l = 0; l < d.n_layers; ++l) any_double |= d.layers[l].kind == FPS_BLOCK_DOUBLE;
  FPS_CHECK_ARG(!any_double || !d.d_mod_table || d.mod_width == 12 * d.H,
                "double-stream blocks need mod_width = 12H (got %d)", d.mod_width);
  FPS_CHECK_ARG(d.mod_width == 0 || d.mod_width == 6 * d.H || d.mod_width == 12 * d.H,
                "mod_width %d", d.mod_width);
  auto* e = new (std::nothrow) fps_engine();
  if (!e) return fail(FPS_ENOMEM, "engine alloc");
  e->d = d;
  e->layers.assign(d.layers, d.layers + d.n_layers);
  e->deltas.assign(d.h_deltas, d.h_deltas + d.n_steps);
  if (d.sampler == FPS_SAMPLER_FLOW_BLEND) e->sigmas.assign(d.h_sigmas, d.h_sigmas + d.n_steps + 1);
  e->d.h_sigmas = nullptr;
  if (d.h_layer_comp) e->layer_comp.assign(d.h_layer_comp, d.h_layer_comp + 2 * d.n_layers);
  e->d.h_layer_comp = nullptr;
  if (d.plan_policy == 3) e->fixed_plan.assign(d.h_plan, d.h_plan + d.n_layers);
  e->d.layers = nullptr;
  e->d.h_deltas = nullptr;
  e->d.h_plan = nullptr;
  e->sdxl_slot.assign(d.n_layers, -1);
  for (int l = 0; l < d.n_layers; ++l) {
    if (d.layers[l].kind == FPS_BLOCK_SDXL) e->sdxl_slot[l] = e->n_sdxl++;
    if (d.layers[l].kind == FPS_BLOCK_DOUBLE) e->has_double = true;
  }
  e->MW = d.mod_width > 0 ? d.mod_width : 6 * d.H;
  e->L = d.L_img + d.L_txt;
  e->elt = d.dtype == FPS_BF16 ? 2 : 4;
  e->W = d.mode == FPS_MODE_KV ? 2 * d.H : d.H;
  e->row_h = (size_t)d.H * e->elt;
  e->row_w = (size_t)e->W * e->elt;
  e->maxR = d.max_batch * e->L;
  const size_t R = e->maxR;
  size_t slot_bytes = R * e->row_w;
  int D = d.slots > 0 ? d.slots : d.n_layers;
  if (d.slots <= 0) {
    const size_t budget = (size_t)16 << 30;
    D = (int)std::max<size_t>(2, std::min<size_t>(d.n_layers, budget / std::max<size_t>(slot_bytes, 1)));
  }
  e->D = std::min(D, d.n_layers);
  e->cross = d.cross_step != 0 && e->D >= d.n_layers;   // needs one slot per block
  cudaError_t err = cudaSuccess;
  auto dmal = [&](char** p, size_t bytes) {
    if (err == cudaSuccess) err = cudaMalloc((void**)p, std::max<size_t>(bytes, 256));
  };
  dmal(&e->x_full, R * e->row_h);
  dmal(&e->full[0], R * e->row_h);
  dmal(&e->full[1], R * e->row_h);
  dmal(&e->y_full, R * e->row_h);
  dmal(&e->act[0], R * e->row_h);
  dmal(&e->act[1], R * e->row_h);
  dmal(&e->kv_scratch, R * 2 * e->row_h);
  if (d.mode == FPS_MODE_KV) dmal(&e->final_slot, R * e->row_h);
  e->ws_bytes = fps_block_workspace_bytes(d.H, d.F, d.dtype, (int)R, (int)R);
  dmal(&e->ws, e->ws_bytes);
  dmal(&e->mod_batch, (size_t)d.n_layers * d.max_batch * e->MW * e->elt);
  const size_t sm_ints = 2 * (3 * R + 2 * (d.max_batch + 1));
  if (e->has_double) {
    if (err == cudaSuccess) err = cudaMalloc((void**)&e->d_sm, sm_ints * 4);
    if (err == cudaSuccess) err = cudaHostAlloc((void**)&e->h_sm, sm_ints * 4, cudaHostAllocDefault);
  }
  e->slots.assign(e->D, nullptr);
  for (int i = 0; i < e->D; ++i) dmal(&e->slots[i], slot_bytes);
  if (e->n_sdxl) {
    dmal(&e->ctx_in, (size_t)d.max_batch * d.L_ctx * d.D_ctx * e->elt);
    dmal(&e->ctx_kv, (size_t)e->n_sdxl * d.max_batch * d.L_ctx * 2 * e->row_h);
    if (err == cudaSuccess) err = cudaMalloc((void**)&e->d_cu_ctx, (d.max_batch + 1) * 4);
    if (err == cudaSuccess)
      err = cudaHostAlloc((void**)&e->h_cu_ctx, (d.max_batch + 1) * 4, cudaHostAllocDefault);
  }
  if (err == cudaSuccess) err = cudaMalloc((void**)&e->d_masks, R);
  const size_t meta_ints = 3 * (d.max_batch + 1) + 2 * R + (size_t)d.n_layers * d.max_batch;
  auto imal = [&](int32_t** p, size_t n) {
    if (err == cudaSuccess) err = cudaMalloc((void**)p, std::max<size_t>(n, 1) * 4);
  };
  imal(&e->d_off, d.max_batch + 1);
  imal(&e->d_mids, R);
  imal(&e->d_uids, R);
  imal(&e->d_nm, d.max_batch);
  imal(&e->d_meta, meta_ints);
  if (err == cudaSuccess) err = cudaMalloc((void**)&e->d_delta, d.max_batch * 4);
  if (err == cudaSuccess) err = cudaMalloc((void**)&e->d_coef, d.max_batch * 8);
  if (err == cudaSuccess) err = cudaMalloc((void**)&e->d_zeps, std::max(1, 2 * d.max_batch) * sizeof(void*));
  if (err == cudaSuccess)
    err = cudaHostAlloc((void**)&e->h_zeps, std::max(1, 2 * d.max_batch) * sizeof(void*), cudaHostAllocDefault);
  auto hmal = [&](void** p, size_t bytes) {
    if (err == cudaSuccess) err = cudaHostAlloc(p, std::max<size_t>(bytes, 16), cudaHostAllocDefault);
  };
  hmal((void**)&e->h_meta, meta_ints * 4);
  hmal((void**)&e->h_mids, R * 4);
  hmal((void**)&e->h_uids, R * 4);
  hmal((void**)&e->h_nm, d.max_batch * 4);
  hmal((void**)&e->h_off, (d.max_batch + 1) * 4);
  hmal((void**)&e->h_delta, d.max_batch * 4);
  e->stage_ints = (size_t)d.n_layers * d.max_batch + 3 * (size_t)d.max_batch;   // mod ids | delta | coef
  hmal((void**)&e->h_stage, fps_engine::kStageRing * e->stage_ints * 4);
  for (int i = 0; i < fps_engine::kStageRing && err == cudaSuccess; ++i)
    err = cudaEventCreateWithFlags(&e->stage_ev[i], cudaEventDisableTiming);
  e->ready.assign(d.n_layers + 1, nullptr);
  e->consumed.assign(d.n_layers + 1, nullptr);
  for (int i = 0; i <= d.n_layers && err == cudaSuccess; ++i) {
    err = cudaEventCreateWithFlags(&e->ready[i], cudaEventDisableTiming);
    if (err == cudaSuccess) err = cudaEventCreateWithFlags(&e->consumed[i], cudaEventDisableTiming);
  }
  if (err == cudaSuccess) err = cudaEventCreateWithFlags(&e->step_start, cudaEventDisableTiming);
  if (err == cudaSuccess) err = cudaEventCreateWithFlags(&e->final_consumed, cudaEventDisableTiming);
  if (err == cudaSuccess) err = cudaEventCreateWithFlags(&e->admit_done, cudaEventDisableTiming);
  if (err != cudaSuccess) {
    cudaGetLastError();
    free_engine(e);
    return fail(err == cudaErrorMemoryAllocation ? FPS_ENOMEM : FPS_ECUDA, "engine create: %s",
                cudaGetErrorString(err));
  }
  *out = e;
  return FPS_OK;
}

fps_status fps_engine_destroy(fps_engine_t e) {
  free_engine(e);
  return FPS_OK;
}

fps_status fps_engine_last_plan(fps_engine_t e, uint8_t* use_cache, double* latency_ms) {
  FPS_CHECK_ARG(e, "NULL engine");
  if (use_cache)
    for (size_t i = 0; i < e->last_plan.size(); ++i) use_cache[i] = e->last_plan[i];
  if (latency_ms) *latency_ms = e->last_latency;
  return FPS_OK;
}

int64_t fps_engine_last_launches(fps_engine_t e) { return e ? e->last_launches : -1; }

void fps_engine_set_admission_reuse(fps_engine_t e, int32_t on) {
  if (e) e->no_reuse = on == 0;
}

void fps_engine_set_record(fps_engine_t e, int32_t on) {
  if (e) e->record = on != 0;
}

void fps_engine_set_skip_loads(fps_engine_t e, int32_t on) {
  if (e) e->skip_loads = on != 0;
}

void fps_engine_set_kv_transition(fps_engine_t e, int32_t on) {
  if (e && e->no_transition != (on == 0)) {
    e->no_transition = on == 0;
    e->last_valid = false;             // the plan depends on it: re-admit on the next call
  }
}

}  // extern "C"

namespace fps {


static fps_status admit(fps_engine* e, fps_request* reqs, const std::vector<int>& live, Batch& B,
                        cudaStream_t cs) {
  const int L = e->L, n = (int)live.size();
  B.n = n;
  B.idx = live;
  for (int i = 0; i < n; ++i) {
    FPS_COPY_TRY(cs, cudaMemcpyAsync(e->d_masks + (size_t)i * L, reqs[live[i]].d_mask, L,
                                 cudaMemcpyDeviceToDevice, cs));
    e->h_off[i] = i * L;
  }
  e->h_off[n] = n * L;
  FPS_COPY_TRY(cs, cudaMemcpyAsync(e->d_off, e->h_off, (n + 1) * 4, cudaMemcpyHostToDevice, cs));
  if (e->d.sampler == FPS_SAMPLER_FLOW_BLEND) {
    for (int i = 0; i < n; ++i) {
      FPS_CHECK_ARG(reqs[live[i]].d_z && reqs[live[i]].d_noise,
                    "request %d: the flow-blend sampler needs d_z and d_noise", live[i]);
      e->h_zeps[2 * i] = const_cast<void*>(reqs[live[i]].d_z);
      e->h_zeps[2 * i + 1] = const_cast<void*>(reqs[live[i]].d_noise);
    }
    FPS_COPY_TRY(cs, cudaMemcpyAsync(e->d_zeps, e->h_zeps, 2 * n * sizeof(void*),
                                     cudaMemcpyHostToDevice, cs));
  }
  FPS_TRY(launch_mask_index(e->d_masks, e->d_off, n, L, e->d_mids, e->d_uids, e->d_nm, cs));
  FPS_COPY_TRY(cs, cudaMemcpyAsync(e->h_nm, e->d_nm, n * 4, cudaMemcpyDeviceToHost, cs));
  FPS_COPY_TRY(cs, cudaMemcpyAsync(e->h_mids, e->d_mids, (size_t)n * L * 4, cudaMemcpyDeviceToHost, cs));
  FPS_COPY_TRY(cs, cudaMemcpyAsync(e->h_uids, e->d_uids, (size_t)n * L * 4, cudaMemcpyDeviceToHost, cs));
  FPS_CUDA_TRY(cudaEventRecord(e->admit_done, cs));
  FPS_CUDA_TRY(cudaEventSynchronize(e->admit_done));   // the one admission sync
  // host metadata, laid out in h_meta exactly like d_meta
  const int nb = e->d.max_batch;
  int32_t* m = e->h_meta;
  int32_t *cu_q = m, *cu_k = m + (nb + 1), *cu_u = m + 2 * (nb + 1);
  int32_t* q_row = m + 3 * (nb + 1);
  int32_t* u_row = q_row + e->maxR;
  int32_t* mod_ids = u_row + e->maxR;
  B.nq.assign(n, 0);
  B.nu.assign(n, 0);
  cu_q[0] = cu_k[0] = cu_u[0] = 0;
  B.max_q = 0;
  for (int i = 0; i < n; ++i) {
    const int nq = e->h_nm[i], nu = L - nq;
    B.nq[i] = nq;
    B.nu[i] = nu;
    for (int j = 0; j < nq; ++j) q_row[cu_q[i] + j] = i * L + e->h_mids[i * L + j];
    for (int j = 0; j < nu; ++j) u_row[cu_u[i] + j] = i * L + e->h_uids[i * L + j];
    cu_q[i + 1] = cu_q[i] + nq;
    cu_k[i + 1] = cu_k[i] + L;
    cu_u[i + 1] = cu_u[i] + nu;
    B.max_q = std::max(B.max_q, nq);
  }
  B.tq = cu_q[n];
  B.tk = cu_k[n];
  B.tu = cu_u[n];
  (void)mod_ids;
  FPS_COPY_TRY(cs, cudaMemcpyAsync(e->d_meta, e->h_meta,
                               (size_t)(3 * (nb + 1) + 2 * e->maxR) * 4, cudaMemcpyHostToDevice, cs));
  int32_t* dm = e->d_meta;
  B.cu_q = dm;
  B.cu_k = dm + (nb + 1);
  B.cu_u = dm + 2 * (nb + 1);
  B.q_row = dm + 3 * (nb + 1);
  B.u_row = B.q_row + e->maxR;
  B.mod_ids = B.u_row + e->maxR;
  B.h_cu_q = cu_q;
  B.h_cu_k = cu_k;
  B.h_cu_u = cu_u;
  if (e->has_double) {
    // stream-major order (all image rows, then all text rows) of the masked and dense batches
    const int R = e->maxR, nb1 = e->d.max_batch + 1, Li = e->d.L_img;
    const size_t per = 3 * (size_t)R + 2 * nb1;
    for (int v = 0; v < 2; ++v) {
      int32_t* base = e->h_sm + (size_t)v * per;
      int32_t *perm = base, *kvr = base + R, *ci = base + 2 * R, *ct = ci + nb1;
      int32_t* inv = ct + nb1;
      int k = 0;
      ci[0] = ct[0] = 0;
      for (int i = 0; i < n; ++i) {          // image rows
        const int cnt = v == 0 ? B.nq[i] : L;
        int ni = 0;
        for (int j = 0; j < cnt; ++j) {
          const int tok = v == 0 ? e->h_mids[i * L + j] : j;
          if (tok >= Li) break;                // ascending ids: text rows come last
          perm[k] = v == 0 ? cu_q[i] + j : i * L + j;
          kvr[k] = v == 0 ? q_row[cu_q[i] + j] : i * L + j;
          ++k, ++ni;
        }
        ci[i + 1] = ci[i] + ni;
      }
      B.ti[v] = k;
      for (int i = 0; i < n; ++i) {          // text rows
        const int cnt = v == 0 ? B.nq[i] : L;
        const int first = ci[i + 1] - ci[i];
        for (int j = first; j < cnt; ++j) {
          perm[k] = v == 0 ? cu_q[i] + j : i * L + j;
          kvr[k] = v == 0 ? q_row[cu_q[i] + j] : i * L + j;
          ++k;
        }
        ct[i + 1] = ct[i] + (cnt - first);
      }
      for (int j = 0; j < k; ++j) inv[perm[j]] = j;
      int32_t* dbase = e->d_sm + (size_t)v * per;
      B.sm_perm[v] = dbase;
      B.sm_kvrow[v] = dbase + R;
      B.cu_img[v] = dbase + 2 * R;
      B.cu_txt[v] = dbase + 2 * R + nb1;
      B.sm_inv[v] = dbase + 2 * R + 2 * nb1;
    }
    FPS_COPY_TRY(cs, cudaMemcpyAsync(e->d_sm, e->h_sm, 2 * per * 4, cudaMemcpyHostToDevice, cs));
  }
  if (e->n_sdxl) {
    // SDXL blocks: the prompt is fixed over the steps, so each block's cross-attention K|V
    // is projected once per admission (one GEMM per SDXL block over the batch's prompts)
    const int Lc = e->d.L_ctx;
    const size_t ctx_row = (size_t)e->d.D_ctx * e->elt;
    for (int i = 0; i < n; ++i) {
      FPS_CHECK_ARG(reqs[live[i]].d_ctx, "request %d: SDXL blocks need d_ctx", live[i]);
      FPS_COPY_TRY(cs, cudaMemcpyAsync(e->ctx_in + (size_t)i * Lc * ctx_row, reqs[live[i]].d_ctx,
                                       Lc * ctx_row, cudaMemcpyDeviceToDevice, cs));
    }
    for (int i = 0; i <= n; ++i) e->h_cu_ctx[i] = i * Lc;
    FPS_COPY_TRY(cs, cudaMemcpyAsync(e->d_cu_ctx, e->h_cu_ctx, (n + 1) * 4, cudaMemcpyHostToDevice, cs));
    for (int l = 0; l < e->d.n_layers; ++l)
      if (e->sdxl_slot[l] >= 0)
        FPS_TRY(fps_context_kv(&e->layers[l], e->ctx_in, n * Lc,
                               e->ctx_kv + (size_t)e->sdxl_slot[l] * e->d.max_batch * Lc * 2 * e->row_h,
                               cs));
  }
  return FPS_OK;
}

static void make_plan(fps_engine* e, const Batch& B) {
  const int N = e->d.n_layers;
  e->last_plan.assign(N, 0);
  const double a = e->d.cost_model[0] > 0 ? e->d.cost_model[0] : 1.0 / 1.0e12;  // ms per FLOP
  const double b = e->d.cost_model[1] > 0 ? e->d.cost_model[1] : 0.01;
  const double c = e->d.cost_model[2] > 0 ? e->d.cost_model[2] : 1.0 / 5.0e7;   // ms per byte
  const double ec = e->d.cost_model[3] > 0 ? e->d.cost_model[3] : 0.01;
  double by = 0, byf = 0;
  const double H = e->d.H, F = e->d.F, L = e->L, Lc = e->d.L_ctx;
  std::vector<double> Cw(N), Cwo(N), Ct(N), Lm(N);
  for (int l = 0; l < N; ++l) {
    const int kind = e->layers[l].kind;
    double fm = 0, fd = 0, ft = 0;
    for (int i = 0; i < B.n; ++i) {
      fm += flops_block(e->d.mode, B.nq[i], L, H, F, kind, Lc);
      fd += flops_block(FPS_MODE_KV, L, L, H, F, kind, Lc);
      ft += flops_block(FPS_MODE_Y, B.nq[i], L, H, F, kind, Lc);
    }
    // the block's own compute model (fitted per block kind) when given, else the stack's
    const double al = e->layer_comp.empty() ? a : e->layer_comp[2 * l];
    const double bl = e->layer_comp.empty() ? b : e->layer_comp[2 * l + 1];
    Cw[l] = al * fm + bl;
    Cwo[l] = al * fd + bl;
    Ct[l] = al * ft + bl;   // transition block (R28): Y-mode work over the fresh full input
  }
  for (int i = 0; i < B.n; ++i) {
    // rows the load moves: U, or the whole entry for the whole-entry DMA method
    const double rows = (B.nu[i] > 0 && cache_writes_all_rows(e->d.cache)) ? e->d.L_img : B.nu[i];
    by += rows * e->row_w;
    byf += rows * e->row_h;
  }
  for (int l = 0; l < N; ++l) Lm[l] = by > 0 ? c * by + ec : 0.0;
  const double fin = byf > 0 ? c * byf + ec : 0.0;
  const bool trans = e->d.mode == FPS_MODE_KV && !e->no_transition;
  auto latency = e->cross ? fps_pipeline_latency_cross : fps_pipeline_latency;
  // KV-mode plans are the N+1 suffixes; with the transition block (R28) the prefix's last block
  // costs Ct instead of Cwo, so each suffix is priced with its own cost vector.
  auto priced = [&](const uint8_t* use) {
    int k = 0;
    while (k < N && !use[k]) ++k;
    if (!trans || k == 0 || k == N) return latency(use, Cw.data(), Cwo.data(), Lm.data(), N,
                                                   e->d.mode, fin);
    std::vector<double> C2(Cwo);
    C2[k - 1] = Ct[k - 1];
    return latency(use, Cw.data(), C2.data(), Lm.data(), N, e->d.mode, fin);
  };
  if (e->d.plan_policy == 0 && trans) {
    fps_plan_pipeline_kv_transition(Cw.data(), Cwo.data(), Ct.data(), Lm.data(), N, fin,
                                    e->cross ? 1 : 0, e->last_plan.data(), &e->last_latency);
  } else if (e->d.plan_policy == 0) {
    if (e->cross)
      fps_plan_pipeline_cross(Cw.data(), Cwo.data(), Lm.data(), N, e->d.mode, fin,
                              e->last_plan.data(), &e->last_latency);
    else
      fps_plan_pipeline(Cw.data(), Cwo.data(), Lm.data(), N, e->d.mode, fin, e->last_plan.data(),
                        &e->last_latency);
  } else {
    for (int l = 0; l < N; ++l)
      e->last_plan[l] = e->d.plan_policy == 1 ? 1 : e->d.plan_policy == 2 ? 0 : e->fixed_plan[l];
    e->last_latency = priced(e->last_plan.data());
  }
}

// One denoising step of the running batch.
static fps_status run_step(fps_engine* e, fps_request* reqs, Batch& B, cudaStream_t cs,
                           cudaStream_t ls) {
  const int N = e->d.n_layers, n = B.n, H = e->d.H;
  const bool kv = e->d.mode == FPS_MODE_KV;
  const std::vector<uint8_t>& use = e->last_plan;
  // adaLN vectors of every block for every request at its own step (rows of the table)
  const int slot = (int)(e->stage_ctr++ % fps_engine::kStageRing);
  FPS_CUDA_TRY(cudaEventSynchronize(e->stage_ev[slot]));   // its last copy has run
  int32_t* mod_ids = e->h_stage + (size_t)slot * e->stage_ints;
  float* h_delta = reinterpret_cast<float*>(mod_ids + (size_t)N * e->d.max_batch);
  if (e->d.d_mod_table) {
    for (int l = 0; l < N; ++l)
      for (int i = 0; i < n; ++i) mod_ids[l * n + i] = l * e->d.n_steps + reqs[B.idx[i]].step;
    FPS_COPY_TRY(cs, cudaMemcpyAsync(B.mod_ids, mod_ids, (size_t)N * n * 4, cudaMemcpyHostToDevice, cs));
    FPS_TRY(launch_copy_rows(e->d.d_mod_table, B.mod_ids, nullptr, N * n, e->MW * e->elt,
                             e->mod_batch, cs));
  }
  for (int i = 0; i < n; ++i) h_delta[i] = e->deltas[reqs[B.idx[i]].step];
  FPS_COPY_TRY(cs, cudaMemcpyAsync(e->d_delta, h_delta, n * 4, cudaMemcpyHostToDevice, cs));
  if (e->d.sampler == FPS_SAMPLER_FLOW_BLEND) {
    float* h_coef = h_delta + e->d.max_batch;
    for (int i = 0; i < n; ++i) {
      const int st = reqs[B.idx[i]].step;
      h_coef[2 * i] = e->sigmas[st + 1] - e->sigmas[st];
      h_coef[2 * i + 1] = e->sigmas[st + 1];
    }
    FPS_COPY_TRY(cs, cudaMemcpyAsync(e->d_coef, h_coef, n * 8, cudaMemcpyHostToDevice, cs));
  }
  FPS_CUDA_TRY(cudaEventRecord(e->stage_ev[slot], cs));

  // ---- load schedule: ring loads (cached blocks in order) + KV-mode final Y load ----------
  std::vector<int> loads;                  // block of each ring load
  std::vector<int> pos(N, -1);
  for (int l = 0; l < N; ++l)
    if (use[l]) {
      pos[l] = (int)loads.size();
      loads.push_back(l);
    }
  const int n_ring = (int)loads.size();
  const bool final_load = kv && n_ring > 0;
  // the gather's SMs are kept only in steps that load: a plan without cached blocks (the dense
  // reference) and the no-load arm compute on every SM, so the reservation's compute cost
  // counts as load cost in the exposed-load measurement
  g_sm_reserved = (n_ring > 0 && !e->skip_loads) ? e->sm_reserve_call : 0;
  std::vector<char> consumed_rec(n_ring + 1, 0);
  int issued = 0;
  bool final_issued = false;
  std::vector<fps_prefetch_item> items(n);
  FPS_CUDA_TRY(cudaEventRecord(e->step_start, cs));
  // per-step pipeline: this step's loads start with the step; cross-step prefetch (R26): a
  // load waits only for the previous step's consumer of its slot (below)
  // (the first step of a call also waits: the caller's stream work before the call -- e.g. the
  // host-to-device copy of the latents -- must not queue behind this step's cache loads)
  if (!e->cross || e->call_start) FPS_CUDA_TRY(stream_wait(ls, e->step_start, 0));
  e->call_start = false;
  auto issue = [&](int block, char* dst, size_t row_bytes, cudaEvent_t ev) -> fps_status {
    for (int i = 0; i < n; ++i) {
      const fps_request& r = reqs[B.idx[i]];
      fps_prefetch_item& it = items[i];
      it.template_id = r.template_id;
      it.step = r.step;
      it.layer = block;
      it.n_rows = B.nu[i];
      it.d_rows = e->d_uids + (size_t)i * e->L;
      it.h_rows = e->h_uids + (size_t)i * e->L;
      it.d_dst = dst + (size_t)B.h_cu_k[i] * row_bytes;
      it.dst_row_bytes = (int)row_bytes;
    }
    if (e->skip_loads) {   // the no-load arm: only the ordering events, no bytes moved
      FPS_CUDA_TRY(cudaEventRecord(ev, ls));
      return FPS_OK;
    }
    return fps_cache_prefetch(e->d.cache, items.data(), n, ls, ev);
  };
  auto try_issue = [&]() -> fps_status {
    while (issued < n_ring && (issued < e->D || consumed_rec[issued - e->D])) {
      if (issued >= e->D) FPS_CUDA_TRY(stream_wait(ls, e->consumed[issued - e->D], 0));
      // the previous step's consumer of this slot (recorded before this step re-records it)
      if (e->cross && issued < e->prev_ring) FPS_CUDA_TRY(stream_wait(ls, e->consumed[issued], 0));
      FPS_TRY(issue(loads[issued], e->slots[issued % e->D], e->row_w, e->ready[issued]));
      ++issued;
    }
    if (final_load && issued == n_ring && !final_issued) {
      if (e->cross && e->prev_ring > 0) FPS_CUDA_TRY(stream_wait(ls, e->final_consumed, 0));
      FPS_TRY(issue(N, e->final_slot, e->row_h, e->ready[n_ring]));
      final_issued = true;
    }
    return FPS_OK;
  };
  auto consume = [&](int j) -> fps_status {
    FPS_CUDA_TRY(cudaEventRecord(e->consumed[j], cs));
    consumed_rec[j] = 1;
    return FPS_OK;
  };
  FPS_TRY(try_issue());

  // ---- compute ------------------------------------------------------------------------
  fps_varlen_batch vb{};
  vb.n_req = n;
  vb.total_q = B.tq;
  vb.total_k = B.tk;
  vb.max_q = B.max_q;
  vb.max_k = e->L;
  vb.d_cu_q = B.cu_q;
  vb.d_cu_k = B.cu_k;
  vb.h_cu_q = B.h_cu_q;
  vb.h_cu_k = B.h_cu_k;
  vb.d_q_row = B.q_row;
  vb.mode = e->d.mode;
  vb.total_u = B.tu;
  vb.d_cu_u = B.cu_u;
  vb.d_u_src = B.u_row;
  vb.d_u_row = B.u_row;
  vb.mod_stride = e->MW;
  vb.total_q_img = B.ti[0];
  vb.d_sm_perm = B.sm_perm[0];
  vb.d_sm_kvrow = B.sm_kvrow[0];
  vb.d_cu_img = B.cu_img[0];
  vb.d_cu_txt = B.cu_txt[0];
  vb.d_sm_inv = B.sm_inv[0];
  fps_varlen_batch vd = vb;             // dense: every row of every request is active
  vd.total_q_img = B.ti[1];
  vd.d_sm_perm = B.sm_perm[1];
  vd.d_sm_kvrow = B.sm_kvrow[1];
  vd.d_cu_img = B.cu_img[1];
  vd.d_cu_txt = B.cu_txt[1];
  vd.d_sm_inv = B.sm_inv[1];
  vd.total_q = B.tk;
  vd.max_q = e->L;
  vd.d_cu_q = B.cu_k;
  vd.h_cu_q = B.h_cu_k;
  vd.d_q_row = nullptr;
  vd.mode = FPS_MODE_KV;
  vd.total_u = 0;

  const char* cur_full = e->x_full;     // valid full-row activations when rep == FULL
  int full_toggle = 0, act_cur = 0;
  bool rep_full = true;
  for (int l = 0; l < N; ++l) {
    const fps_block_weights* w = &e->layers[l];
    const void* mod = e->d.d_mod_table ? e->mod_batch + (size_t)l * n * e->MW * e->elt : nullptr;
    vb.d_mod = mod;
    vd.d_mod = mod;
    if (e->sdxl_slot[l] >= 0) {
      vb.d_ctx_kv = e->ctx_kv +
                    (size_t)e->sdxl_slot[l] * e->d.max_batch * e->d.L_ctx * 2 * e->row_h;
      vb.d_cu_ctx = e->d_cu_ctx;
      vb.h_cu_ctx = e->h_cu_ctx;
    } else {
      vb.d_ctx_kv = nullptr;
      vb.d_cu_ctx = vb.h_cu_ctx = nullptr;
    }
    vd.d_ctx_kv = vb.d_ctx_kv;
    vd.d_cu_ctx = vb.d_cu_ctx;
    vd.h_cu_ctx = vb.h_cu_ctx;
    if (!use[l] && kv && rep_full && !e->no_transition && l + 1 < N && use[l + 1]) {
      // KV-mode transition block (reading R28): the last uncached block before the cached
      // suffix.  Block l+1 reads only its masked rows' input (its unmasked K|V come from the
      // cache), so block l's unmasked output rows are dead: run it as a masked block over the
      // fresh full input -- K|V of all rows from cur_full (the Y-mode path with d_xu = the
      // full input), Q / attention / O / MLP on the active rows only.  Same values for every
      // row that is read afterwards; nothing loaded for it.
      // (its active rows are read straight from the full input: a2 fused into the block)
      fps_varlen_batch vt = vb;
      vt.mode = FPS_MODE_Y;
      vt.x_full_rows = 1;
      FPS_TRY(fps_masked_block_forward(w, &vt, cur_full, e->act[act_cur ^ 1], e->kv_scratch,
                                       cur_full, nullptr, e->ws, e->ws_bytes, cs));
      act_cur ^= 1;
      rep_full = false;
    } else if (!use[l]) {
      if (!rep_full) {
        // Y-mode cached -> uncached: rebuild the full input from act rows M and the cached
        // output rows U of block l-1 (reading R11)
        char* dst = e->full[full_toggle];
        FPS_TRY(launch_copy_rows(e->act[act_cur], nullptr, B.q_row, B.tq, (int)e->row_h, dst, cs));
        FPS_CUDA_TRY(stream_wait(cs, e->ready[pos[l - 1]], 0));
        FPS_TRY(launch_copy_rows(e->slots[pos[l - 1] % e->D], B.u_row, B.u_row, B.tu,
                                 (int)e->row_h, dst, cs));
        FPS_TRY(consume(pos[l - 1]));
        cur_full = dst;
        full_toggle ^= 1;
      }
      char* dst = e->full[full_toggle];
      FPS_TRY(fps_dense_block_forward(w, &vd, cur_full, dst, e->kv_scratch, e->ws, e->ws_bytes, cs));
      if (e->record)     // template run (L130, L203): this block's cache entry of every request
        for (int i = 0; i < n; ++i) {
          const fps_request& r = reqs[B.idx[i]];
          const char* src = kv ? e->kv_scratch + (size_t)B.h_cu_k[i] * 2 * e->row_h
                               : dst + (size_t)B.h_cu_k[i] * e->row_h;
          FPS_TRY(fps_cache_store(e->d.cache, r.template_id, r.step, l, src,
                                  (int)(kv ? 2 * e->row_h : e->row_h), cs));
        }
      cur_full = dst;
      full_toggle ^= 1;
      rep_full = true;
    } else {
      const char* x_in;
      const char* xu = nullptr;
      cudaEvent_t ev = nullptr;
      int consumed_after = -1;
      fps_varlen_batch vx = vb;
      x_in = e->act[act_cur];
      if (rep_full) {
        // a2 fused into the block: the first cached block reads its active rows straight out
        // of the full activations (first norm and residual at d_q_row), no gathered copy
        x_in = cur_full;
        vx.x_full_rows = 1;
        xu = cur_full;
      } else if (!kv) {
        xu = e->slots[pos[l - 1] % e->D];
        ev = e->ready[pos[l - 1]];
        consumed_after = pos[l - 1];
      }
      char* kvbuf;
      if (kv) {
        kvbuf = e->slots[pos[l] % e->D];
        ev = e->ready[pos[l]];
        consumed_after = pos[l];
        if (cache_writes_all_rows(e->d.cache)) {
          // whole-entry DMA also lands on the masked rows: the QKV epilogue's fresh K/V must
          // come after it (the load was issued layers ahead, so this rarely waits)
          FPS_CUDA_TRY(stream_wait(cs, ev, 0));
          ev = nullptr;
        }
      } else {
        kvbuf = e->kv_scratch;
      }
      FPS_TRY(fps_masked_block_forward(w, &vx, x_in, e->act[act_cur ^ 1], kvbuf, kv ? nullptr : xu,
                                       ev, e->ws, e->ws_bytes, cs));
      if (consumed_after >= 0) FPS_TRY(consume(consumed_after));
      act_cur ^= 1;
      rep_full = false;
    }
    FPS_TRY(try_issue());
  }

  // ---- replenish (a9) + sampler update ---------------------------------------------------
  const char* y_src;
  if (rep_full) {
    y_src = cur_full;
  } else {
    FPS_TRY(launch_copy_rows(e->act[act_cur], nullptr, B.q_row, B.tq, (int)e->row_h, e->y_full, cs));
    const int j = kv ? n_ring : pos[N - 1];
    const char* src = kv ? e->final_slot : e->slots[pos[N - 1] % e->D];
    FPS_CUDA_TRY(stream_wait(cs, e->ready[j], 0));
    FPS_TRY(launch_copy_rows(src, B.u_row, B.u_row, B.tu, (int)e->row_h, e->y_full, cs));
    if (kv) FPS_CUDA_TRY(cudaEventRecord(e->final_consumed, cs));
    else FPS_TRY(consume(j));          // Y-mode: block N-1's slot is read by the replenish
    y_src = e->y_full;
  }
  if (e->record && kv && rep_full)   // KV-mode replenish entry: the final block's Y rows
    for (int i = 0; i < n; ++i) {
      const fps_request& r = reqs[B.idx[i]];
      FPS_TRY(fps_cache_store(e->d.cache, r.template_id, r.step, N,
                              y_src + (size_t)B.h_cu_k[i] * e->row_h, (int)e->row_h, cs));
    }
  if (e->d.sampler == FPS_SAMPLER_FLOW_BLEND)
    FPS_TRY(launch_flow_blend(e->d.dtype, e->x_full, y_src, n, e->L, e->d.L_img, H, e->d_masks,
                              reinterpret_cast<const float2*>(e->d_coef), e->d_zeps, cs));
  else
    FPS_TRY(launch_euler(e->d.dtype, e->x_full, y_src, B.tk, H, B.cu_k, n, e->d_delta, cs));
  e->prev_ring = n_ring;
  if (!e->cross) {
    // the load stream must not run ahead into the next step's slots before this step is done
    FPS_CUDA_TRY(cudaEventRecord(e->step_start, cs));
    FPS_CUDA_TRY(stream_wait(ls, e->step_start, 0));
  }
  return FPS_OK;
}

}  // namespace fps

extern "C" fps_status fps_run_batch(fps_engine_t e, fps_request* reqs, int32_t n_req,
                                    int32_t n_steps, void* compute_stream, void* load_stream) {
  FPS_CHECK_ARG(e, "NULL engine");
  FPS_CHECK_ARG(n_req >= 0 && n_req <= e->d.max_batch, "n_req %d > max_batch %d", n_req,
                e->d.max_batch);
  FPS_CHECK_ARG(n_req == 0 || reqs, "NULL reqs");
  FPS_CHECK_ARG(n_steps >= 0, "n_steps < 0");
  for (int i = 0; i < n_req; ++i) {
    FPS_CHECK_ARG(reqs[i].d_mask && reqs[i].d_x, "request %d: NULL mask or latent", i);
    FPS_CHECK_ARG(reqs[i].n_steps <= e->d.n_steps && reqs[i].step >= 0, "request %d: steps", i);
  }
  cudaStream_t cs = as_stream(compute_stream);
  cudaStream_t ls = load_stream ? as_stream(load_stream) : cs;
  const long long launches0 = g_launches;
  // the TMA row gather (copy_method 3) keeps its SMs for the whole call: size the compute grids
  // to the rest (restored on every return path)
  struct SmReserve {
    int prev;
    explicit SmReserve(int n) : prev(g_sm_reserved) { g_sm_reserved = n; }
    ~SmReserve() { g_sm_reserved = prev; }
  } reserve(load_stream ? reserved_sms(e->d.cache) : 0);
  e->sm_reserve_call = g_sm_reserved;
  e->call_start = true;
  int done_steps = 0;
  while (done_steps < n_steps) {
    std::vector<int> live;
    for (int i = 0; i < n_req; ++i) {
      reqs[i].status = reqs[i].step >= reqs[i].n_steps ? 1 : 0;
      if (!reqs[i].status) live.push_back(i);
    }
    if (live.empty()) break;
    // the same live requests as the last admitted batch (same order, buffers and template):
    // reuse its admission -- mask index, batch metadata, prompt K|V, plan -- without the host
    // synchronisation (callers stepping one step per call, e.g. a serving loop, pay it once)
    std::vector<const void*> key;
    for (int i : live)
      key.insert(key.end(), {reqs[i].d_mask, reqs[i].d_x, reqs[i].d_ctx, reqs[i].d_z,
                             reqs[i].d_noise,
                             reinterpret_cast<const void*>((uintptr_t)reqs[i].template_id)});
    const bool reuse = e->last_valid && !e->no_reuse && key == e->last_key;
    Batch& B = e->last_B;
    B.idx = live;           // same requests, possibly at other positions of the caller's array
    if (!reuse) {
      e->last_valid = false;
      B = Batch{};
      // a new batch: its index arrays and slots are rewritten, so the load stream drains first
      FPS_CUDA_TRY(cudaEventRecord(e->final_consumed, ls));
      FPS_CUDA_TRY(stream_wait(cs, e->final_consumed, 0));
      e->prev_ring = 0;
      FPS_TRY(admit(e, reqs, live, B, cs));
      make_plan(e, B);
      e->last_key = key;
      e->last_valid = true;
    }
    // load each request's latent into the contiguous batch buffer
    for (int i = 0; i < B.n; ++i)
      FPS_COPY_TRY(cs, cudaMemcpyAsync(e->x_full + (size_t)i * e->L * e->row_h, reqs[live[i]].d_x,
                                   (size_t)e->L * e->row_h, cudaMemcpyDeviceToDevice, cs));
    bool changed = false;
    while (done_steps < n_steps && !changed) {
      FPS_TRY(run_step(e, reqs, B, cs, ls));
      ++done_steps;
      for (int i = 0; i < B.n; ++i) {
        fps_request& r = reqs[live[i]];
        r.step += 1;
        if (r.step >= r.n_steps) {
          r.status = 1;
          changed = true;   // leaves at this step boundary (L237); the batch is rebuilt
          e->last_valid = false;
        }
      }
    }
    for (int i = 0; i < B.n; ++i)
      FPS_COPY_TRY(cs, cudaMemcpyAsync(reqs[live[i]].d_x, e->x_full + (size_t)i * e->L * e->row_h,
                                   (size_t)e->L * e->row_h, cudaMemcpyDeviceToDevice, cs));
  }
  for (int i = 0; i < n_req; ++i) reqs[i].status = reqs[i].step >= reqs[i].n_steps ? 1 : 0;
  // make sure the load stream has drained before the caller reuses buffers
  FPS_CUDA_TRY(cudaEventRecord(e->step_start, ls));
  FPS_CUDA_TRY(stream_wait(cs, e->step_start, 0));
  e->last_launches = g_launches - launches0;
  return FPS_OK;
}
