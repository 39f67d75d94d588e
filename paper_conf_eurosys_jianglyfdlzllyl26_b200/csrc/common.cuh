// Shared device/host helpers for libflashps (sm_100a). Internal header.
#pragma once

#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <string>
#include <utility>

#include "../../include/flashps.h"

namespace fps {

// ---- error reporting (thread-local last error) ----------------------------------------
void set_error(const char* fmt, ...);
fps_status fail(fps_status code, const char* fmt, ...);

#define FPS_CHECK_ARG(cond, ...)                              \
  do {                                                        \
    if (!(cond)) return ::fps::fail(FPS_EINVAL, __VA_ARGS__); \
  } while (0)

#define FPS_CUDA_TRY(expr)                                                                  \
  do {                                                                                      \
    cudaError_t _e = (expr);                                                                \
    if (_e != cudaSuccess)                                                                  \
      return ::fps::fail(FPS_ECUDA, "%s:%d %s: %s", __FILE__, __LINE__, #expr,              \
                         cudaGetErrorString(_e));                                           \
  } while (0)

// Dynamic shared memory above 48 KB needs cudaFuncSetAttribute once per kernel AND per device:
// each call site keeps a bit per device it has already set up (atomic: engines on different
// devices may launch from different threads).  Wrap a templated kernel name in parentheses.
#define FPS_SMEM_ATTR(kernel, bytes)                                                        \
  do {                                                                                      \
    static std::atomic<unsigned long long> fps_attr_mask_{0};                               \
    int fps_dev_ = 0;                                                                       \
    FPS_CUDA_TRY(cudaGetDevice(&fps_dev_));                                                 \
    const unsigned long long fps_bit_ = 1ull << (fps_dev_ & 63);                            \
    if (!(fps_attr_mask_.load(std::memory_order_acquire) & fps_bit_)) {                     \
      FPS_CUDA_TRY(cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, \
                                        (int)(bytes)));                                     \
      fps_attr_mask_.fetch_or(fps_bit_, std::memory_order_acq_rel);                         \
    }                                                                                       \
  } while (0)

#define FPS_LAUNCH_CHECK()                                                                  \
  do {                                                                                      \
    cudaError_t _e = cudaGetLastError();                                                    \
    if (_e != cudaSuccess)                                                                  \
      return ::fps::fail(FPS_ECUDA, "%s:%d launch: %s", __FILE__, __LINE__,                 \
                         cudaGetErrorString(_e));                                           \
  } while (0)

#define FPS_TRY(expr)                     \
  do {                                    \
    fps_status _s = (expr);               \
    if (_s != FPS_OK) return _s;          \
  } while (0)

inline cudaStream_t as_stream(void* s) { return reinterpret_cast<cudaStream_t>(s); }
inline bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
inline int ceil_div(long a, long b) { return (int)((a + b - 1) / b); }

// ---- programmatic dependent launch ---------------------------------------------------------
// Compute-stream kernels are launched with programmatic stream serialization: the next kernel's
// CTAs start (barrier init, TMEM alloc, descriptor prefetch) as SMs free up at the tail of the
// previous one, and block in pdl_wait() until it has completed and its writes are visible.
// Without the launch attribute both instructions are no-ops.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
extern int g_y_grouped;   // 1 = Y-mode parallel block's two projections in one launch
extern int g_pdl;   // 1 = launch with PDL (default), 0 = plain launches (fps_set_disable_tc bit 6)
// Set by every cross-stream wait / copy the library enqueues: the next kernel is launched
// WITHOUT the PDL attribute, so PDL only ever overlaps two back-to-back library kernels.
// Measured on B200: a PDL launch right after cudaStreamWaitEvent on a load-stream device-to-
// device copy (HBM-tier whole-entry DMA) hung intermittently (3 of 6 C2B bench runs; 0 of 6
// without PDL) -- the early-resident CTAs of a persistent kernel fill every SM while the event's
// producer still needs them.
struct PdlFence {             // streams whose next library kernel must not use PDL
  cudaStream_t s[8];
  int n = 0;
  void add(cudaStream_t st) {
    for (int i = 0; i < n; ++i)
      if (s[i] == st) return;
    if (n < 8) s[n++] = st;
    else s[7] = st;
  }
  bool take(cudaStream_t st) {
    for (int i = 0; i < n; ++i)
      if (s[i] == st) {
        s[i] = s[--n];
        return true;
      }
    return false;
  }
};
extern thread_local PdlFence g_pdl_fence;
inline cudaError_t stream_wait(cudaStream_t s, cudaEvent_t ev, unsigned flags = 0) {
  g_pdl_fence.add(s);
  return cudaStreamWaitEvent(s, ev, flags);
}
inline void pdl_fence(cudaStream_t s) { g_pdl_fence.add(s); }
#define FPS_COPY_TRY(stream, x) \
  do {                          \
    ::fps::pdl_fence(stream);   \
    FPS_CUDA_TRY(x);            \
  } while (0)

template <typename... KArgs, typename... Args>
inline cudaError_t launch_k(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem,
                            cudaStream_t s, Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  const bool fenced = g_pdl_fence.take(s);
  attr[0].val.programmaticStreamSerializationAllowed = (g_pdl && !fenced) ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

// Counts kernels launched through the library (for the bench's gpu_launches claim).
extern thread_local long long g_launches;
inline void count_launch(int n = 1) { g_launches += n; }

constexpr int kNumSMs = 148;
// SMs left to the compute kernels: the pinned-host TMA row gather (cache copy_method 3) keeps
// g_sm_reserved SMs (whole TPCs) for its CTAs while fps_run_batch runs, and the persistent
// compute grids (GEMM, split-KV wave model) are sized to the rest, so neither waits for the other.
extern int g_sm_reserved;
inline int sm_budget() { return kNumSMs - g_sm_reserved; }

// ---- per-kernel-class timing (fps_profile_enable / fps_profile_read) ----------------------
// When enabled, every library launch is bracketed by a pair of CUDA events on its own stream;
// fps_profile_read sums the event durations per class with the algorithmic FLOPs / bytes.
namespace prof {
enum Kind { GEMM = 0, ATTN = 1, LN = 2, ROWS = 3, PREFETCH = 4, EULER = 5, INDEX = 6, NKIND = 7 };
bool enabled();
void begin(cudaStream_t s);
void end(cudaStream_t s, int kind, double flops, double bytes);
}  // namespace prof

// ---- element access ----------------------------------------------------------------------
template <typename T> struct Elt;
template <> struct Elt<float> {
  __device__ __forceinline__ static float load(const float* p) { return *p; }
  __device__ __forceinline__ static void store(float* p, float v) { *p = v; }
  static constexpr int dtype = FPS_F32;
};
template <> struct Elt<__nv_bfloat16> {
  __device__ __forceinline__ static float load(const __nv_bfloat16* p) { return __bfloat162float(*p); }
  __device__ __forceinline__ static void store(__nv_bfloat16* p, float v) { *p = __float2bfloat16_rn(v); }
  static constexpr int dtype = FPS_BF16;
};

__device__ __forceinline__ float to_f(float v) { return v; }
__device__ __forceinline__ float to_f(__nv_bfloat16 v) { return __bfloat162float(v); }
template <typename T> __device__ __forceinline__ T from_f(float v);
template <> __device__ __forceinline__ float from_f<float>(float v) { return v; }
template <> __device__ __forceinline__ __nv_bfloat16 from_f<__nv_bfloat16>(float v) {
  return __float2bfloat16_rn(v);
}

// 16-byte vector <-> floats
template <typename T> struct Vec16;
template <> struct Vec16<float> {
  static constexpr int N = 4;
  __device__ __forceinline__ static void unpack(const uint4& u, float* f) {
    f[0] = __uint_as_float(u.x); f[1] = __uint_as_float(u.y);
    f[2] = __uint_as_float(u.z); f[3] = __uint_as_float(u.w);
  }
  __device__ __forceinline__ static uint4 pack(const float* f) {
    return make_uint4(__float_as_uint(f[0]), __float_as_uint(f[1]), __float_as_uint(f[2]),
                      __float_as_uint(f[3]));
  }
};
__device__ __forceinline__ uint32_t pack_bf16x2(float lo, float hi) {
  __nv_bfloat162 v = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&v);
}
__device__ __forceinline__ void unpack_bf16x2(uint32_t u, float& lo, float& hi) {
  lo = __uint_as_float(u << 16);
  hi = __uint_as_float(u & 0xffff0000u);
}
template <> struct Vec16<__nv_bfloat16> {
  static constexpr int N = 8;
  __device__ __forceinline__ static void unpack(const uint4& u, float* f) {
    unpack_bf16x2(u.x, f[0], f[1]); unpack_bf16x2(u.y, f[2], f[3]);
    unpack_bf16x2(u.z, f[4], f[5]); unpack_bf16x2(u.w, f[6], f[7]);
  }
  __device__ __forceinline__ static uint4 pack(const float* f) {
    return make_uint4(pack_bf16x2(f[0], f[1]), pack_bf16x2(f[2], f[3]), pack_bf16x2(f[4], f[5]),
                      pack_bf16x2(f[6], f[7]));
  }
};

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// Request owning row `i` of a prefix-sum array cu[0..n_req] (largest r with cu[r] <= i).
__device__ __forceinline__ int find_req(const int32_t* __restrict__ cu, int n_req, int i) {
  int lo = 0, hi = n_req - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (__ldg(cu + mid) <= i) lo = mid; else hi = mid - 1;
  }
  return lo;
}

__device__ __forceinline__ float gelu_tanh(float x) {
  const float k0 = 0.7978845608028654f, k1 = 0.044715f;
  float u = k0 * (x + k1 * x * x * x);
  return 0.5f * x * (1.0f + tanhf(u));
}
// bf16-output epilogues: tanh.approx.f32 (MUFU, ~2^-11 relative error, far below the bf16 output
// rounding of 2^-9) instead of the ~20-instruction accurate tanhf, which made the MLP-up GEMM's
// epilogue the slowest part of its last tile.  The fp32 path keeps gelu_tanh (1e-5 parity).
__device__ __forceinline__ float gelu_tanh_fast(float x) {
  const float k0 = 0.7978845608028654f, k1 = 0.044715f;
  const float u = k0 * fmaf(k1 * x, x * x, x);
  float t;
  asm("tanh.approx.f32 %0, %1;" : "=f"(t) : "f"(u));
  return 0.5f * x * (1.0f + t);
}

// ---- GEMM epilogue description (shared by the SIMT and tcgen05 GEMMs) --------------------
// out[r, c] = epilogue(acc[r, c]) with
//   v = acc + bias[c]
//   act == 1: v = GELU_tanh(v)
//   resid: v = resid[r, c] + gate[req(r), c] * v      (gate NULL -> 1)
//   routing: columns [0, split) -> out0 (row r, ld0), columns [split, N) -> out1 with row
//            map1[r] (NULL -> r), column c - split, ld1.  split = N when there is no out1.
// Row-norm output transform: out = LN(x) * (one + scale[req]) + shift[req], the request's vectors
// `stride` elements apart (req from cu over rows); stride 0 = one shared vector (affine LN with
// scale = gamma, shift = beta, one = 0); shift == nullptr = plain LN.
template <typename T>
struct LnMod {
  const T* shift;
  const T* scale;
  int stride;
  float one;
  const int32_t* cu;
  int n_req;
  // two row groups in one launch (double-stream block): rows >= split take their request
  // from cu2 (indexed from split) and their vectors `soff` elements further on
  int split;
  int soff;
  const int32_t* cu2;
  // optional second SOURCE for rows >= split (Y-mode parallel block: rows M from the active
  // input, rows U from the cached input): row split + i reads x2 at rows2[i] (or i)
  const T* x2;
  const int32_t* rows2;
  // optional SECOND OUTPUT (Y-mode sequential / SDXL block: the normalised rows M also land in
  // the all-rows buffer at their token rows, next to the normalised cached rows U): row r < split
  // is also stored at outb[outb_rows1[r]]; with x2, rows >= split are stored ONLY there, at
  // outb[outb_rows2[r - split]]
  T* outb;
  const int32_t* outb_rows1;
  const int32_t* outb_rows2;
};

struct Epilogue {
  const void* bias;          // [N] or null
  int act;                   // 0 none, 1 gelu_tanh, 2 GEGLU over 32-column (value, gate) pairs:
                             //   columns [64j, 64j+32) x GELU_tanh([64j+32, 64j+64)) -> output
                             //   columns [32j, 32j+32) of out0 (tcgen05 path; no resid/gate)
  const void* resid;         // [M, ld_resid] or null
  int ld_resid;
  const void* gate;          // per-request gate vectors: gate + req * gate_stride, or null
  int gate_stride;
  const int32_t* cu;         // request prefix sums over rows (for gate lookup)
  int n_req;
  void* out0; int ld0; const int32_t* map0;   // map0: output row for row r (null -> r)
  void* out1; int ld1; const int32_t* map1;
  int split;
  // optional third column range [split2, N) -> out2 (row r, no remap), and the activation
  // applied only to columns >= act_from (the parallel block's fused QKV|MLP projection)
  void* out2; int ld2; int split2;
  int act_from;
  // fp32 residual stream (SDXL block, tcgen05 path only): out0 and/or resid hold fp32 rows
  int out0_f32, resid_f32;
  // residual row of output row r: resid_map[r] (null -> r)
  const int32_t* resid_map;
};

}  // namespace fps
