// a1 mask index, a2/a9/a3 row movement, a4 row-norm + modulation, sampler update.
// PAPER.md L130 (token categorisation), L157 (extract / replenish rows), L134 (token-wise LN).
#include <algorithm>

#include "kernels.h"

namespace fps {

// ---------------------------------------------------------------------------------------
// a1: one CTA (1024 threads) per request; per 1024-token chunk a warp ballot gives each
// token its rank inside the warp, a warp-0 scan over the 32 warp counts gives the rank
// inside the chunk, and a running total carries it across chunks. Stable (ascending ids).
__global__ void __launch_bounds__(1024) mask_index_kernel(const uint8_t* __restrict__ masks,
                                                          const int32_t* __restrict__ off,
                                                          int32_t* __restrict__ mids,
                                                          int32_t* __restrict__ uids,
                                                          int32_t* __restrict__ nm) {
  __shared__ int warp_off[32];
  __shared__ int chunk_total;
  const int r = blockIdx.x;
  const int beg = off[r], L = off[r + 1] - beg;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nwarps = blockDim.x >> 5;
  const unsigned lt_mask = (1u << lane) - 1u;
  int running = 0;
  for (int chunk = 0; chunk < L; chunk += blockDim.x) {
    const int t = chunk + threadIdx.x;
    const bool valid = t < L;
    const bool act = valid && masks[beg + t] != 0;
    const unsigned bal = __ballot_sync(0xffffffffu, act);
    const int rank_in_warp = __popc(bal & lt_mask);
    if (lane == 0) warp_off[warp] = __popc(bal);
    __syncthreads();
    if (warp == 0) {
      int v = lane < nwarps ? warp_off[lane] : 0;
      int incl = v;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int u = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += u;
      }
      if (lane < nwarps) warp_off[lane] = incl - v;
      if (lane == 31) chunk_total = incl;
    }
    __syncthreads();
    const int before = running + warp_off[warp] + rank_in_warp;   // active tokens with id < t
    if (valid) {
      if (act) mids[beg + before] = t;
      else uids[beg + (t - before)] = t;
    }
    running += chunk_total;
    __syncthreads();
  }
  if (threadIdx.x == 0) nm[r] = running;
}

fps_status launch_mask_index(const uint8_t* masks, const int32_t* off, int n_req, int max_len,
                             int32_t* mids, int32_t* uids, int32_t* nm, cudaStream_t s) {
  (void)max_len;
  if (n_req == 0) return FPS_OK;
  prof::begin(s);
  mask_index_kernel<<<n_req, 1024, 0, s>>>(masks, off, mids, uids, nm);
  prof::end(s, prof::INDEX, 0, 0);
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

// ---------------------------------------------------------------------------------------
// NEXT-4 (reading R8): pixel mask [Hp, Wp] -> token mask; token (i, j) is active iff any pixel
// of its f x f block is nonzero; L_txt text tokens appended active.  Thread per token; rows of
// the block read as 16-B vectors when the geometry allows (f % 16 == 0, Wp % 16 == 0).
__global__ void __launch_bounds__(256) mask_pool_kernel(const uint8_t* __restrict__ pix, int Hp,
                                                        int Wp, int f, int L_txt,
                                                        uint8_t* __restrict__ tok) {
  const int Wt = Wp / f, T = (Hp / f) * Wt;
  const int r = blockIdx.y;
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= T + L_txt) return;
  uint8_t* out = tok + (size_t)r * (T + L_txt);
  if (t >= T) {
    out[t] = 1;
    return;
  }
  const uint8_t* p = pix + (size_t)r * Hp * Wp + (size_t)(t / Wt) * f * Wp + (t % Wt) * f;
  bool hit = false;
  if ((f & 15) == 0 && (Wp & 15) == 0 && (reinterpret_cast<uintptr_t>(pix) & 15) == 0) {
    for (int y = 0; y < f && !hit; ++y)
      for (int x = 0; x < f; x += 16) {
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(p + (size_t)y * Wp + x));
        hit |= (v.x | v.y | v.z | v.w) != 0u;
      }
  } else {
    for (int y = 0; y < f && !hit; ++y)
      for (int x = 0; x < f; ++x) hit |= __ldg(p + (size_t)y * Wp + x) != 0;
  }
  out[t] = hit ? 1 : 0;
}

fps_status launch_mask_pool(const uint8_t* pix, int n_req, int Hp, int Wp, int f, int L_txt,
                            uint8_t* tok, cudaStream_t s) {
  const int T = (Hp / f) * (Wp / f) + L_txt;
  if (n_req == 0 || T == 0) return FPS_OK;
  prof::begin(s);
  mask_pool_kernel<<<dim3(ceil_div(T, 256), n_req), 256, 0, s>>>(pix, Hp, Wp, f, L_txt, tok);
  prof::end(s, prof::INDEX, 0, (double)n_req * ((double)Hp * Wp + T));
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

// ---------------------------------------------------------------------------------------
// Row copy by index, 16-B vectors, 4 independent vectors in flight per thread (the source may
// be mapped pinned host memory read over PCIe, so memory-level parallelism matters).
__global__ void __launch_bounds__(256) copy_rows_kernel(const uint4* __restrict__ src,
                                                        const int32_t* __restrict__ src_ids,
                                                        const int32_t* __restrict__ dst_ids,
                                                        long long total, int vpr,
                                                        uint4* __restrict__ dst) {
  pdl_trigger();
  pdl_wait();
  const long long stride = (long long)gridDim.x * blockDim.x;
  long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i < total; i += 4 * stride) {
    uint4 v[4];
    long long di[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      long long idx = i + u * stride;
      di[u] = -1;
      if (idx < total) {
        int row = (int)(idx / vpr), c = (int)(idx - (long long)row * vpr);
        long long sr = src_ids ? __ldg(src_ids + row) : row;
        long long dr = dst_ids ? __ldg(dst_ids + row) : row;
        v[u] = src[sr * vpr + c];
        di[u] = dr * vpr + c;
      }
    }
#pragma unroll
    for (int u = 0; u < 4; ++u)
      if (di[u] >= 0) dst[di[u]] = v[u];
  }
}

fps_status launch_copy_rows(const void* src, const int32_t* src_ids, const int32_t* dst_ids,
                            int n, int row_bytes, void* dst, cudaStream_t s, int max_ctas,
                            bool profile) {
  if (n <= 0) return FPS_OK;
  const int vpr = row_bytes / 16;
  const long long total = (long long)n * vpr;
  long long want = (total + 256 * 4 - 1) / (256 * 4);
  int cap = max_ctas > 0 ? max_ctas : kNumSMs * 8;
  int grid = (int)(want < cap ? want : cap);
  if (grid < 1) grid = 1;
  if (profile) prof::begin(s);
  FPS_CUDA_TRY(launch_k(copy_rows_kernel, dim3(grid), dim3(256), 0, s,
                        reinterpret_cast<const uint4*>(src), src_ids, dst_ids, total, vpr,
                        reinterpret_cast<uint4*>(dst)));
  if (profile) prof::end(s, prof::ROWS, 0, 2.0 * n * row_bytes);
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

// ---------------------------------------------------------------------------------------
// GEGLU weight packing (SDXL block, R24): output row j of group k = j / 64 takes value row
// 32k + (j % 64) for j % 64 < 32, else gate row F + 32k + (j % 64 - 32).  Not on the hot path
// (run once when weights are loaded).
__device__ __forceinline__ int geglu_src_row(int j, int F) {
  const int k = j >> 6, w = j & 63;
  return w < 32 ? 32 * k + w : F + 32 * k + (w - 32);
}

__global__ void __launch_bounds__(256) geglu_pack_kernel(const uint4* __restrict__ w,
                                                         uint4* __restrict__ w_out, int F, int vpr,
                                                         const char* __restrict__ b,
                                                         char* __restrict__ b_out, int elt) {
  const long long total = 2LL * F * vpr;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const int row = (int)(i / vpr), c = (int)(i - (long long)row * vpr);
    w_out[i] = w[(long long)geglu_src_row(row, F) * vpr + c];
  }
  if (b && blockIdx.x == 0)
    for (int j = threadIdx.x; j < 2 * F; j += blockDim.x)
      for (int e = 0; e < elt; ++e) b_out[(size_t)j * elt + e] = b[(size_t)geglu_src_row(j, F) * elt + e];
}

fps_status launch_geglu_pack(int dtype, const void* w, const void* b, int F, int K, void* w_out,
                             void* b_out, cudaStream_t s) {
  const int elt = dtype == FPS_BF16 ? 2 : 4;
  const int vpr = K * elt / 16;
  const long long total = 2LL * F * vpr;
  const int grid = (int)std::min<long long>((total + 255) / 256, kNumSMs * 8LL);
  geglu_pack_kernel<<<grid, 256, 0, s>>>(reinterpret_cast<const uint4*>(w),
                                         reinterpret_cast<uint4*>(w_out), F, vpr,
                                         reinterpret_cast<const char*>(b),
                                         reinterpret_cast<char*>(b_out), elt);
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

// ---------------------------------------------------------------------------------------
// a4: one warp per row; the row stays in registers (VPT 16-B vectors per lane), two-pass
// mean / variance in fp32, then the per-request adaLN modulation (reading R2/R3).
template <typename T, int VPT>
__global__ void __launch_bounds__(128) ln_mod_kernel(const T* __restrict__ x,
                                                     const int32_t* __restrict__ rows, int n,
                                                     int H, T* __restrict__ out, LnMod<T> md,
                                                     const int32_t* __restrict__ out_rows) {
  constexpr int NV = Vec16<T>::N;
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= n) return;
  const bool src2 = md.x2 != nullptr && warp >= md.split;
  const int32_t* rmap = src2 ? md.rows2 : rows;
  const int ridx = src2 ? warp - md.split : warp;
  const int src_row = rmap ? __ldg(rmap + ridx) : ridx;
  const int nvec = H / NV;
  const uint4* xr = reinterpret_cast<const uint4*>((src2 ? md.x2 : x) + (size_t)src_row * H);
  float v[VPT][NV];
  float sum = 0.f;
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    int vi = lane + 32 * k;
    if (vi < nvec) {
      Vec16<T>::unpack(xr[vi], v[k]);
#pragma unroll
      for (int e = 0; e < NV; ++e) sum += v[k][e];
    } else {
#pragma unroll
      for (int e = 0; e < NV; ++e) v[k][e] = 0.f;
    }
  }
  const float mean = warp_sum(sum) / (float)H;
  float sq = 0.f;
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    if (lane + 32 * k < nvec) {
#pragma unroll
      for (int e = 0; e < NV; ++e) {
        float d = v[k][e] - mean;
        sq += d * d;
      }
    }
  }
  const float var = warp_sum(sq) / (float)H;
  const float rstd = 1.0f / sqrtf(var + 1e-6f);
  const bool mod = md.shift != nullptr;
  const T* shift = nullptr;
  const T* scale = nullptr;
  if (mod) {
    const bool g2 = warp >= md.split;
    const size_t off = (md.stride ? (size_t)find_req(g2 ? md.cu2 : md.cu, md.n_req,
                                                     g2 ? warp - md.split : warp) * md.stride : 0) +
                       (g2 ? md.soff : 0);
    shift = md.shift + off;
    scale = md.scale + off;
  }
  uint4* o = (src2 && md.outb) ? nullptr
                               : reinterpret_cast<uint4*>(out + (size_t)(out_rows ? __ldg(out_rows + warp) : warp) * H);
  uint4* ob = md.outb ? reinterpret_cast<uint4*>(
                            md.outb + (size_t)(src2 ? __ldg(md.outb_rows2 + warp - md.split)
                                                    : __ldg(md.outb_rows1 + warp)) * H)
                      : nullptr;
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    int vi = lane + 32 * k;
    if (vi < nvec) {
      float r[NV];
      if (mod) {
        float sh[NV], sc[NV];
        Vec16<T>::unpack(reinterpret_cast<const uint4*>(shift)[vi], sh);
        Vec16<T>::unpack(reinterpret_cast<const uint4*>(scale)[vi], sc);
#pragma unroll
        for (int e = 0; e < NV; ++e) r[e] = (v[k][e] - mean) * rstd * (md.one + sc[e]) + sh[e];
      } else {
#pragma unroll
        for (int e = 0; e < NV; ++e) r[e] = (v[k][e] - mean) * rstd;
      }
      const uint4 pr = Vec16<T>::pack(r);
      if (o) o[vi] = pr;
      if (ob) ob[vi] = pr;
    }
  }
}

// Wide rows (H >= 1024 bf16): one 128-thread CTA per row, VPT 16-B vectors per thread.  Every
// global load of the row -- x and the request's shift / scale vectors -- is issued up front, so a
// row costs one memory round trip plus two block reductions (mean, then centred variance).
template <typename T, int VPT>
__global__ void __launch_bounds__(128) ln_mod_row_kernel(const T* __restrict__ x,
                                                         const int32_t* __restrict__ rows, int H,
                                                         T* __restrict__ out, LnMod<T> md,
                                                         const int32_t* __restrict__ out_rows) {
  constexpr int NV = Vec16<T>::N;
  __shared__ float red[4];
  pdl_trigger();
  pdl_wait();
  const int row = blockIdx.x, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nvec = H / NV;
  const bool src2 = md.x2 != nullptr && row >= md.split;
  const int32_t* rmap = src2 ? md.rows2 : rows;
  const int ridx = src2 ? row - md.split : row;
  const int src_row = rmap ? __ldg(rmap + ridx) : ridx;
  const uint4* xr = reinterpret_cast<const uint4*>((src2 ? md.x2 : x) + (size_t)src_row * H);
  const bool mod = md.shift != nullptr;
  const uint4* sh = nullptr;
  const uint4* sc = nullptr;
  if (mod) {
    const bool g2 = row >= md.split;
    const size_t off = (md.stride ? (size_t)find_req(g2 ? md.cu2 : md.cu, md.n_req,
                                                     g2 ? row - md.split : row) * md.stride : 0) +
                       (g2 ? md.soff : 0);
    sh = reinterpret_cast<const uint4*>(md.shift + off);
    sc = reinterpret_cast<const uint4*>(md.scale + off);
  }
  uint4 xv[VPT], shv[VPT], scv[VPT];
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    const int vi = tid + 128 * k;
    const bool ok = vi < nvec;
    xv[k] = ok ? __ldg(xr + vi) : make_uint4(0, 0, 0, 0);
    shv[k] = (ok && mod) ? __ldg(sh + vi) : make_uint4(0, 0, 0, 0);
    scv[k] = (ok && mod) ? __ldg(sc + vi) : make_uint4(0, 0, 0, 0);
  }
  float v[VPT][NV];
  float sum = 0.f;
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    Vec16<T>::unpack(xv[k], v[k]);
#pragma unroll
    for (int e = 0; e < NV; ++e) sum += v[k][e];
  }
  sum = warp_sum(sum);
  if (lane == 0) red[warp] = sum;
  __syncthreads();
  const float mean = (red[0] + red[1] + red[2] + red[3]) / (float)H;
  __syncthreads();
  float sq = 0.f;
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    if (tid + 128 * k < nvec) {
#pragma unroll
      for (int e = 0; e < NV; ++e) {
        const float d = v[k][e] - mean;
        sq += d * d;
      }
    }
  }
  sq = warp_sum(sq);
  if (lane == 0) red[warp] = sq;
  __syncthreads();
  const float rstd = 1.0f / sqrtf((red[0] + red[1] + red[2] + red[3]) / (float)H + 1e-6f);
  uint4* o = (src2 && md.outb) ? nullptr
                               : reinterpret_cast<uint4*>(out + (size_t)(out_rows ? __ldg(out_rows + row) : row) * H);
  uint4* ob = md.outb ? reinterpret_cast<uint4*>(
                            md.outb + (size_t)(src2 ? __ldg(md.outb_rows2 + row - md.split)
                                                    : __ldg(md.outb_rows1 + row)) * H)
                      : nullptr;
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    const int vi = tid + 128 * k;
    if (vi < nvec) {
      float r[NV], a[NV], b[NV];
      Vec16<T>::unpack(shv[k], a);
      Vec16<T>::unpack(scv[k], b);
#pragma unroll
      for (int e = 0; e < NV; ++e) r[e] = (v[k][e] - mean) * rstd * (md.one + b[e]) + a[e];
      const uint4 pr = Vec16<T>::pack(r);
      if (o) o[vi] = pr;
      if (ob) ob[vi] = pr;
    }
  }
}

template <typename T>
static fps_status ln_mod_t(const void* x, const int32_t* rows, int n, int H, void* out,
                           LnMod<T> Md, cudaStream_t s, const int32_t* out_rows) {
  constexpr int NV = Vec16<T>::N;
  const int per_lane = ceil_div(H / NV, 32);
  const int grid = ceil_div(n, 4);
  auto X = reinterpret_cast<const T*>(x);
  auto O = reinterpret_cast<T*>(out);
  if (!Md.shift) Md.one = 1.0f;
  const int per_thread = ceil_div(H / NV, 128);
  if (H / NV >= 128 && per_thread <= 8) {
    prof::begin(s);
    cudaError_t le;
#define FPS_LNR_CASE(VPT)                                                                  \
    if (per_thread <= VPT)                                                                 \
      le = launch_k(ln_mod_row_kernel<T, VPT>, dim3(n), dim3(128), 0, s, X, rows, H, O, Md, \
                    out_rows);                                                             \
    else
    FPS_LNR_CASE(1) FPS_LNR_CASE(2) FPS_LNR_CASE(3) FPS_LNR_CASE(4) FPS_LNR_CASE(6)
    le = launch_k(ln_mod_row_kernel<T, 8>, dim3(n), dim3(128), 0, s, X, rows, H, O, Md, out_rows);
#undef FPS_LNR_CASE
    FPS_CUDA_TRY(le);
    prof::end(s, prof::LN, 0, 2.0 * n * H * sizeof(T));
    count_launch();
    FPS_LAUNCH_CHECK();
    return FPS_OK;
  }
#define FPS_LN_CASE(VPT)                                                                  \
  if (per_lane <= VPT) {                                                                  \
    prof::begin(s);                                                                       \
    ln_mod_kernel<T, VPT><<<grid, 128, 0, s>>>(X, rows, n, H, O, Md, out_rows);           \
    prof::end(s, prof::LN, 0, 2.0 * n * H * sizeof(T));                                   \
    count_launch();                                                                       \
    FPS_LAUNCH_CHECK();                                                                   \
    return FPS_OK;                                                                        \
  }
  FPS_LN_CASE(1)
  FPS_LN_CASE(2)
  FPS_LN_CASE(4)
  FPS_LN_CASE(8)
  FPS_LN_CASE(12)
  FPS_LN_CASE(16)
#undef FPS_LN_CASE
  return fail(FPS_EUNSUPPORTED, "ln_mod: H=%d too large", H);
}

// SDXL block norms over the fp32 residual stream (R24): one 128-thread CTA per row, fp32 input
// (VPT float4 per thread), bf16 output LN(x) * gamma + beta.
template <int VPT>
__global__ void __launch_bounds__(128) ln_affine_f32_kernel(const float* __restrict__ x, int H,
                                                            __nv_bfloat16* __restrict__ out,
                                                            const __nv_bfloat16* __restrict__ gamma,
                                                            const __nv_bfloat16* __restrict__ beta) {
  __shared__ float red[4];
  pdl_trigger();
  pdl_wait();
  const int row = blockIdx.x, tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nvec = H / 4;
  const float4* xr = reinterpret_cast<const float4*>(x + (size_t)row * H);
  float4 v[VPT];
  float sum = 0.f;
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    const int vi = tid + 128 * k;
    v[k] = vi < nvec ? __ldg(xr + vi) : make_float4(0.f, 0.f, 0.f, 0.f);
    sum += (v[k].x + v[k].y) + (v[k].z + v[k].w);
  }
  sum = warp_sum(sum);
  if (lane == 0) red[warp] = sum;
  __syncthreads();
  const float mean = (red[0] + red[1] + red[2] + red[3]) / (float)H;
  __syncthreads();
  float sq = 0.f;
#pragma unroll
  for (int k = 0; k < VPT; ++k)
    if (tid + 128 * k < nvec) {
      const float a = v[k].x - mean, b = v[k].y - mean, c = v[k].z - mean, d = v[k].w - mean;
      sq += (a * a + b * b) + (c * c + d * d);
    }
  sq = warp_sum(sq);
  if (lane == 0) red[warp] = sq;
  __syncthreads();
  const float rstd = 1.0f / sqrtf((red[0] + red[1] + red[2] + red[3]) / (float)H + 1e-6f);
  uint2* o = reinterpret_cast<uint2*>(out + (size_t)row * H);
  const uint2* gp = reinterpret_cast<const uint2*>(gamma);
  const uint2* bp = reinterpret_cast<const uint2*>(beta);
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    const int vi = tid + 128 * k;
    if (vi < nvec) {
      const uint2 gv = __ldg(gp + vi), bv = __ldg(bp + vi);
      float g0, g1, g2, g3, b0, b1, b2, b3;
      unpack_bf16x2(gv.x, g0, g1); unpack_bf16x2(gv.y, g2, g3);
      unpack_bf16x2(bv.x, b0, b1); unpack_bf16x2(bv.y, b2, b3);
      o[vi] = make_uint2(pack_bf16x2((v[k].x - mean) * rstd * g0 + b0, (v[k].y - mean) * rstd * g1 + b1),
                         pack_bf16x2((v[k].z - mean) * rstd * g2 + b2, (v[k].w - mean) * rstd * g3 + b3));
    }
  }
}

// Narrow rows (H <= 1024): one warp per row, VPT float4 per lane, shuffle-only reductions.
template <int VPT>
__global__ void __launch_bounds__(128) ln_affine_f32_warp_kernel(const float* __restrict__ x, int n,
                                                                 int H, __nv_bfloat16* __restrict__ out,
                                                                 const __nv_bfloat16* __restrict__ gamma,
                                                                 const __nv_bfloat16* __restrict__ beta) {
  pdl_trigger();
  pdl_wait();
  const int row = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (row >= n) return;
  const int nvec = H / 4;
  const float4* xr = reinterpret_cast<const float4*>(x + (size_t)row * H);
  const uint2* gp = reinterpret_cast<const uint2*>(gamma);
  const uint2* bp = reinterpret_cast<const uint2*>(beta);
  float4 v[VPT];
  uint2 gv[VPT], bv[VPT];
  float sum = 0.f;
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    const int vi = lane + 32 * k;
    const bool ok = vi < nvec;
    v[k] = ok ? __ldg(xr + vi) : make_float4(0.f, 0.f, 0.f, 0.f);
    gv[k] = ok ? __ldg(gp + vi) : make_uint2(0, 0);
    bv[k] = ok ? __ldg(bp + vi) : make_uint2(0, 0);
    sum += (v[k].x + v[k].y) + (v[k].z + v[k].w);
  }
  const float mean = warp_sum(sum) / (float)H;
  float sq = 0.f;
#pragma unroll
  for (int k = 0; k < VPT; ++k)
    if (lane + 32 * k < nvec) {
      const float a = v[k].x - mean, b = v[k].y - mean, c = v[k].z - mean, d = v[k].w - mean;
      sq += (a * a + b * b) + (c * c + d * d);
    }
  const float rstd = 1.0f / sqrtf(warp_sum(sq) / (float)H + 1e-6f);
  uint2* o = reinterpret_cast<uint2*>(out + (size_t)row * H);
#pragma unroll
  for (int k = 0; k < VPT; ++k) {
    const int vi = lane + 32 * k;
    if (vi < nvec) {
      float g0, g1, g2, g3, b0, b1, b2, b3;
      unpack_bf16x2(gv[k].x, g0, g1); unpack_bf16x2(gv[k].y, g2, g3);
      unpack_bf16x2(bv[k].x, b0, b1); unpack_bf16x2(bv[k].y, b2, b3);
      o[vi] = make_uint2(pack_bf16x2((v[k].x - mean) * rstd * g0 + b0, (v[k].y - mean) * rstd * g1 + b1),
                         pack_bf16x2((v[k].z - mean) * rstd * g2 + b2, (v[k].w - mean) * rstd * g3 + b3));
    }
  }
}

fps_status launch_ln_affine_f32in(const float* x, int n, int H, void* out, const void* gamma,
                                  const void* beta, cudaStream_t s) {
  if (n <= 0) return FPS_OK;
  if (H % 4) return fail(FPS_EUNSUPPORTED, "ln_affine_f32: H=%d not a multiple of 4", H);
  const int per = ceil_div(H / 4, 128);
  auto G = reinterpret_cast<const __nv_bfloat16*>(gamma);
  auto Bt = reinterpret_cast<const __nv_bfloat16*>(beta);
  auto O = reinterpret_cast<__nv_bfloat16*>(out);
  prof::begin(s);
  cudaError_t le;
  const int per_lane = ceil_div(H / 4, 32), wgrid = ceil_div(n, 4);
  if (per_lane <= 4)
    le = launch_k(ln_affine_f32_warp_kernel<4>, dim3(wgrid), dim3(128), 0, s, x, n, H, O, G, Bt);
  else if (per_lane <= 8)
    le = launch_k(ln_affine_f32_warp_kernel<8>, dim3(wgrid), dim3(128), 0, s, x, n, H, O, G, Bt);
  else if (per <= 2) le = launch_k(ln_affine_f32_kernel<2>, dim3(n), dim3(128), 0, s, x, H, O, G, Bt);
  else if (per <= 4) le = launch_k(ln_affine_f32_kernel<4>, dim3(n), dim3(128), 0, s, x, H, O, G, Bt);
  else if (per <= 8) le = launch_k(ln_affine_f32_kernel<8>, dim3(n), dim3(128), 0, s, x, H, O, G, Bt);
  else if (per <= 16) le = launch_k(ln_affine_f32_kernel<16>, dim3(n), dim3(128), 0, s, x, H, O, G, Bt);
  else return fail(FPS_EUNSUPPORTED, "ln_affine_f32: H=%d too large", H);
  FPS_CUDA_TRY(le);
  prof::end(s, prof::LN, 0, 6.0 * n * H);
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

template <typename T>
static LnMod<T> ln_params(const void* shift, const void* scale, int stride, float one,
                          const int32_t* cu, int n_req, int split = 0x7fffffff, int soff = 0,
                          const int32_t* cu2 = nullptr, const void* x2 = nullptr,
                          const int32_t* rows2 = nullptr) {
  return LnMod<T>{reinterpret_cast<const T*>(shift), reinterpret_cast<const T*>(scale), stride, one,
                  cu, n_req, split, soff, cu2, reinterpret_cast<const T*>(x2), rows2};
}

fps_status launch_ln_mod2(int dtype, const void* x, const int32_t* rows, int n, int H, void* out,
                          const int32_t* cu, const int32_t* cu2, int split, int n_req,
                          const void* mod, int shift_off, int soff, cudaStream_t s,
                          int mod_stride) {
  if (n <= 0) return FPS_OK;
  const size_t e = dtype == FPS_BF16 ? 2 : 4;
  const char* sh = mod ? (const char*)mod + (size_t)shift_off * e : nullptr;
  const char* sc = mod ? sh + (size_t)H * e : nullptr;
  if (dtype == FPS_BF16)
    return ln_mod_t<__nv_bfloat16>(
        x, rows, n, H, out,
        ln_params<__nv_bfloat16>(sh, sc, mod_stride, 1.0f, cu, n_req, split, soff, cu2), s, nullptr);
  return ln_mod_t<float>(x, rows, n, H, out,
                         ln_params<float>(sh, sc, mod_stride, 1.0f, cu, n_req, split, soff, cu2), s,
                         nullptr);
}

fps_status launch_ln_mod(int dtype, const void* x, const int32_t* rows, int n, int H, void* out,
                         const int32_t* cu, int n_req, const void* mod, int shift_off,
                         cudaStream_t s, const int32_t* out_rows, int mod_stride) {
  if (n <= 0) return FPS_OK;
  if (mod_stride <= 0) mod_stride = 6 * H;
  const size_t e = dtype == FPS_BF16 ? 2 : 4;
  const char* sh = mod ? (const char*)mod + (size_t)shift_off * e : nullptr;
  const char* sc = mod ? sh + (size_t)H * e : nullptr;
  if (dtype == FPS_BF16)
    return ln_mod_t<__nv_bfloat16>(x, rows, n, H, out,
                                   ln_params<__nv_bfloat16>(sh, sc, mod_stride, 1.0f, cu, n_req),
                                   s, out_rows);
  return ln_mod_t<float>(x, rows, n, H, out, ln_params<float>(sh, sc, mod_stride, 1.0f, cu, n_req),
                         s, out_rows);
}

// Two row sources in one launch, one output: rows [0, n0) are LN-mod of x0 at rows0 (requests
// from cu0), rows [n0, n0 + n1) of x1 at rows1 (requests from cu1); the same modulation vectors
fps_status launch_ln_mod_2src(int dtype, const void* x0, const int32_t* rows0, int n0,
                              const void* x1, const int32_t* rows1, int n1, int H, void* out,
                              const int32_t* cu0, const int32_t* cu1, int n_req, const void* mod,
                              int shift_off, cudaStream_t s, int mod_stride) {
  if (n1 <= 0) return launch_ln_mod(dtype, x0, rows0, n0, H, out, cu0, n_req, mod, shift_off, s,
                                    nullptr, mod_stride);
  if (mod_stride <= 0) mod_stride = 6 * H;
  const size_t e = dtype == FPS_BF16 ? 2 : 4;
  const char* sh = mod ? (const char*)mod + (size_t)shift_off * e : nullptr;
  const char* sc = mod ? sh + (size_t)H * e : nullptr;
  if (dtype == FPS_BF16)
    return ln_mod_t<__nv_bfloat16>(x0, rows0, n0 + n1, H, out,
                                   ln_params<__nv_bfloat16>(sh, sc, mod_stride, 1.0f, cu0, n_req, n0,
                                                            0, cu1, x1, rows1),
                                   s, nullptr);
  return ln_mod_t<float>(x0, rows0, n0 + n1, H, out,
                         ln_params<float>(sh, sc, mod_stride, 1.0f, cu0, n_req, n0, 0, cu1, x1,
                                          rows1),
                         s, nullptr);
}

// The y_split norm in one launch: rows [0, n0) of x0 at rows0 -> out[r] and outb[outb_rows0[r]];
// rows [n0, n0 + n1) of x1 at rows1 -> outb[outb_rows1[r - n0]] only.  Modulation as
// launch_ln_mod_2src (cu0 / cu1), or the affine LN (gamma / beta) when `gamma` is given.
fps_status launch_ln_ysplit(int dtype, const void* x0, const int32_t* rows0, int n0,
                            const void* x1, const int32_t* rows1, int n1, int H, void* out,
                            void* outb, const int32_t* outb_rows0, const int32_t* outb_rows1,
                            const int32_t* cu0, const int32_t* cu1, int n_req, const void* mod,
                            int shift_off, int mod_stride, const void* gamma, const void* beta,
                            cudaStream_t s) {
  if (n0 + n1 <= 0) return FPS_OK;
  if (mod_stride <= 0) mod_stride = 6 * H;
  const size_t e = dtype == FPS_BF16 ? 2 : 4;
  const char* sh = gamma ? (const char*)beta : mod ? (const char*)mod + (size_t)shift_off * e : nullptr;
  const char* sc = gamma ? (const char*)gamma : mod ? sh + (size_t)H * e : nullptr;
  const int stride = gamma ? 0 : mod_stride;
  const float one = gamma ? 0.0f : 1.0f;
  if (dtype == FPS_BF16) {
    auto md = ln_params<__nv_bfloat16>(sh, sc, stride, one, gamma ? nullptr : cu0, n_req, n0, 0,
                                       gamma ? nullptr : cu1, x1, rows1);
    md.outb = reinterpret_cast<__nv_bfloat16*>(outb);
    md.outb_rows1 = outb_rows0;
    md.outb_rows2 = outb_rows1;
    return ln_mod_t<__nv_bfloat16>(x0, rows0, n0 + n1, H, out, md, s, nullptr);
  }
  auto md = ln_params<float>(sh, sc, stride, one, gamma ? nullptr : cu0, n_req, n0, 0,
                             gamma ? nullptr : cu1, x1, rows1);
  md.outb = reinterpret_cast<float*>(outb);
  md.outb_rows1 = outb_rows0;
  md.outb_rows2 = outb_rows1;
  return ln_mod_t<float>(x0, rows0, n0 + n1, H, out, md, s, nullptr);
}

fps_status launch_ln_affine(int dtype, const void* x, const int32_t* rows, int n, int H, void* out,
                            const void* gamma, const void* beta, cudaStream_t s,
                            const int32_t* out_rows) {
  if (n <= 0) return FPS_OK;
  if (dtype == FPS_BF16)
    return ln_mod_t<__nv_bfloat16>(x, rows, n, H, out,
                                   ln_params<__nv_bfloat16>(beta, gamma, 0, 0.0f, nullptr, 0), s,
                                   out_rows);
  return ln_mod_t<float>(x, rows, n, H, out, ln_params<float>(beta, gamma, 0, 0.0f, nullptr, 0), s,
                         out_rows);
}

// ---------------------------------------------------------------------------------------
// Synthetic sampler update over the full latent (reading R21): x <- x + delta_req * y.
template <typename T>
__global__ void __launch_bounds__(256) euler_kernel(T* __restrict__ x, const T* __restrict__ y,
                                                    long long nvec, int vpr,
                                                    const int32_t* __restrict__ cu, int n_req,
                                                    const float* __restrict__ delta) {
  constexpr int NV = Vec16<T>::N;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nvec;
       i += (long long)gridDim.x * blockDim.x) {
    const int row = (int)(i / vpr);
    const float d = __ldg(delta + find_req(cu, n_req, row));
    float a[NV], b[NV];
    Vec16<T>::unpack(reinterpret_cast<const uint4*>(x)[i], a);
    Vec16<T>::unpack(reinterpret_cast<const uint4*>(y)[i], b);
#pragma unroll
    for (int e = 0; e < NV; ++e) a[e] = a[e] + d * b[e];
    reinterpret_cast<uint4*>(x)[i] = Vec16<T>::pack(a);
  }
}

// Flow-matching Euler step with inpainting blend (reading R29, NEXT-4; PAPER.md L73-L79 the
// latent goes through N denoising steps, L157 masked rows computed / unmasked rows kept from the
// template).  Per request r at its step s (coefficients coef[r] = (sigma_{s+1} - sigma_s,
// sigma_{s+1})), row t of its latent:
//   text row (t >= L_img)          unchanged (the prompt tokens are re-fed every step)
//   masked image row (mask[t] != 0) x += (sigma_{s+1} - sigma_s) * y      (Euler on the velocity)
//   unmasked image row               x  = (1 - sigma_{s+1}) * z[t] + sigma_{s+1} * eps[t]
//                                        (the template latent re-noised to the next level)
template <typename T>
__global__ void __launch_bounds__(256) flow_blend_kernel(T* __restrict__ x, const T* __restrict__ y,
                                                         long long nvec, int vpr, int L, int L_img,
                                                         const uint8_t* __restrict__ mask,
                                                         const float2* __restrict__ coef,
                                                         const void* const* __restrict__ zeps) {
  constexpr int NV = Vec16<T>::N;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nvec;
       i += (long long)gridDim.x * blockDim.x) {
    const int row = (int)(i / vpr), c = (int)(i - (long long)row * vpr);
    const int r = row / L, t = row - r * L;
    if (t >= L_img) continue;
    const float2 cf = __ldg(coef + r);
    float a[NV];
    if (__ldg(mask + row)) {
      float b[NV];
      Vec16<T>::unpack(reinterpret_cast<const uint4*>(x)[i], a);
      Vec16<T>::unpack(reinterpret_cast<const uint4*>(y)[i], b);
#pragma unroll
      for (int e = 0; e < NV; ++e) a[e] = a[e] + cf.x * b[e];
    } else {
      const uint4* z = reinterpret_cast<const uint4*>(zeps[2 * r]);
      const uint4* ep = reinterpret_cast<const uint4*>(zeps[2 * r + 1]);
      float b[NV];
      Vec16<T>::unpack(z[(long long)t * vpr + c], a);
      Vec16<T>::unpack(ep[(long long)t * vpr + c], b);
#pragma unroll
      for (int e = 0; e < NV; ++e) a[e] = (1.0f - cf.y) * a[e] + cf.y * b[e];
    }
    reinterpret_cast<uint4*>(x)[i] = Vec16<T>::pack(a);
  }
}

fps_status launch_flow_blend(int dtype, void* x, const void* y, int n_req, int L, int L_img, int H,
                             const uint8_t* mask, const float2* coef, const void* const* zeps,
                             cudaStream_t s) {
  const int n = n_req * L;
  if (n <= 0) return FPS_OK;
  const int elt = dtype == FPS_BF16 ? 2 : 4;
  const int vpr = H * elt / 16;
  const long long nvec = (long long)n * vpr;
  int grid = (int)((nvec + 255) / 256);
  if (grid > kNumSMs * 16) grid = kNumSMs * 16;
  prof::begin(s);
  if (dtype == FPS_BF16)
    flow_blend_kernel<__nv_bfloat16><<<grid, 256, 0, s>>>(
        (__nv_bfloat16*)x, (const __nv_bfloat16*)y, nvec, vpr, L, L_img, mask, coef, zeps);
  else
    flow_blend_kernel<float><<<grid, 256, 0, s>>>((float*)x, (const float*)y, nvec, vpr, L, L_img,
                                                  mask, coef, zeps);
  prof::end(s, prof::EULER, 2.0 * n * H, 3.0 * n * H * elt);
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

fps_status launch_euler(int dtype, void* x, const void* y, int n, int H, const int32_t* cu,
                        int n_req, const float* delta, cudaStream_t s) {
  if (n <= 0) return FPS_OK;
  const int elt = dtype == FPS_BF16 ? 2 : 4;
  const int vpr = H * elt / 16;
  const long long nvec = (long long)n * vpr;
  int grid = (int)((nvec + 255) / 256);
  if (grid > kNumSMs * 16) grid = kNumSMs * 16;
  prof::begin(s);
  if (dtype == FPS_BF16)
    euler_kernel<__nv_bfloat16><<<grid, 256, 0, s>>>((__nv_bfloat16*)x, (const __nv_bfloat16*)y,
                                                     nvec, vpr, cu, n_req, delta);
  else
    euler_kernel<float><<<grid, 256, 0, s>>>((float*)x, (const float*)y, nvec, vpr, cu, n_req,
                                             delta);
  prof::end(s, prof::EULER, 2.0 * n * H, 3.0 * n * H * elt);
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

}  // namespace fps
