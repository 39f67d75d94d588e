// a5/a7/a8: the masked-row projections and MLP as persistent, warp-specialised tcgen05 GEMMs.
// C[M, N] = A[M, K] . B[N, K]^T, bf16 in, fp32 accumulate in TMEM, fused epilogue (bias, GELU,
// gated residual, K/V row scatter into the merged key buffer -- PAPER.md L157/L161).
//
// Two kernels share the epilogue:
//  * gemm_tc_kernel (1 SM per tile, M=128 x BN): for small M.
//  * gemm_tc2_kernel (CTA pair, tcgen05 cta_group::2, 256 x 256 tile): each CTA of the pair loads
//    its 128 rows of A and its 128 rows of B; the leader's single thread issues M=256 MMAs that read
//    both CTAs' shared memory and accumulate rows 0-127 in CTA 0's TMEM, 128-255 in CTA 1's.
//    Per SM this halves the operand bytes per FLOP (L2 -> SM traffic) and the 6-stage ring gives
//    a deeper prefetch than the 4-stage 1-SM ring; 256-row tiles also cut wave quantisation for
//    the M of masked blocks (e.g. M = 1331: 72 or 216 pair tiles on 74 SM pairs).
//
//   warp 0      TMA producer (both CTAs), STAGES-deep 128B-swizzled smem ring
//   warp 1      MMA issuer (one thread; leader CTA only in the pair kernel)
//   warp 2      TMEM allocator (two accumulators: tile i's epilogue overlaps tile i+1's MMAs)
//   warps 4-7   epilogue: tcgen05.ld 32 columns at a time (thread = output row), fused ops,
//               all global loads of a chunk issued before use, 16-B stores
// Tiles are visited n-major so the CTAs working at the same time share one weight tile (L2).
#include <algorithm>

#include "epilogue.cuh"
#include "kernels.h"
#include "tc_util.cuh"

namespace fps {

// Grouped raster: tiles walk groups of GM m-blocks, n-major inside a group, so the CTAs running
// at the same time touch GM row panels of A and a few column panels of B -- both stay in L2 even
// when A is large (continuous batches: M ~ 30k rows).  For num_m <= GM this is plain n-major.
template <int GM>
__device__ __forceinline__ void tile_coords(int tile, int num_m, int num_n, int& m_blk, int& n_blk) {
  const int group = tile / (GM * num_n);
  const int first_m = group * GM;
  const int gm = min(num_m - first_m, GM);
  const int local = tile - group * GM * num_n;
  m_blk = first_m + local % gm;
  n_blk = local / gm;
}

// Grouped launch: problem 0 = rows [0, M) of A with B [N, K] and `ep`, problem 1 = rows
// [M, M + M1) with B1 [N1, K] and `ep1` (row-local epilogue indexing), the same K.  Used by the
// double-stream block (R25: image / text rows on their own weights, N1 = N) and by the Y-mode
// parallel block (rows M on [Q|K|V|Z], cached rows U on [K|V]: N1 = 2H < N), so one persistent
// grid covers both problems' tiles -- no second partial wave.  Tiles [0, T0) belong to
// problem 0, the rest to problem 1.
template <int GM>
__device__ __forceinline__ void group_coords(int tile, int T0, int num_m0, int num_m1, int num_n0,
                                             int num_n1, int& p, int& m_blk, int& n_blk) {
  if (tile < T0) {
    p = 0;
    tile_coords<GM>(tile, num_m0, num_n0, m_blk, n_blk);
  } else {
    p = 1;
    tile_coords<GM>(tile - T0, num_m1, num_n1, m_blk, n_blk);
  }
}

// Per-row epilogue context: gate vector of the row's request and the output rows of both
// column ranges (K/V scatter into the merged key buffer).
struct RowCtx {
  const __nv_bfloat16* gate;
  int row, orow0, orow1, rrow;
  bool ok;
};
__device__ __forceinline__ RowCtx row_ctx(const Epilogue& ep, int M, int row) {
  RowCtx c{nullptr, row, row, row, row, row < M};
  if (c.ok) {
    if (ep.resid_map) c.rrow = __ldg(ep.resid_map + row);
    if (ep.gate)
      c.gate = reinterpret_cast<const __nv_bfloat16*>(ep.gate) +
               (size_t)find_req(ep.cu, ep.n_req, row) * ep.gate_stride;
    if (ep.map0) c.orow0 = __ldg(ep.map0 + row);
    if (ep.map1) c.orow1 = __ldg(ep.map1 + row);
  }
  return c;
}

// Global loads of the fused operands of 32 columns col0.. of one row (issued before use).
struct ChunkIn {
  uint4 bv[4], rv[8], gv[4];   // rv[4..7]: second halves of an fp32 residual
};
__device__ __forceinline__ void chunk_load(const Epilogue& ep, const RowCtx& rc, int N, int row,
                                           int col0, ChunkIn& in, bool skip_resid = false) {
  const __nv_bfloat16* __restrict__ bias = reinterpret_cast<const __nv_bfloat16*>(ep.bias);
  const __nv_bfloat16* __restrict__ resid =
      skip_resid ? nullptr : reinterpret_cast<const __nv_bfloat16*>(ep.resid);
#pragma unroll
  for (int g = 0; g < 4; ++g) {
    const int c0 = col0 + g * 8;
    const bool ok = rc.ok && c0 < N;
    in.bv[g] = (bias && ok) ? __ldg(reinterpret_cast<const uint4*>(bias + c0)) : make_uint4(0, 0, 0, 0);
    if (ep.resid_f32) {
      const float* rf = reinterpret_cast<const float*>(ep.resid) + (size_t)rc.rrow * ep.ld_resid + c0;
      in.rv[g] = (resid && ok) ? __ldg(reinterpret_cast<const uint4*>(rf)) : make_uint4(0, 0, 0, 0);
      in.rv[g + 4] = (resid && ok) ? __ldg(reinterpret_cast<const uint4*>(rf + 4)) : make_uint4(0, 0, 0, 0);
    } else {
      in.rv[g] = (resid && ok)
                     ? __ldg(reinterpret_cast<const uint4*>(resid + (size_t)rc.rrow * ep.ld_resid + c0))
                     : make_uint4(0, 0, 0, 0);
    }
    in.gv[g] = (rc.gate && ok) ? __ldg(reinterpret_cast<const uint4*>(rc.gate + c0))
                               : make_uint4(0, 0, 0, 0);
  }
}

// Fused ops + 16-B stores of 32 accumulator values (fp32 bits) of one row, columns col0..
__device__ __forceinline__ void chunk_store(const Epilogue& ep, const RowCtx& rc, int N, int col0,
                                            const uint32_t* r, const ChunkIn& in) {
  if (!rc.ok) return;
#pragma unroll
  for (int g = 0; g < 4; ++g) {
    const int c0 = col0 + g * 8;
    if (c0 >= N) continue;
    float v[8], t[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) v[e] = __uint_as_float(r[g * 8 + e]);
    if (ep.bias) {
      Vec16<__nv_bfloat16>::unpack(in.bv[g], t);
#pragma unroll
      for (int e = 0; e < 8; ++e) v[e] += t[e];
    }
    if (ep.act == 1 && c0 >= ep.act_from) {
#pragma unroll
      for (int e = 0; e < 8; ++e) v[e] = gelu_tanh_fast(v[e]);
    }
    if (ep.resid) {
      float rr[8];
      if (ep.resid_f32) {
        Vec16<float>::unpack(in.rv[g], rr);
        Vec16<float>::unpack(in.rv[g + 4], rr + 4);
      } else {
        Vec16<__nv_bfloat16>::unpack(in.rv[g], rr);
      }
      if (rc.gate) {
        Vec16<__nv_bfloat16>::unpack(in.gv[g], t);
#pragma unroll
        for (int e = 0; e < 8; ++e) v[e] = rr[e] + t[e] * v[e];
      } else {
#pragma unroll
        for (int e = 0; e < 8; ++e) v[e] = rr[e] + v[e];
      }
    }
    if (ep.out0_f32 && c0 < ep.split) {
      float* df = reinterpret_cast<float*>(ep.out0) + (size_t)rc.orow0 * ep.ld0 + c0;
      reinterpret_cast<uint4*>(df)[0] = Vec16<float>::pack(v);
      reinterpret_cast<uint4*>(df)[1] = Vec16<float>::pack(v + 4);
      continue;
    }
    __nv_bfloat16* dst =
        c0 < ep.split ? reinterpret_cast<__nv_bfloat16*>(ep.out0) + (size_t)rc.orow0 * ep.ld0 + c0
        : (ep.out2 && c0 >= ep.split2)
            ? reinterpret_cast<__nv_bfloat16*>(ep.out2) + (size_t)rc.row * ep.ld2 + (c0 - ep.split2)
            : reinterpret_cast<__nv_bfloat16*>(ep.out1) + (size_t)rc.orow1 * ep.ld1 +
                  (c0 - ep.split);
    *reinterpret_cast<uint4*>(dst) = Vec16<__nv_bfloat16>::pack(v);
  }
}

// GEGLU (act 2, SDXL block R24): accumulator columns col0..+31 are the value half and
// col0+32..+63 the gate half of output columns col0/2..+31 (weights packed by
// launch_geglu_pack); out = (value + b) * GELU_tanh(gate + b').
__device__ __forceinline__ void geglu_store(const Epilogue& ep, const RowCtx& rc, int N, int col0,
                                            const uint32_t* ra, const uint32_t* rg,
                                            const ChunkIn& ia, const ChunkIn& ig) {
  if (!rc.ok || col0 >= N) return;
  __nv_bfloat16* out =
      reinterpret_cast<__nv_bfloat16*>(ep.out0) + (size_t)rc.orow0 * ep.ld0 + (col0 >> 1);
#pragma unroll
  for (int g = 0; g < 4; ++g) {
    float v[8], t[8], b[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      v[e] = __uint_as_float(ra[g * 8 + e]);
      t[e] = __uint_as_float(rg[g * 8 + e]);
    }
    if (ep.bias) {
      Vec16<__nv_bfloat16>::unpack(ia.bv[g], b);
#pragma unroll
      for (int e = 0; e < 8; ++e) v[e] += b[e];
      Vec16<__nv_bfloat16>::unpack(ig.bv[g], b);
#pragma unroll
      for (int e = 0; e < 8; ++e) t[e] += b[e];
    }
#pragma unroll
    for (int e = 0; e < 8; ++e) v[e] *= gelu_tanh_fast(t[e]);
    *reinterpret_cast<uint4*>(out + g * 8) = Vec16<__nv_bfloat16>::pack(v);
  }
}

#ifdef FPS_GEMM_TRACE
// developer instrumentation (separate build, `make VARIANT=gtrace EXTRA=-DFPS_GEMM_TRACE`):
// %globaltimer stamps of every CTA of the last 1-SM GEMM launch -- entry, setup done, PDL wait
// done, first stage landed (MMA warp), last MMA of its first tile issued, its accumulator
// ready (epilogue warp 4), its epilogue done, exit
__device__ unsigned long long g_gemm_trace[160][8];
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define GEMM_TRACE(slot) g_gemm_trace[blockIdx.x < 160 ? blockIdx.x : 159][slot] = gtimer()
#else
#define GEMM_TRACE(slot) do {} while (0)
#endif

// Row-major tiles are written through a warp-private shared-memory transpose: the thread that
// owns a row (TMEM lane) leaves its 32 packed outputs there, then the warp stores 8 rows x 64 B
// per instruction (4 lanes per row segment) instead of 32 rows x 16 B -- whole, contiguous
// sectors.  Measured on B200 (tools/gemm_trace.py, one 128 x 256 tile per CTA, no fused ops):
// the epilogue took 8.5 us against 3.1 us of MMAs with per-row stores and the descriptor read
// from kernel parameters per chunk, 6.7 us with both changes (4916 x 640 x 640: 19.7 -> 13.9 us;
// 4916 x 5120 x 640: 63.3 -> 51.6 us); the SDXL block 0.279 -> 0.272 ms, the Flux-scale blocks
// and the C3 step unchanged within noise (tools/scripts/r02y_epi5.sh).  Handling 64 columns per
// iteration (two TMEM loads in flight) measured slower (254 registers).
// Layout: 32 rows x 64 B per warp; piece p (16 B) of row r at r * 64 + ((p ^ (r >> 1 & 3)) << 4)
// (conflict-free for both the row-per-lane writes and the 4-lanes-per-row reads).
constexpr int kXsWarpBytes = 32 * 64;

__device__ __forceinline__ uint32_t xs_off(int r, int p) { return r * 64 + ((p ^ ((r >> 1) & 3)) << 4); }

// Destination of output columns col0..col0+31 of the row (one column region: out0 / out1 /
// out2, as chunk_store decides per 8 columns); nullptr = nothing to store.
__device__ __forceinline__ __nv_bfloat16* chunk_dst(const Epilogue& ep, const RowCtx& rc, int N,
                                                    int col0) {
  if (!rc.ok || col0 >= N) return nullptr;
  if (col0 < ep.split)
    return reinterpret_cast<__nv_bfloat16*>(ep.out0) + (size_t)rc.orow0 * ep.ld0 + col0;
  if (ep.out2 && col0 >= ep.split2)
    return reinterpret_cast<__nv_bfloat16*>(ep.out2) + (size_t)rc.row * ep.ld2 + (col0 - ep.split2);
  return reinterpret_cast<__nv_bfloat16*>(ep.out1) + (size_t)rc.orow1 * ep.ld1 + (col0 - ep.split);
}

// Fused ops of 32 accumulator values (fp32 bits) of one row -> 4 x 8 packed bf16 (as chunk_store)
__device__ __forceinline__ void chunk_values(const Epilogue& ep, const RowCtx& rc, int col0,
                                             const uint32_t* r, const ChunkIn& in, uint4* out) {
#pragma unroll
  for (int g = 0; g < 4; ++g) {
    const int c0 = col0 + g * 8;
    float v[8], t[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) v[e] = __uint_as_float(r[g * 8 + e]);
    if (ep.bias) {
      Vec16<__nv_bfloat16>::unpack(in.bv[g], t);
#pragma unroll
      for (int e = 0; e < 8; ++e) v[e] += t[e];
    }
    if (ep.act == 1 && c0 >= ep.act_from) {
#pragma unroll
      for (int e = 0; e < 8; ++e) v[e] = gelu_tanh_fast(v[e]);
    }
    if (ep.resid) {
      float rr[8];
      if (ep.resid_f32) {
        Vec16<float>::unpack(in.rv[g], rr);
        Vec16<float>::unpack(in.rv[g + 4], rr + 4);
      } else {
        Vec16<__nv_bfloat16>::unpack(in.rv[g], rr);
      }
      if (rc.gate) {
        Vec16<__nv_bfloat16>::unpack(in.gv[g], t);
#pragma unroll
        for (int e = 0; e < 8; ++e) v[e] = rr[e] + t[e] * v[e];
      } else {
#pragma unroll
        for (int e = 0; e < 8; ++e) v[e] = rr[e] + v[e];
      }
    }
    out[g] = Vec16<__nv_bfloat16>::pack(v);
  }
}

// Epilogue of one accumulator tile for the calling thread's output row (thread = TMEM lane).
// xs: this warp's kXsWarpBytes of shared memory (transposed stores), or nullptr.
template <int BN>
__device__ __forceinline__ void epilogue_tile(const Epilogue& ep_param, int M, int N, int row,
                                              int col_base, uint32_t taddr, uint8_t* xs) {
  // one copy of the epilogue descriptor in registers per tile: the caller's `p ? ep1 : ep`
  // is an indexed kernel-parameter access, which re-read field by field (register-indexed
  // constant loads) cost ~300 cycles per 32-column chunk
  const Epilogue ep = ep_param;
  const RowCtx rc = row_ctx(ep, M, row);
  if (ep.act == 2) {
#pragma unroll 1
    for (int c = 0; c < BN / 64; ++c) {
      uint32_t ra[32], rg[32];
      tc::tmem_ld32(taddr + c * 64, ra);
      tc::tmem_ld32(taddr + c * 64 + 32, rg);
      const int col0 = col_base + c * 64;
      ChunkIn ia, ig;
      chunk_load(ep, rc, N, row, col0, ia);
      chunk_load(ep, rc, N, row, col0 + 32, ig);
      tc::tmem_wait_ld();
      geglu_store(ep, rc, N, col0, ra, rg, ia, ig);
    }
    return;
  }
  // the transposed path needs every 32-column chunk inside one output region and bf16 rows
  const bool staged = xs != nullptr && !ep.out0_f32 && (ep.split & 31) == 0 &&
                      (!ep.out2 || (ep.split2 & 31) == 0) && (ep.act != 1 || (ep.act_from & 31) == 0);
  const int lane = threadIdx.x & 31;
  const uint32_t xs_base = tc::smem_u32(xs);
  // bf16 residual rows read the same way: 8 rows x 64 B per warp instruction into the staging
  // buffer, then each thread takes its row (the per-row 16-B loads touched 32 lines per
  // instruction)
  const bool coop_resid = staged && ep.resid && !ep.resid_f32;
  const unsigned long long res_row =
      (coop_resid && rc.ok)
          ? reinterpret_cast<unsigned long long>(reinterpret_cast<const __nv_bfloat16*>(ep.resid) +
                                                 (size_t)rc.rrow * ep.ld_resid)
          : 0ull;
  // Whole 32-column chunks inside one output region (the common case) take a branch-light path:
  // the fused-op flags are tested once per chunk, not per 8 columns, and no operand is
  // zero-filled (the generic path below costs ~330 instructions per chunk, ~half of them guards)
  const bool aligned = (ep.split & 31) == 0 && (!ep.out2 || (ep.split2 & 31) == 0) &&
                       (ep.act != 1 || (ep.act_from & 31) == 0);
#pragma unroll 1
  for (int c = 0; c < BN / 32; ++c) {
    uint32_t r[32];
    tc::tmem_ld32(taddr + c * 32, r);
    const int col0 = col_base + c * 32;
    if (aligned && col0 + 32 <= N) {
      const bool f_bias = ep.bias != nullptr;
      const bool f_res = ep.resid != nullptr && rc.ok;
      const bool f_gate = rc.gate != nullptr;
      uint4 bv[4], gv[4], rv[8];
      if (f_bias) {
        const uint4* b = reinterpret_cast<const uint4*>(reinterpret_cast<const __nv_bfloat16*>(ep.bias) + col0);
#pragma unroll
        for (int g = 0; g < 4; ++g) bv[g] = __ldg(b + g);
      }
      if (f_gate) {
        const uint4* gp = reinterpret_cast<const uint4*>(rc.gate + col0);
#pragma unroll
        for (int g = 0; g < 4; ++g) gv[g] = __ldg(gp + g);
      }
      if (ep.resid_f32) {
        if (f_res) {
          const uint4* rp = reinterpret_cast<const uint4*>(reinterpret_cast<const float*>(ep.resid) +
                                                           (size_t)rc.rrow * ep.ld_resid + col0);
#pragma unroll
          for (int g = 0; g < 8; ++g) rv[g] = __ldg(rp + g);
        }
      } else if (coop_resid) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int rr = j * 8 + (lane >> 2), piece = lane & 3;
          const unsigned long long pr = __shfl_sync(0xffffffffu, res_row, rr);
          uint4 v = make_uint4(0, 0, 0, 0);
          if (pr) v = __ldg(reinterpret_cast<const uint4*>(reinterpret_cast<const char*>(pr) +
                                                           (size_t)col0 * 2 + piece * 16));
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(xs_base + xs_off(rr, piece)),
                       "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                       : "memory");
        }
        __syncwarp();
#pragma unroll
        for (int g = 0; g < 4; ++g)
          asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                       : "=r"(rv[g].x), "=r"(rv[g].y), "=r"(rv[g].z), "=r"(rv[g].w)
                       : "r"(xs_base + xs_off(lane, g))
                       : "memory");
        __syncwarp();
      } else if (f_res) {
        const uint4* rp = reinterpret_cast<const uint4*>(reinterpret_cast<const __nv_bfloat16*>(ep.resid) +
                                                         (size_t)rc.rrow * ep.ld_resid + col0);
#pragma unroll
        for (int g = 0; g < 4; ++g) rv[g] = __ldg(rp + g);
      }
      tc::tmem_wait_ld();
      float v[32];
#pragma unroll
      for (int e = 0; e < 32; ++e) v[e] = __uint_as_float(r[e]);
      if (f_bias) {
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          float t[8];
          Vec16<__nv_bfloat16>::unpack(bv[g], t);
#pragma unroll
          for (int e = 0; e < 8; ++e) v[g * 8 + e] += t[e];
        }
      }
      if (ep.act == 1 && col0 >= ep.act_from) {
#pragma unroll
        for (int e = 0; e < 32; ++e) v[e] = gelu_tanh_fast(v[e]);
      }
      if (f_res) {
        float rr[32];
        if (ep.resid_f32) {
#pragma unroll
          for (int g = 0; g < 8; ++g) Vec16<float>::unpack(rv[g], rr + g * 4);
        } else {
#pragma unroll
          for (int g = 0; g < 4; ++g) Vec16<__nv_bfloat16>::unpack(rv[g], rr + g * 8);
        }
        if (f_gate) {
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            float t[8];
            Vec16<__nv_bfloat16>::unpack(gv[g], t);
#pragma unroll
            for (int e = 0; e < 8; ++e) v[g * 8 + e] = rr[g * 8 + e] + t[e] * v[g * 8 + e];
          }
        } else {
#pragma unroll
          for (int e = 0; e < 32; ++e) v[e] += rr[e];
        }
      }
      if (ep.out0_f32 && col0 < ep.split) {                // fp32 rows: 128 B per row per chunk
        if (rc.ok) {
          uint4* df = reinterpret_cast<uint4*>(reinterpret_cast<float*>(ep.out0) +
                                               (size_t)rc.orow0 * ep.ld0 + col0);
#pragma unroll
          for (int g = 0; g < 8; ++g) df[g] = Vec16<float>::pack(v + g * 4);
        }
        continue;
      }
      uint4 pk[4];
#pragma unroll
      for (int g = 0; g < 4; ++g) pk[g] = Vec16<__nv_bfloat16>::pack(v + g * 8);
      __nv_bfloat16* const dst = chunk_dst(ep, rc, N, col0);
      if (!staged) {
        if (dst) {
#pragma unroll
          for (int g = 0; g < 4; ++g) reinterpret_cast<uint4*>(dst)[g] = pk[g];
        }
        continue;
      }
#pragma unroll
      for (int g = 0; g < 4; ++g)
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(xs_base + xs_off(lane, g)),
                     "r"(pk[g].x), "r"(pk[g].y), "r"(pk[g].z), "r"(pk[g].w)
                     : "memory");
      const unsigned long long dd = reinterpret_cast<unsigned long long>(dst);
      __syncwarp();
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int rr = j * 8 + (lane >> 2), piece = lane & 3;
        const unsigned long long p = __shfl_sync(0xffffffffu, dd, rr);
        if (p) {
          uint4 v4;
          asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                       : "=r"(v4.x), "=r"(v4.y), "=r"(v4.z), "=r"(v4.w)
                       : "r"(xs_base + xs_off(rr, piece))
                       : "memory");
          *reinterpret_cast<uint4*>(reinterpret_cast<char*>(p) + piece * 16) = v4;
        }
      }
      __syncwarp();
      continue;
    }
    ChunkIn in;
    chunk_load(ep, rc, N, row, col0, in, coop_resid);
    if (coop_resid) {
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int rr = j * 8 + (lane >> 2), piece = lane & 3;
        const unsigned long long p = __shfl_sync(0xffffffffu, res_row, rr);
        uint4 v = make_uint4(0, 0, 0, 0);
        if (p && col0 + piece * 8 < N)
          v = __ldg(reinterpret_cast<const uint4*>(reinterpret_cast<const char*>(p) +
                                                    (size_t)col0 * 2 + piece * 16));
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(xs_base + xs_off(rr, piece)),
                     "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                     : "memory");
      }
      __syncwarp();
#pragma unroll
      for (int g = 0; g < 4; ++g)
        asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(in.rv[g].x), "=r"(in.rv[g].y), "=r"(in.rv[g].z), "=r"(in.rv[g].w)
                     : "r"(xs_base + xs_off(lane, g))
                     : "memory");
      __syncwarp();
    }
    tc::tmem_wait_ld();
    if (!staged) {
      chunk_store(ep, rc, N, col0, r, in);
      continue;
    }
    uint4 pk[4];
    chunk_values(ep, rc, col0, r, in, pk);
#pragma unroll
    for (int g = 0; g < 4; ++g)
      asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(xs_base + xs_off(lane, g)),
                   "r"(pk[g].x), "r"(pk[g].y), "r"(pk[g].z), "r"(pk[g].w)
                   : "memory");
    const unsigned long long dst =
        reinterpret_cast<unsigned long long>(chunk_dst(ep, rc, N, col0));
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int rr = j * 8 + (lane >> 2), piece = lane & 3;
      const unsigned long long p = __shfl_sync(0xffffffffu, dst, rr);
      if (p && col0 + piece * 8 < N) {
        uint4 v;
        asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                     : "r"(xs_base + xs_off(rr, piece))
                     : "memory");
        *reinterpret_cast<uint4*>(reinterpret_cast<char*>(p) + piece * 16) = v;
      }
    }
    __syncwarp();
  }
}

// ============================================================================================
// 1-SM kernel
// EPI epilogue warps: 4 (thread = TMEM lane = output row, all BN columns) or 8 (two warps per
// TMEM lane quarter, BN / 2 columns each).  The epilogue of a 128-row tile is issue-bound in
// its warp (~330 instructions per 32-column chunk with the fused-op guards), so for short-K
// problems -- the SDXL-scale projections at K = 640, one tile per CTA -- it, not the MMAs, sets
// the CTA's time; two warps per quarter halve that chain.
template <int BN, int STAGES, int EPI = 8>
struct GemmCfg {
  static constexpr int BM = 128, BK = 64;
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int TMEM_COLS = 2 * BN;
  static constexpr int XS_BYTES = EPI * kXsWarpBytes;
  static constexpr int THREADS = 128 + 32 * EPI;
  static constexpr int SMEM = STAGES * STAGE_BYTES + XS_BYTES + 1024 + 256;
};



template <int BN, int STAGES, int EPI>
__global__ void __launch_bounds__(GemmCfg<BN, STAGES, EPI>::THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ CUtensorMap tmB1, int M, int N, int K, Epilogue ep,
                   int M1, Epilogue ep1, int N1) {
  using Cfg = GemmCfg<BN, STAGES, EPI>;
  constexpr int kGroupM = 16;                              // 2048 rows of A per group
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * Cfg::A_BYTES;
  uint8_t* sXs = smem + STAGES * Cfg::STAGE_BYTES;           // epilogue transpose staging
  uint64_t* full = reinterpret_cast<uint64_t*>(sXs + Cfg::XS_BYTES);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) GEMM_TRACE(0);
  const int num_m = (M + Cfg::BM - 1) / Cfg::BM;
  const int num_m1 = (M1 + Cfg::BM - 1) / Cfg::BM;
  const int num_n = (N + BN - 1) / BN;
  const int num_n1 = M1 > 0 ? (N1 + BN - 1) / BN : 0;
  const int T0 = num_m * num_n;
  const int num_tiles = T0 + num_m1 * num_n1;
  const int num_k = K / Cfg::BK;

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      tc::mbar_init(&full[s], 1);
      tc::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      tc::mbar_init(&tfull[a], 1);
      tc::mbar_init(&tempty[a], EPI);
    }
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmA);
    tc::tma_prefetch_desc(&tmB);
    if (M1 > 0) tc::tma_prefetch_desc(&tmB1);
  }
  if (warp == 2) tc::tmem_alloc<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem_base = *tmem_holder;
  if (threadIdx.x == 0) GEMM_TRACE(1);
  pdl_trigger();   // setup done: let the next kernel's CTAs start as ours retire
  pdl_wait();      // inputs of this GEMM come from the previous kernel
  if (threadIdx.x == 0) GEMM_TRACE(2);

  if (EPI == 8 && warp < 4) tc::regs_dec<72>();
  if (warp == 0) {
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
        int p, m_blk, n_blk;
        group_coords<kGroupM>(tile, T0, num_m, num_m1, num_n, num_n1, p, m_blk, n_blk);
        const CUtensorMap* tb = p ? &tmB1 : &tmB;
        const int arow = (p ? M : 0) + m_blk * Cfg::BM;
        for (int kb = 0; kb < num_k; ++kb) {
          tc::mbar_wait(&empty[stage], phase ^ 1);
          tc::mbar_expect_tx(&full[stage], Cfg::STAGE_BYTES);
          tc::tma_load_2d(sA + stage * Cfg::A_BYTES, &tmA, &full[stage], kb * Cfg::BK, arow);
          tc::tma_load_2d(sB + stage * Cfg::B_BYTES, tb, &full[stage], kb * Cfg::BK, n_blk * BN);
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      constexpr uint32_t idesc = tc::idesc_bf16(128, BN);
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, ++it) {
        const int acc = it & 1;
        tc::mbar_wait(&tempty[acc], ((it >> 1) & 1) ^ 1);
        tc::fence_after();
        const uint32_t d = tmem_base + acc * BN;
        for (int kb = 0; kb < num_k; ++kb) {
          tc::mbar_wait(&full[stage], phase);
          tc::fence_after();
          if (it == 0 && kb == 0) GEMM_TRACE(3);
          const uint32_t a0 = tc::smem_u32(sA + stage * Cfg::A_BYTES);
          const uint32_t b0 = tc::smem_u32(sB + stage * Cfg::B_BYTES);
#pragma unroll
          for (int k = 0; k < Cfg::BK / 16; ++k)
            tc::mma_bf16(d, tc::sdesc_k_sw128(a0 + k * 32), tc::sdesc_k_sw128(b0 + k * 32), idesc,
                         (kb | k) != 0);
          tc::mma_commit(&empty[stage]);
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        tc::mma_commit(&tfull[acc]);
        if (it == 0) GEMM_TRACE(4);
      }
    }
  } else if (warp >= 4) {
    if (EPI == 8) tc::regs_inc<216>();
    const int q = warp & 3;                                // TMEM lane quarter (warp id % 4)
    constexpr int CW = BN * 4 / EPI;                       // columns per epilogue warp
    const int h = (warp - 4) >> 2;                         // column part of this warp
    int it = 0;
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, ++it) {
      int p, m_blk, n_blk;
      group_coords<kGroupM>(tile, T0, num_m, num_m1, num_n, num_n1, p, m_blk, n_blk);
      const int acc = it & 1;
      tc::mbar_wait(&tfull[acc], (it >> 1) & 1);
      tc::fence_after();
      if (it == 0 && warp == 4 && lane == 0) GEMM_TRACE(5);
      epilogue_tile<CW>(p ? ep1 : ep, p ? M1 : M, p ? N1 : N, m_blk * Cfg::BM + q * 32 + lane,
                        n_blk * BN + h * CW,
                        tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + h * CW,
                        sXs + (warp - 4) * kXsWarpBytes);
      if (it == 0 && warp == 4 && lane == 0) GEMM_TRACE(6);
      tc::fence_before();
      __syncwarp();
      if (lane == 0) tc::mbar_arrive(&tempty[acc]);
    }
  }
  __syncwarp();     // each role warp reconverged (lane 0 ran the producer / MMA loop alone)
  __syncthreads();
  if (threadIdx.x == 0) GEMM_TRACE(7);
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc<Cfg::TMEM_COLS>(tmem_base);
  }
}

#ifdef FPS_GEMM_TRACE
}  // namespace fps
extern "C" int fps_debug_gemm_trace(unsigned long long* out) {
  return (int)cudaMemcpyFromSymbol(out, fps::g_gemm_trace, sizeof(fps::g_gemm_trace));
}

namespace fps {
#endif

// ============================================================================================
// CTA-pair kernel (cta_group::2): 256 x 256 tile per pair
// EPI epilogue warps per CTA: 4 or 8 (two per TMEM lane quarter, 128 columns each), as the
// 1-SM kernel; the epilogue of the last wave's tiles is exposed
template <int STAGES, int EPI = 4>
struct Gemm2Cfg {
  static constexpr int BM = 256, BN = 256, BK = 64;        // per pair
  static constexpr int A_BYTES = 128 * BK * 2;             // per CTA: its 128 rows of A
  static constexpr int B_BYTES = 128 * BK * 2;             // per CTA: its 128 rows of B
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int TMEM_COLS = 512;                    // 2 accumulators x 256 columns
  static constexpr int XS_BYTES = EPI * kXsWarpBytes;
  static constexpr int THREADS = 128 + 32 * EPI;
  static constexpr int SMEM = STAGES * STAGE_BYTES + XS_BYTES + 1024 + 256;
};

template <int STAGES, int EPI>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(Gemm2Cfg<STAGES, EPI>::THREADS, 1)
    gemm_tc2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                    const __grid_constant__ CUtensorMap tmB1, int M, int N, int K, Epilogue ep,
                    int M1, Epilogue ep1, int N1) {
  using Cfg = Gemm2Cfg<STAGES, EPI>;
  constexpr int kGroupM = 8;                               // 2048 rows of A per group
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * Cfg::A_BYTES;
  uint8_t* sXs = smem + STAGES * Cfg::STAGE_BYTES;           // epilogue transpose staging
  uint64_t* full = reinterpret_cast<uint64_t*>(sXs + Cfg::XS_BYTES);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = tc::cluster_ctarank();
  const int pair = blockIdx.x >> 1, num_pairs = gridDim.x >> 1;
  const int num_m = (M + Cfg::BM - 1) / Cfg::BM;
  const int num_m1 = (M1 + Cfg::BM - 1) / Cfg::BM;
  const int num_n = (N + Cfg::BN - 1) / Cfg::BN;
  const int num_n1 = M1 > 0 ? (N1 + Cfg::BN - 1) / Cfg::BN : 0;
  const int T0 = num_m * num_n;
  const int num_tiles = T0 + num_m1 * num_n1;
  const int num_k = K / Cfg::BK;

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      tc::mbar_init(&full[s], 1);                          // used in the leader only
      tc::mbar_init(&empty[s], 1);                         // both: leader's MMA commit multicasts
    }
    for (int a = 0; a < 2; ++a) {
      tc::mbar_init(&tfull[a], 1);                         // both: multicast commit
      tc::mbar_init(&tempty[a], 2 * EPI);                  // leader: EPI epilogue warps x 2 CTAs
    }
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmA);
    tc::tma_prefetch_desc(&tmB);
    if (M1 > 0) tc::tma_prefetch_desc(&tmB1);
  }
  if (warp == 2) tc::tmem_alloc_2sm<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::cluster_sync();                                      // peer barriers initialised
  tc::fence_after();
  const uint32_t tmem_base = *tmem_holder;
  pdl_trigger();   // setup done: let the next kernel's CTAs start as ours retire
  pdl_wait();      // inputs of this GEMM come from the previous kernel

  if (EPI == 8 && warp < 4) tc::regs_dec<72>();
  if (warp == 0) {
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      for (int tile = pair; tile < num_tiles; tile += num_pairs) {
        int p, m_blk, n_blk;
        group_coords<kGroupM>(tile, T0, num_m, num_m1, num_n, num_n1, p, m_blk, n_blk);
        const CUtensorMap* tb = p ? &tmB1 : &tmB;
        const int arow = (p ? M : 0) + m_blk * Cfg::BM + rank * 128;
        const int brow = n_blk * Cfg::BN + rank * 128;
        for (int kb = 0; kb < num_k; ++kb) {
          tc::mbar_wait(&empty[stage], phase ^ 1);
          if (rank == 0) tc::mbar_expect_tx(&full[stage], 2 * Cfg::STAGE_BYTES);
          tc::tma_load_2d_2sm(sA + stage * Cfg::A_BYTES, &tmA, &full[stage], kb * Cfg::BK, arow);
          tc::tma_load_2d_2sm(sB + stage * Cfg::B_BYTES, tb, &full[stage], kb * Cfg::BK, brow);
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {
      constexpr uint32_t idesc = tc::idesc_bf16(256, 256);
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int tile = pair; tile < num_tiles; tile += num_pairs, ++it) {
        const int acc = it & 1;
        tc::mbar_wait(&tempty[acc], ((it >> 1) & 1) ^ 1);
        tc::fence_after();
        const uint32_t d = tmem_base + acc * 256;
        for (int kb = 0; kb < num_k; ++kb) {
          tc::mbar_wait(&full[stage], phase);
          tc::fence_after();
          const uint32_t a0 = tc::smem_u32(sA + stage * Cfg::A_BYTES);
          const uint32_t b0 = tc::smem_u32(sB + stage * Cfg::B_BYTES);
#pragma unroll
          for (int k = 0; k < Cfg::BK / 16; ++k)
            tc::mma_bf16_2sm(d, tc::sdesc_k_sw128(a0 + k * 32), tc::sdesc_k_sw128(b0 + k * 32),
                             idesc, (kb | k) != 0);
          tc::mma_commit_2sm(&empty[stage]);
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        tc::mma_commit_2sm(&tfull[acc]);
      }
    }
  } else if (warp >= 4) {
    if (EPI == 8) tc::regs_inc<216>();
    const int q = warp & 3;
    constexpr int CW = 256 * 4 / EPI;                      // columns per epilogue warp
    const int h = (warp - 4) >> 2;
    const uint32_t tempty_leader = tc::mapa(tc::smem_u32(tempty), 0);
    int it = 0;
    for (int tile = pair; tile < num_tiles; tile += num_pairs, ++it) {
      int p, m_blk, n_blk;
      group_coords<kGroupM>(tile, T0, num_m, num_m1, num_n, num_n1, p, m_blk, n_blk);
      const int acc = it & 1;
      tc::mbar_wait(&tfull[acc], (it >> 1) & 1);
      tc::fence_after();
      epilogue_tile<CW>(p ? ep1 : ep, p ? M1 : M, p ? N1 : N,
                        m_blk * Cfg::BM + rank * 128 + q * 32 + lane, n_blk * Cfg::BN + h * CW,
                        tmem_base + ((uint32_t)(q * 32) << 16) + acc * 256 + h * CW,
                        sXs + (warp - 4) * kXsWarpBytes);
      tc::fence_before();
      __syncwarp();
      if (lane == 0) tc::mbar_arrive_cluster(tempty_leader + acc * 8);
    }
  }
  __syncthreads();
  tc::cluster_sync();                                      // both CTAs done with TMEM / barriers
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc_2sm<Cfg::TMEM_COLS>(tmem_base);
  }
}

// ============================================================================================
// CTA-pair kernel, operands swapped (C^T = B . A^T): the MMA's M=256 side walks the weight rows
// (N of the GEMM, a multiple of 256 at every block shape) and its N side walks the activation
// rows in blocks of NA (runtime, multiple of 16, <= 256).  For the active-row counts of masked
// blocks this removes the M padding of 256-row tiles (M = 1331: 6 x 224 = 1344 rows instead of
// 6 x 256 = 1536, -12.5% tensor work at the same number of waves).  Each CTA loads its 128
// weight rows and NA/2 activation rows per k-step; the accumulator holds D[n][m] (TMEM lane =
// output column), so the epilogue warps transpose 32 x 32 chunks through shared memory and then
// run the same per-row fused epilogue (thread = output row, 16-B stores) as the other kernels.
template <int STAGES>
struct Gemm2sCfg {
  static constexpr int BK = 64;
  static constexpr int A_BYTES = 128 * BK * 2;             // per CTA: 128 weight rows
  static constexpr int B_BYTES = 128 * BK * 2;             // per CTA: up to 128 activation rows
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int TMEM_COLS = 512;                    // 2 accumulators x up to 256 columns
  static constexpr int XPOSE_BYTES = 4 * 32 * 33 * 4;      // per epilogue warp: 32 x 33 floats
  static constexpr int SMEM = STAGES * STAGE_BYTES + XPOSE_BYTES + 1024 + 256;
};

template <int STAGES>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(256, 1)
    gemm_tc2s_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                     int M, int N, int K, int NA, Epilogue ep) {
  using Cfg = Gemm2sCfg<STAGES>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sW = smem;                                      // weight rows (MMA operand A)
  uint8_t* sX = smem + STAGES * Cfg::A_BYTES;              // activation rows (MMA operand B)
  float* sT = reinterpret_cast<float*>(smem + STAGES * Cfg::STAGE_BYTES);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * Cfg::STAGE_BYTES + Cfg::XPOSE_BYTES);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = tc::cluster_ctarank();
  const int pair = blockIdx.x >> 1, num_pairs = gridDim.x >> 1;
  const int num_m = (M + NA - 1) / NA;                     // activation blocks
  const int num_n = (N + 255) / 256;                       // weight blocks
  const int num_tiles = num_m * num_n;
  const int num_k = K / Cfg::BK;
  const int half = NA >> 1;

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      tc::mbar_init(&full[s], 1);
      tc::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      tc::mbar_init(&tfull[a], 1);
      tc::mbar_init(&tempty[a], 8);
    }
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmA);
    tc::tma_prefetch_desc(&tmB);
  }
  if (warp == 2) tc::tmem_alloc_2sm<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::cluster_sync();
  tc::fence_after();
  const uint32_t tmem_base = *tmem_holder;
  pdl_trigger();
  pdl_wait();

  // tile t: weight block t / num_m, activation block t % num_m -- the pairs running at the same
  // time share a few weight panels (read from HBM once) and all of A (L2-resident)
  if (warp == 0) {
    if (lane == 0) {
      const uint32_t bytes = 2 * (Cfg::A_BYTES + half * Cfg::BK * 2);
      int stage = 0;
      uint32_t phase = 0;
      for (int tile = pair; tile < num_tiles; tile += num_pairs) {
        const int n_blk = tile / num_m, m_blk = tile - n_blk * num_m;
        const int wrow = n_blk * 256 + rank * 128, xrow = m_blk * NA + rank * half;
        for (int kb = 0; kb < num_k; ++kb) {
          tc::mbar_wait(&empty[stage], phase ^ 1);
          if (rank == 0) tc::mbar_expect_tx(&full[stage], bytes);
          tc::tma_load_2d_2sm(sW + stage * Cfg::A_BYTES, &tmB, &full[stage], kb * Cfg::BK, wrow);
          tc::tma_load_2d_2sm(sX + stage * Cfg::B_BYTES, &tmA, &full[stage], kb * Cfg::BK, xrow);
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {
      const uint32_t idesc = tc::idesc_bf16(256, NA);
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int tile = pair; tile < num_tiles; tile += num_pairs, ++it) {
        const int acc = it & 1;
        tc::mbar_wait(&tempty[acc], ((it >> 1) & 1) ^ 1);
        tc::fence_after();
        const uint32_t d = tmem_base + acc * 256;
        for (int kb = 0; kb < num_k; ++kb) {
          tc::mbar_wait(&full[stage], phase);
          tc::fence_after();
          const uint32_t a0 = tc::smem_u32(sW + stage * Cfg::A_BYTES);
          const uint32_t b0 = tc::smem_u32(sX + stage * Cfg::B_BYTES);
#pragma unroll
          for (int k = 0; k < Cfg::BK / 16; ++k)
            tc::mma_bf16_2sm(d, tc::sdesc_k_sw128(a0 + k * 32), tc::sdesc_k_sw128(b0 + k * 32),
                             idesc, (kb | k) != 0);
          tc::mma_commit_2sm(&empty[stage]);
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        tc::mma_commit_2sm(&tfull[acc]);
      }
    }
  } else if (warp >= 4) {
    const int q = warp & 3;
    float* xt = sT + q * 32 * 33;
    const uint32_t tempty_leader = tc::mapa(tc::smem_u32(tempty), 0);
    int it = 0;
    for (int tile = pair; tile < num_tiles; tile += num_pairs, ++it) {
      const int n_blk = tile / num_m, m_blk = tile - n_blk * num_m;
      const int acc = it & 1;
      tc::mbar_wait(&tfull[acc], (it >> 1) & 1);
      tc::fence_after();
      // this warp's 32 output columns; TMEM column j of the tile = activation row m_blk*NA + j
      const int col0 = n_blk * 256 + rank * 128 + q * 32;
      const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + acc * 256;
      const int nchunk = NA >> 5, rem = NA & 31;
#pragma unroll 1
      for (int c = 0; c < nchunk + (rem ? 1 : 0); ++c) {
        uint32_t r[32];
        if (c < nchunk) {
          tc::tmem_ld32(taddr + c * 32, r);
        } else {                                           // NA % 32 == 16: last 16 columns
          tc::tmem_ld16(taddr + c * 32, r);
#pragma unroll
          for (int j = 16; j < 32; ++j) r[j] = 0u;
        }
        tc::tmem_wait_ld();
        // transpose: lane = column (col0 + lane), r[j] = row j  ->  lane = row, 32 columns
#pragma unroll
        for (int j = 0; j < 32; ++j) xt[j * 33 + lane] = __uint_as_float(r[j]);
        __syncwarp();
#pragma unroll
        for (int j = 0; j < 32; ++j) r[j] = __float_as_uint(xt[lane * 33 + j]);
        __syncwarp();
        const int row = m_blk * NA + c * 32 + lane;
        const RowCtx rc = row_ctx(ep, (c * 32 + lane < NA) ? M : 0, row);
        ChunkIn in;
        chunk_load(ep, rc, N, row, col0, in);
        chunk_store(ep, rc, N, col0, r, in);
      }
      tc::fence_before();
      __syncwarp();
      if (lane == 0) tc::mbar_arrive_cluster(tempty_leader + acc * 8);
    }
  }
  __syncthreads();
  tc::cluster_sync();
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc_2sm<Cfg::TMEM_COLS>(tmem_base);
  }
}

// ============================================================================================
bool gemm_tc_supported(int dtype, int M, int N, int K) {
  return dtype == FPS_BF16 && M > 0 && K >= 64 && K % 64 == 0 && N % 8 == 0;
}

int g_gemm_force = 0;   // tests: 1 = force the 1-SM kernel, 2 = force the CTA-pair kernel

// Optional second problem of a grouped launch (see group_coords): B1 [N1, K], M1 rows of A after
// the first M, its own epilogue.  M1 = 0: a plain GEMM.
struct Group2 {
  const void* B1;
  int M1;
  Epilogue ep1;
  int N1;
};

int g_gemm_epi4 = 0;    // tests / A-B: 1 = 4 epilogue warps instead of 8 (1-SM and pair kernels)

template <int BN, int STAGES, int EPI>
static fps_status launch_cfg_e(const void* A, const void* B, int M, int N, int K,
                               const Epilogue& ep, cudaStream_t s, const Group2& g2) {
  using Cfg = GemmCfg<BN, STAGES, EPI>;
  CUtensorMap ta, tb, tb1;
  if (!make_tmap_2d_bf16(&ta, A, M + g2.M1, K, (uint64_t)K * 2, Cfg::BK, Cfg::BM) ||
      !make_tmap_2d_bf16(&tb, B, N, K, (uint64_t)K * 2, Cfg::BK, BN) ||
      (g2.M1 > 0 && !make_tmap_2d_bf16(&tb1, g2.B1, g2.N1, K, (uint64_t)K * 2, Cfg::BK, BN)))
    return fail(FPS_ECUDA, "gemm_tc: cuTensorMapEncodeTiled failed (M=%d N=%d K=%d)", M, N, K);
  if (g2.M1 == 0) tb1 = tb;
  FPS_SMEM_ATTR((gemm_tc_kernel<BN, STAGES, EPI>), Cfg::SMEM);
  const int tiles = ceil_div(M, Cfg::BM) * ceil_div(N, BN) + ceil_div(g2.M1, Cfg::BM) * ceil_div(g2.N1, BN);
  const int grid = tiles < sm_budget() ? tiles : sm_budget();
  FPS_CUDA_TRY(launch_k(gemm_tc_kernel<BN, STAGES, EPI>, dim3(grid), dim3(Cfg::THREADS), Cfg::SMEM, s, ta, tb,
                        tb1, M, N, K, ep, g2.M1, g2.ep1, g2.N1));
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

template <int BN, int STAGES>
static fps_status launch_cfg(const void* A, const void* B, int M, int N, int K,
                             const Epilogue& ep, cudaStream_t s, const Group2& g2 = Group2{}) {
  if (g_gemm_epi4) return launch_cfg_e<BN, STAGES, 4>(A, B, M, N, K, ep, s, g2);
  return launch_cfg_e<BN, STAGES, 8>(A, B, M, N, K, ep, s, g2);
}

template <int STAGES, int EPI>
static fps_status launch_pair_e(const void* A, const void* B, int M, int N, int K,
                                const Epilogue& ep, cudaStream_t s, const Group2& g2) {
  using Cfg = Gemm2Cfg<STAGES, EPI>;
  CUtensorMap ta, tb, tb1;
  if (!make_tmap_2d_bf16(&ta, A, M + g2.M1, K, (uint64_t)K * 2, Cfg::BK, 128) ||
      !make_tmap_2d_bf16(&tb, B, N, K, (uint64_t)K * 2, Cfg::BK, 128) ||
      (g2.M1 > 0 && !make_tmap_2d_bf16(&tb1, g2.B1, g2.N1, K, (uint64_t)K * 2, Cfg::BK, 128)))
    return fail(FPS_ECUDA, "gemm_tc2: cuTensorMapEncodeTiled failed (M=%d N=%d K=%d)", M, N, K);
  if (g2.M1 == 0) tb1 = tb;
  FPS_SMEM_ATTR((gemm_tc2_kernel<STAGES, EPI>), Cfg::SMEM);
  const int tiles = ceil_div(M, Cfg::BM) * ceil_div(N, Cfg::BN) +
                    ceil_div(g2.M1, Cfg::BM) * ceil_div(g2.N1, Cfg::BN);
  const int pairs = tiles < sm_budget() / 2 ? tiles : sm_budget() / 2;
  FPS_CUDA_TRY(launch_k(gemm_tc2_kernel<STAGES, EPI>, dim3(2 * pairs), dim3(Cfg::THREADS), Cfg::SMEM,
                        s, ta, tb, tb1, M, N, K, ep, g2.M1, g2.ep1, g2.N1));
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

template <int STAGES>
static fps_status launch_pair(const void* A, const void* B, int M, int N, int K,
                              const Epilogue& ep, cudaStream_t s, const Group2& g2 = Group2{}) {
  if (g_gemm_epi4) return launch_pair_e<STAGES, 4>(A, B, M, N, K, ep, s, g2);
  return launch_pair_e<STAGES, 8>(A, B, M, N, K, ep, s, g2);
}

template <int STAGES>
static fps_status launch_pair_swap(const void* A, const void* B, int M, int N, int K, int NA,
                                   const Epilogue& ep, cudaStream_t s) {
  using Cfg = Gemm2sCfg<STAGES>;
  CUtensorMap ta, tb;
  if (!make_tmap_2d_bf16(&ta, A, M, K, (uint64_t)K * 2, Cfg::BK, NA / 2) ||
      !make_tmap_2d_bf16(&tb, B, N, K, (uint64_t)K * 2, Cfg::BK, 128))
    return fail(FPS_ECUDA, "gemm_tc2s: cuTensorMapEncodeTiled failed (M=%d N=%d K=%d)", M, N, K);
  FPS_SMEM_ATTR((gemm_tc2s_kernel<STAGES>), Cfg::SMEM);
  const int tiles = ceil_div(M, NA) * ceil_div(N, 256);
  const int pairs = tiles < sm_budget() / 2 ? tiles : sm_budget() / 2;
  FPS_CUDA_TRY(launch_k(gemm_tc2s_kernel<STAGES>, dim3(2 * pairs), dim3(256), Cfg::SMEM, s, ta,
                        tb, M, N, K, NA, ep));
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

int g_gemm_bn = 0;      // tests / A-B: 1 = force the 1-SM kernel's 128-column tile, 2 = 256

// 1-SM tile width: the wave model's per-SM tensor time (waves x BN), ties to the 256 tile.
// An epilogue-aware tie-break (the 128 tile's last epilogue is half as long) measured worse
// where it changed the choice: 4916 x 640 x 2560 29.4 vs 20.5 us, 4916 x 640 x 640 11.7 vs
// 11.0 us (tools/gemm_probe.py, flag bits 13-14) -- with twice the tiles the 128 tile reads the
// activation panel twice as often and the short-K problems are L2-bound at one wave.
static bool prefer_bn256(long c256, long c128, int) {
  if (g_gemm_bn) return g_gemm_bn == 2;
  return c256 <= c128;
}

// Activation-block height for the swapped pair kernel: minimise waves x NA (per-SM tensor work
// of the critical path), ties to the larger NA (fewer tiles, fewer epilogue passes).
static int swap_block(int M, int N, long* cost) {
  int best = 256;
  long bc = -1;
  for (int na = 256; na >= 64; na -= 16) {
    const long tiles = (long)ceil_div(M, na) * ceil_div(N, 256);
    const long c = ((tiles + sm_budget() / 2 - 1) / (sm_budget() / 2)) * na;
    if (bc < 0 || c < bc) {
      bc = c;
      best = na;
    }
  }
  *cost = bc;
  return best;
}

// Grouped pair of GEMMs in one launch (double-stream block: image rows on the image weights,
// text rows on the text weights): both problems' tiles share the persistent grid, so the two
// small problems fill the machine like one of their combined size.  Kernel choice as for one
// GEMM with the combined tile counts.
fps_status launch_gemm_tc_grouped(const void* A, const void* B0, const void* B1, int M0, int M1,
                                  int N, int K, const Epilogue& ep0, const Epilogue& ep1,
                                  cudaStream_t s, int N1) {
  if (!aligned16(A) || !aligned16(B0) || !aligned16(B1))
    return fail(FPS_EINVAL, "gemm_tc: unaligned operand");
  if (N1 <= 0) N1 = N;
  if (N1 % 8 != 0) return fail(FPS_EINVAL, "gemm_tc: N1 %% 8 != 0");
  const Group2 g2{B1, M1, ep1, N1};
  // tile counts of both problems (problem 1 has N1 columns)
  const long t256 = (long)ceil_div(M0, 128) * ceil_div(N, 256) + (long)ceil_div(M1, 128) * ceil_div(N1, 256);
  const long t128 = (long)ceil_div(M0, 128) * ceil_div(N, 128) + (long)ceil_div(M1, 128) * ceil_div(N1, 128);
  const long tp = (long)ceil_div(M0, 256) * ceil_div(N, 256) + (long)ceil_div(M1, 256) * ceil_div(N1, 256);
  const long c256 = ((t256 + sm_budget() - 1) / sm_budget()) * 256;
  const long c128 = ((t128 + sm_budget() - 1) / sm_budget()) * 128;
  const long cp = ((tp + sm_budget() / 2 - 1) / (sm_budget() / 2)) * 256;
  const long cmin = std::min(c256, c128);
  const long pair_multi = g_sm_reserved > 0 ? 2L * (sm_budget() / 2) : sm_budget() / 2;
  // a tie in the wave model goes to the pair kernel (FPS_GROUPED_TIE overrides: 0 never, 1 at
  // K >= 8192, 2 always): the double-stream block's O and down projections at C3's masked size
  // (819 image + 512 text rows, 72 pair tiles) run one pair wave instead of 132 1-SM tiles --
  // Y-mode C3 step 27.40 -> 27.03 ms (mean of 2 runs each, profiles/r02/grouped_tie.txt)
  static const int tie = [] {
    const char* v = getenv("FPS_GROUPED_TIE");
    return v ? atoi(v) : 2;
  }();
  const bool pair_wins = (tp > pair_multi && K >= 1024) || cp < cmin ||
                         (cp == cmin && (tie == 2 || (tie == 1 && K >= 8192)));
  if (g_gemm_force == 2 || (g_gemm_force != 1 && pair_wins))
    return launch_pair<6>(A, B0, M0, N, K, ep0, s, g2);
  if (prefer_bn256(c256, c128, K)) return launch_cfg<256, 4>(A, B0, M0, N, K, ep0, s, g2);
  return launch_cfg<128, 6>(A, B0, M0, N, K, ep0, s, g2);
}

fps_status launch_gemm_tc(const void* A, const void* B, int M, int N, int K, const Epilogue& ep,
                          cudaStream_t s) {
  if (!aligned16(A) || !aligned16(B)) return fail(FPS_EINVAL, "gemm_tc: unaligned operand");
  // Cost model: time ~ waves x tile work; the pair kernel's 256x256 tile does 2x the work of a
  // 128x256 tile on two SMs, i.e. the same per-SM time per wave, but at half the operand traffic
  // per FLOP.  Prefer it unless it needs more waves.
  const int m1 = ceil_div(M, 128), m2 = ceil_div(M, 256);
  const long t256 = (long)m1 * ceil_div(N, 256), t128 = (long)m1 * ceil_div(N, 128);
  const long tp = (long)m2 * ceil_div(N, 256);
  const long c256 = ((t256 + sm_budget() - 1) / sm_budget()) * 256;
  const long c128 = ((t128 + sm_budget() - 1) / sm_budget()) * 128;
  const long cp = ((tp + sm_budget() / 2 - 1) / (sm_budget() / 2)) * 256;
  // Measured (tools/gemm_probe.py, B200): the pair kernel reaches 95% tensor-pipe activity at
  // large M where the 1-SM kernel is L2-bound (1480 vs 1070 TFLOP/s at M = 29491); at one wave
  // the extra M padding of 256-row tiles can make it lose, so then padding decides.
  const long cmin = std::min(c256, c128);
  // multi-wave problems: the pair kernel (lower L2 traffic per FLOP) regardless of the small
  // quantisation differences the wave model sees; one wave: the wave model and M padding decide
  // (one wave, long K: the pair's deeper ring wins -- 80.5 vs 83.3 us at 1331x3072x12288;
  //  short K: its longer prologue / epilogue lose -- 27.3 vs 23.2 us at 1331x3072x3072)
  // short K (< 1024, the SDXL-scale projections at C = 640): the pair's longer prologue and
  // epilogue are not amortised even over several waves (4916x1920x640: 30.2 vs 23.3 us for the
  // 1-SM kernel; 4916x5120x640: 54.8 vs 52.9; 16384x1920x640: 64.7 vs 61.3; K >= 1280: ties)
  // with SMs reserved for the method-3 gather (sm_budget() < 148) a problem just over one pair
  // wave (C3's W2: 72 pair tiles on 70 pairs) would take two; there the pair kernel's L2
  // advantage must span at least two full waves to outweigh the wave model
  const long pair_multi = g_sm_reserved > 0 ? 2L * (sm_budget() / 2) : sm_budget() / 2;
  const bool pair_wins = (tp > pair_multi && K >= 1024) || cp < cmin ||
                         (cp == cmin && (m2 * 256 - M < 128 || K >= 8192));
  // swapped operands (activation rows on the MMA's N side, no 256-row M padding): correct and
  // tested, but measured no faster at the masked-block shapes (1331x9216x3072: 59.8 vs 59.2 us
  // for the pair kernel -- under the power cap the MMAs on TMA zero-fill rows cost little) and
  // slow for small activation blocks (NA = 144: 3.6x), so it is only selectable by force
  if (g_gemm_force == 3 && ep.act != 2) {
    long cs = 0;
    return launch_pair_swap<6>(A, B, M, N, K, swap_block(M, N, &cs), ep, s);
  }
  if (g_gemm_force == 2 || (g_gemm_force == 0 && pair_wins))
    return launch_pair<6>(A, B, M, N, K, ep, s);
  if (prefer_bn256(c256, c128, K)) return launch_cfg<256, 4>(A, B, M, N, K, ep, s);
  return launch_cfg<128, 6>(A, B, M, N, K, ep, s);
}

}  // namespace fps
