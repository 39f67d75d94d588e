// a6: masked-query attention over the merged (fresh + cached) key set, tcgen05 + TMEM + TMA.
// PAPER.md L146 (QK^T and softmax are the only inter-token op), L159 ("the Q matrix of only the
// new tokens along with the K and V matrices of all present tokens"), L161 (K/V variant).
//
// One CTA per (request, 128-query tile, head); varlen: the tile -> request map is decoded from
// cu_q in-kernel, keys are the request's rows [cu_k[r], cu_k[r+1]) of the merged buffer.
//   warp 0     TMA: Q tile once; K and V tiles (128 keys x d) through a 2-stage ring
//   warp 1     MMA: S_j = Q K_j^T into one of two TMEM S buffers (issued one tile ahead), then
//              O += P_j V_j with V as an MN-major operand; commits free the K/V stage
//   warps 4-7  softmax, thread = query row: S row from TMEM (tcgen05.ld), online softmax in the
//              exp2 domain with a lazy max (O in TMEM is rescaled only when the running max grows
//              by more than 2^8, FA4-style), P as bf16 into one of two smem P buffers in the UMMA
//              K-major SW128 layout; the exponentials of tile j are computed while PV_{j-1} still
//              runs; final O / l from TMEM to global.
#include <algorithm>

#include "kernels.h"
#include "tc_util.cuh"

namespace fps {

template <int D>
struct AttnCfg {
  static constexpr int BM = 128, BN = 128, STAGES = 2;
  static constexpr int CH = D / 64;                        // 64-wide (128 B) chunks along d
  static constexpr int Q_BYTES = BM * D * 2;
  static constexpr int KV_TILE = BN * D * 2;
  static constexpr int P_BYTES = BM * BN * 2;              // one P tile; two are kept
  static constexpr int SMEM = Q_BYTES + STAGES * 2 * KV_TILE + 2 * P_BYTES + 1024 + 256;
  static constexpr int TMEM_COLS = 512;                    // S0 [0,128) S1 [128,256) O [256,256+D)
};

template <int D>
__global__ void __launch_bounds__(256, 1)
    attn_tc_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmKV,
                   __nv_bfloat16* __restrict__ O, const int32_t* __restrict__ cu_q,
                   const int32_t* __restrict__ cu_k, int n_req, int heads, float scale_log2, int ldo) {
  using Cfg = AttnCfg<D>;
  constexpr int CHUNK = 128 * 128;                         // bytes of one [128 rows x 128 B] chunk
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + Cfg::Q_BYTES;                          // [stage][CH chunks]
  uint8_t* sV = sK + Cfg::STAGES * Cfg::KV_TILE;
  uint8_t* sP = sV + Cfg::STAGES * Cfg::KV_TILE;            // [2 buffers][2 chunks of 64 keys]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sP + 2 * Cfg::P_BYTES);
  uint64_t* bar_q = bars;
  uint64_t* k_full = bars + 1;                              // K and V rings are separate so
  uint64_t* k_empty = bars + 3;                             // K_j+2 loads as soon as S_j is
  uint64_t* bar_s = bars + 5;                               // done, long before PV_j frees V
  uint64_t* bar_p = bars + 7;                               // [2]: P_j written (buffer j % 2)
  uint64_t* bar_o = bars + 9;                               // [2]: PV_j done (buffer j % 2)
  uint64_t* v_full = bars + 11;
  uint64_t* v_empty = bars + 13;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + 15);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int head = blockIdx.y;
  const int H = heads * D;
  // decode (request, q tile) of this CTA
  int r = 0, qt = blockIdx.x;
  for (; r < n_req; ++r) {
    const int nt = (__ldg(cu_q + r + 1) - __ldg(cu_q + r) + 127) >> 7;
    if (qt < nt) break;
    qt -= nt;
  }
  const int q0 = __ldg(cu_q + r) + qt * 128;
  const int n_rows = min(128, __ldg(cu_q + r + 1) - q0);
  const int Lr = __ldg(cu_k + r + 1) - __ldg(cu_k + r);
  const int nk_all = (Lr + 127) >> 7;
  const int nsplit = gridDim.z, split = blockIdx.z;
  const int kb = (int)(((long long)nk_all * split) / nsplit);       // first key tile of this CTA
  const int nk = (int)(((long long)nk_all * (split + 1)) / nsplit) - kb;
  const int k0 = __ldg(cu_k + r) + kb * 128;                         // its first key row
  const int Lr_rem = Lr - kb * 128;                                  // keys from k0 to the end

  if (threadIdx.x == 0) {
    tc::mbar_init(bar_q, 1);
    for (int s = 0; s < 2; ++s) {
      tc::mbar_init(&k_full[s], 1);
      tc::mbar_init(&k_empty[s], 1);
      tc::mbar_init(&v_full[s], 1);
      tc::mbar_init(&v_empty[s], 1);
      tc::mbar_init(&bar_s[s], 1);
      tc::mbar_init(&bar_p[s], 4);
      tc::mbar_init(&bar_o[s], 1);
    }
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmQ);
    tc::tma_prefetch_desc(&tmKV);
  }
  if (warp == 2) tc::tmem_alloc<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = *tmem_holder;
  pdl_trigger();
  pdl_wait();
  const uint32_t tS = tmem, tO = tmem + 256;

  if (warp == 0) {
    if (lane == 0 && nk > 0) {
      tc::mbar_expect_tx(bar_q, Cfg::Q_BYTES);
#pragma unroll
      for (int c = 0; c < Cfg::CH; ++c)
        tc::tma_load_2d(sQ + c * CHUNK, &tmQ, bar_q, head * D + c * 64, q0);
      for (int kt = 0; kt < nk; ++kt) {
        const int st = kt & 1;
        tc::mbar_wait_sleep(&k_empty[st], ((kt >> 1) & 1) ^ 1);
        tc::mbar_expect_tx(&k_full[st], Cfg::KV_TILE);
#pragma unroll
        for (int c = 0; c < Cfg::CH; ++c)
          tc::tma_load_2d(sK + st * Cfg::KV_TILE + c * CHUNK, &tmKV, &k_full[st],
                          head * D + c * 64, k0 + kt * 128);
      }
    }
  } else if (warp == 3) {
    if (lane == 0) {
      for (int kt = 0; kt < nk; ++kt) {
        const int st = kt & 1;
        tc::mbar_wait_sleep(&v_empty[st], ((kt >> 1) & 1) ^ 1);
        tc::mbar_expect_tx(&v_full[st], Cfg::KV_TILE);
#pragma unroll
        for (int c = 0; c < Cfg::CH; ++c)
          tc::tma_load_2d(sV + st * Cfg::KV_TILE + c * CHUNK, &tmKV, &v_full[st],
                          H + head * D + c * 64, k0 + kt * 128);
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && nk > 0) {
      constexpr uint32_t idesc_s = tc::idesc_bf16(128, 128);
      constexpr uint32_t idesc_o = tc::idesc_bf16(128, D, /*b_mn_major=*/true);
      tc::mbar_wait_sleep(bar_q, 0);
      auto issue_s = [&](int kt) {
        const int st = kt & 1;
        tc::mbar_wait_sleep(&k_full[st], (kt >> 1) & 1);
        tc::fence_after();
        const uint32_t qa = tc::smem_u32(sQ), kb = tc::smem_u32(sK + st * Cfg::KV_TILE);
#pragma unroll
        for (int ks = 0; ks < D / 16; ++ks) {
          const uint32_t off = (ks >> 2) * CHUNK + (ks & 3) * 32;
          tc::mma_bf16(tS + st * 128, tc::sdesc_k_sw128(qa + off), tc::sdesc_k_sw128(kb + off),
                       idesc_s, ks > 0);
        }
        tc::mma_commit(&bar_s[st]);
        tc::mma_commit(&k_empty[st]);
      };
      issue_s(0);
      for (int kt = 0; kt < nk; ++kt) {
        // S buffer (kt+1)&1 was released by the softmax of tile kt-1 (bar_p waited below)
        if (kt + 1 < nk) issue_s(kt + 1);
        const int pb = kt & 1;
        tc::mbar_wait_sleep(&bar_p[pb], (kt >> 1) & 1);
        tc::fence_after();
        const int st = kt & 1;
        tc::mbar_wait_sleep(&v_full[st], (kt >> 1) & 1);
        tc::fence_after();
        const uint32_t pa = tc::smem_u32(sP + pb * Cfg::P_BYTES);
        const uint32_t vb = tc::smem_u32(sV + st * Cfg::KV_TILE);
#pragma unroll
        for (int ks = 0; ks < 8; ++ks) {
          tc::mma_bf16(tO, tc::sdesc_k_sw128(pa + (ks >> 2) * CHUNK + (ks & 3) * 32),
                       tc::sdesc_mn_sw128(vb + ks * 2048, CHUNK), idesc_o, (kt | ks) != 0);
        }
        tc::mma_commit(&bar_o[pb]);
        tc::mma_commit(&v_empty[st]);
      }
    }
  } else if (warp >= 4) {
    const int q = warp & 3;
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    float m_used = -INFINITY, l = 0.f;                      // m_used in the scaled log2 domain
    const int sw = row & 7;
    for (int kt = 0; kt < nk; ++kt) {
      const int st = kt & 1;
      tc::mbar_wait(&bar_s[st], (kt >> 1) & 1);
      tc::fence_after();
      float s[128];
#pragma unroll
      for (int c = 0; c < 4; ++c)
        tc::tmem_ld32(tS + lane_off + st * 128 + c * 32, reinterpret_cast<uint32_t*>(s + c * 32));
      tc::tmem_wait_ld();
      const int valid = Lr - kt * 128;                    // keys of this request in the tile
      if (valid < 128) {
#pragma unroll
        for (int i = 0; i < 128; ++i) s[i] = (i < valid) ? s[i] : -INFINITY;
      }
      // row max as 8 independent chains (latency 16 + 3 steps instead of 127)
      float m8[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) m8[j] = s[j];
#pragma unroll
      for (int i = 8; i < 128; ++i) m8[i & 7] = fmaxf(m8[i & 7], s[i]);
#pragma unroll
      for (int j = 0; j < 4; ++j) m8[j] = fmaxf(m8[j], m8[j + 4]);
      float mx = fmaxf(fmaxf(m8[0], m8[1]), fmaxf(m8[2], m8[3])) * scale_log2;
      const bool need = mx > m_used + 8.0f;
      const bool any_need = __any_sync(0xffffffffu, need);
      float factor = 1.0f;
      if (need) {
        factor = tc::ex2(m_used - mx);                    // ex2(-inf) = 0 on the first tile
        l *= factor;
        m_used = mx;
      }
      // p = 2^(s*scale - m) while PV_{kt-1} may still be running; packed FFMA2 for the
      // scale-and-shift, packed FADD2 into 8 independent partial sums
      const float nm = -m_used;
      float a8[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
      for (int i = 0; i < 128; i += 2) {
        tc::ffma2(s[i], s[i + 1], s[i], s[i + 1], scale_log2, scale_log2, nm, nm);
        if (((i >> 3) & 3) == 3) {                         // 1/4 of the exponentials on the FMA pipe
          tc::ex2_poly2(s[i], s[i + 1]);
        } else {                                           // 3/4 on the MUFU unit
          s[i] = tc::ex2(s[i]);
          s[i + 1] = tc::ex2(s[i + 1]);
        }
        const int j = (i >> 1) & 3;
        tc::fadd2(a8[2 * j], a8[2 * j + 1], a8[2 * j], a8[2 * j + 1], s[i], s[i + 1]);
      }
      l += ((a8[0] + a8[1]) + (a8[2] + a8[3])) + ((a8[4] + a8[5]) + (a8[6] + a8[7]));
      if (any_need && kt > 0) {
        // O += P_{kt-1} V_{kt-1} must land before O is rescaled (rare: max grew by > 2^8)
        tc::mbar_wait(&bar_o[(kt - 1) & 1], ((kt - 1) >> 1) & 1);
        tc::fence_after();
#pragma unroll 1
        for (int c = 0; c < D / 32; ++c) {
          uint32_t o[32];
          tc::tmem_ld32(tO + lane_off + c * 32, o);
          tc::tmem_wait_ld();
#pragma unroll
          for (int e = 0; e < 32; ++e) o[e] = __float_as_uint(__uint_as_float(o[e]) * factor);
          tc::tmem_st32(tO + lane_off + c * 32, o);
        }
        tc::tmem_wait_st();
      }
      // P buffer kt&1 was last read by PV_{kt-2}
      const int pb = kt & 1;
      if (kt >= 2) {
        tc::mbar_wait(&bar_o[pb], ((kt - 2) >> 1) & 1);
        tc::fence_after();
      }
      uint8_t* prow = sP + pb * Cfg::P_BYTES + row * 128;
#pragma unroll
      for (int u = 0; u < 16; ++u) {
        const uint4 v = make_uint4(pack_bf16x2(s[u * 8 + 0], s[u * 8 + 1]),
                                   pack_bf16x2(s[u * 8 + 2], s[u * 8 + 3]),
                                   pack_bf16x2(s[u * 8 + 4], s[u * 8 + 5]),
                                   pack_bf16x2(s[u * 8 + 6], s[u * 8 + 7]));
        const int chunk = u >> 3, unit = u & 7;
        *reinterpret_cast<uint4*>(prow + chunk * CHUNK + ((unit ^ sw) << 4)) = v;
      }
      tc::fence_proxy_async_smem();
      tc::fence_before();
      __syncwarp();
      if (lane == 0) tc::mbar_arrive(&bar_p[pb]);
    }
    if (nk > 0) {
      tc::mbar_wait(&bar_o[(nk - 1) & 1], ((nk - 1) >> 1) & 1);
      tc::fence_after();
    }
    const float inv = (l > 0.f) ? 1.0f / l : 0.f;
    __nv_bfloat16* orow = O + (size_t)(q0 + row) * ldo + head * D;
#pragma unroll 1
    for (int c = 0; c < D / 32; ++c) {
      uint32_t o[32];
      tc::tmem_ld32(tO + lane_off + c * 32, o);
      tc::tmem_wait_ld();
      if (row < n_rows) {
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          float f[8];
#pragma unroll
          for (int e = 0; e < 8; ++e) f[e] = __uint_as_float(o[g * 8 + e]) * inv;
          *reinterpret_cast<uint4*>(orow + c * 32 + g * 8) = Vec16<__nv_bfloat16>::pack(f);
        }
      }
    }
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

// ============================================================================================
// Two query tiles per CTA (A = rows q0..q0+127, B = the next 128), FA4-style ping-pong: the
// tensor core alternates between the tiles (S_A, S_B, PV_A, S_A', PV_B, S_B', ...) while two
// softmax warpgroups (warps 4-7 for A, 8-11 for B) work on the other tile, so MUFU/issue time of
// one warpgroup hides behind MMAs of the other.  Every K/V tile feeds four MMAs (half the smem
// traffic per FLOP), and a CTA covers 256 query rows (e.g. 6 x 24 = 144 CTAs for n = 1331: one
// wave).  TMEM: S_A [0,128) S_B [128,256) O_A [256,256+D) O_B [384,384+D); one shared smem P tile
// is written alternately by the two warpgroups.  S rows are read from TMEM in two 64-column
// halves (max pass, then exp pass) to stay within 168 registers at 384 threads.
template <int D>
struct Attn2Cfg {
  static constexpr int CH = D / 64;
  static constexpr int Q_BYTES = 128 * D * 2;              // one query tile
  static constexpr int KV_TILE = 128 * D * 2;
  static constexpr int P_BYTES = 128 * 128 * 2;
  static constexpr int SMEM = 2 * Q_BYTES + 4 * KV_TILE + P_BYTES + 1024 + 256;
  static constexpr int TMEM_COLS = 512;
};

template <int D>
__global__ void __launch_bounds__(384, 1)
    attn_tc2_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmKV,
                    __nv_bfloat16* __restrict__ O, const int32_t* __restrict__ cu_q,
                    const int32_t* __restrict__ cu_k, int n_req, int heads, float scale_log2, int ldo) {
  using Cfg = Attn2Cfg<D>;
  constexpr int CHUNK = 128 * 128;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sQ = smem;                                       // [2 tiles][CH chunks]
  uint8_t* sK = sQ + 2 * Cfg::Q_BYTES;                      // [2 stages][CH chunks]
  uint8_t* sV = sK + 2 * Cfg::KV_TILE;
  uint8_t* sP = sV + 2 * Cfg::KV_TILE;                      // [2 chunks of 64 keys]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sP + Cfg::P_BYTES);
  uint64_t* bar_q = bars;
  uint64_t* k_full = bars + 1;
  uint64_t* k_empty = bars + 3;
  uint64_t* v_full = bars + 5;
  uint64_t* v_empty = bars + 7;
  uint64_t* bar_s = bars + 9;                               // [tile]
  uint64_t* bar_p = bars + 11;                              // [tile]
  uint64_t* bar_o = bars + 13;                              // [tile]
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + 15);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int head = blockIdx.y;
  const int H = heads * D;
  int r = 0, qp = blockIdx.x, ntile = 0;
  for (; r < n_req; ++r) {
    ntile = (__ldg(cu_q + r + 1) - __ldg(cu_q + r) + 127) >> 7;
    const int np = (ntile + 1) >> 1;
    if (qp < np) break;
    qp -= np;
  }
  const bool hasB = 2 * qp + 1 < ntile;
  const int q_end = __ldg(cu_q + r + 1);
  const int q0 = __ldg(cu_q + r) + qp * 256;
  const int Lr = __ldg(cu_k + r + 1) - __ldg(cu_k + r);
  const int nk_all = (Lr + 127) >> 7;
  const int nsplit = gridDim.z, split = blockIdx.z;
  const int kb = (int)(((long long)nk_all * split) / nsplit);       // first key tile of this CTA
  const int nk = (int)(((long long)nk_all * (split + 1)) / nsplit) - kb;
  const int k0 = __ldg(cu_k + r) + kb * 128;                         // its first key row
  const int Lr_rem = Lr - kb * 128;                                  // keys from k0 to the end

  if (threadIdx.x == 0) {
    tc::mbar_init(bar_q, 1);
    for (int s = 0; s < 2; ++s) {
      tc::mbar_init(&k_full[s], 1);
      tc::mbar_init(&k_empty[s], 1);
      tc::mbar_init(&v_full[s], 1);
      tc::mbar_init(&v_empty[s], 1);
      tc::mbar_init(&bar_s[s], 1);
      tc::mbar_init(&bar_p[s], 4);
      tc::mbar_init(&bar_o[s], 1);
    }
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmQ);
    tc::tma_prefetch_desc(&tmKV);
  }
  if (warp == 2) tc::tmem_alloc<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = *tmem_holder;
  pdl_trigger();
  pdl_wait();

  if (warp == 0) {
    if (lane == 0 && nk > 0) {
      tc::mbar_expect_tx(bar_q, (hasB ? 2 : 1) * Cfg::Q_BYTES);
      for (int t = 0; t < (hasB ? 2 : 1); ++t)
#pragma unroll
        for (int c = 0; c < Cfg::CH; ++c)
          tc::tma_load_2d(sQ + t * Cfg::Q_BYTES + c * CHUNK, &tmQ, bar_q, head * D + c * 64,
                          q0 + t * 128);
      for (int kt = 0; kt < nk; ++kt) {
        const int st = kt & 1;
        tc::mbar_wait_sleep(&k_empty[st], ((kt >> 1) & 1) ^ 1);
        tc::mbar_expect_tx(&k_full[st], Cfg::KV_TILE);
#pragma unroll
        for (int c = 0; c < Cfg::CH; ++c)
          tc::tma_load_2d(sK + st * Cfg::KV_TILE + c * CHUNK, &tmKV, &k_full[st],
                          head * D + c * 64, k0 + kt * 128);
      }
    }
  } else if (warp == 3) {
    if (lane == 0) {
      for (int kt = 0; kt < nk; ++kt) {
        const int st = kt & 1;
        tc::mbar_wait_sleep(&v_empty[st], ((kt >> 1) & 1) ^ 1);
        tc::mbar_expect_tx(&v_full[st], Cfg::KV_TILE);
#pragma unroll
        for (int c = 0; c < Cfg::CH; ++c)
          tc::tma_load_2d(sV + st * Cfg::KV_TILE + c * CHUNK, &tmKV, &v_full[st],
                          H + head * D + c * 64, k0 + kt * 128);
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && nk > 0) {
      constexpr uint32_t idesc_s = tc::idesc_bf16(128, 128);
      constexpr uint32_t idesc_o = tc::idesc_bf16(128, D, /*b_mn_major=*/true);
      tc::mbar_wait_sleep(bar_q, 0);
      auto issue_s = [&](int t, int kt) {           // S_t = Q_t K_kt^T  (K stage must be full)
        const uint32_t qa = tc::smem_u32(sQ + t * Cfg::Q_BYTES);
        const uint32_t kb = tc::smem_u32(sK + (kt & 1) * Cfg::KV_TILE);
#pragma unroll
        for (int ks = 0; ks < D / 16; ++ks) {
          const uint32_t off = (ks >> 2) * CHUNK + (ks & 3) * 32;
          tc::mma_bf16(tmem + t * 128, tc::sdesc_k_sw128(qa + off), tc::sdesc_k_sw128(kb + off),
                       idesc_s, ks > 0);
        }
        tc::mma_commit(&bar_s[t]);
      };
      auto issue_pv = [&](int t, int kt) {          // O_t += P V_kt  (P and V stage ready)
        const uint32_t pa = tc::smem_u32(sP), vb = tc::smem_u32(sV + (kt & 1) * Cfg::KV_TILE);
#pragma unroll
        for (int ks = 0; ks < 8; ++ks)
          tc::mma_bf16(tmem + 256 + t * 128,
                       tc::sdesc_k_sw128(pa + (ks >> 2) * CHUNK + (ks & 3) * 32),
                       tc::sdesc_mn_sw128(vb + ks * 2048, CHUNK), idesc_o, (kt | ks) != 0);
        tc::mma_commit(&bar_o[t]);
      };
      tc::mbar_wait_sleep(&k_full[0], 0);
      tc::fence_after();
      issue_s(0, 0);
      if (hasB) issue_s(1, 0);
      tc::mma_commit(&k_empty[0]);
      for (int kt = 0; kt < nk; ++kt) {
        const bool more = kt + 1 < nk;
        tc::mbar_wait_sleep(&v_full[kt & 1], (kt >> 1) & 1);
        tc::mbar_wait_sleep(&bar_p[0], kt & 1);
        tc::fence_after();
        issue_pv(0, kt);
        if (!hasB) tc::mma_commit(&v_empty[kt & 1]);
        if (more) {
          tc::mbar_wait_sleep(&k_full[(kt + 1) & 1], ((kt + 1) >> 1) & 1);
          tc::fence_after();
          issue_s(0, kt + 1);
          if (!hasB) tc::mma_commit(&k_empty[(kt + 1) & 1]);
        }
        if (hasB) {
          tc::mbar_wait_sleep(&bar_p[1], kt & 1);
          tc::fence_after();
          issue_pv(1, kt);
          tc::mma_commit(&v_empty[kt & 1]);
          if (more) {
            issue_s(1, kt + 1);
            tc::mma_commit(&k_empty[(kt + 1) & 1]);
          }
        }
      }
    }
  } else if (warp >= 4) {
    const int t = (warp >= 8) ? 1 : 0;                     // query tile of this warpgroup
    if (t == 1 && !hasB) goto done;
    {
      const int q = warp & 3;
      const int row = q * 32 + lane;
      const uint32_t lane_off = (uint32_t)(q * 32) << 16;
      const uint32_t tS = tmem + t * 128, tO = tmem + 256 + t * 128;
      float m_used = -INFINITY, l = 0.f;
      const int sw = row & 7;
      uint8_t* prow = sP + row * 128;
      for (int kt = 0; kt < nk; ++kt) {
        tc::mbar_wait(&bar_s[t], kt & 1);
        tc::fence_after();
        const int valid = Lr - kt * 128;
        // pass 1: row max over the two 64-column halves
        float mx = -INFINITY;
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          float s[64];
          tc::tmem_ld32(tS + lane_off + h * 64, reinterpret_cast<uint32_t*>(s));
          tc::tmem_ld32(tS + lane_off + h * 64 + 32, reinterpret_cast<uint32_t*>(s + 32));
          tc::tmem_wait_ld();
          if (valid < (h + 1) * 64) {                     // only the request's last key tile
#pragma unroll
            for (int i = 0; i < 64; ++i) s[i] = (h * 64 + i < valid) ? s[i] : -INFINITY;
          }
          float m8[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) m8[j] = s[j];
#pragma unroll
          for (int i = 8; i < 64; ++i) m8[i & 7] = fmaxf(m8[i & 7], s[i]);
#pragma unroll
          for (int j = 0; j < 4; ++j) m8[j] = fmaxf(m8[j], m8[j + 4]);
          mx = fmaxf(mx, fmaxf(fmaxf(m8[0], m8[1]), fmaxf(m8[2], m8[3])));
        }
        mx *= scale_log2;
        const bool need = mx > m_used + 8.0f;
        const bool any_need = __any_sync(0xffffffffu, need);
        float factor = 1.0f;
        if (need) {
          factor = tc::ex2(m_used - mx);
          l *= factor;
          m_used = mx;
        }
        if (any_need && kt > 0) {                           // rescale O_t after PV_t(kt-1)
          tc::mbar_wait(&bar_o[t], (kt - 1) & 1);
          tc::fence_after();
#pragma unroll 1
          for (int c = 0; c < D / 32; ++c) {
            uint32_t o[32];
            tc::tmem_ld32(tO + lane_off + c * 32, o);
            tc::tmem_wait_ld();
#pragma unroll
            for (int e = 0; e < 32; ++e) o[e] = __float_as_uint(__uint_as_float(o[e]) * factor);
            tc::tmem_st32(tO + lane_off + c * 32, o);
          }
          tc::tmem_wait_st();
        }
        // pass 2: exponentials per half, then P into the shared P tile once it is free
        const float nm = -m_used;
        float a8[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          float s[64];
          tc::tmem_ld32(tS + lane_off + h * 64, reinterpret_cast<uint32_t*>(s));
          tc::tmem_ld32(tS + lane_off + h * 64 + 32, reinterpret_cast<uint32_t*>(s + 32));
          tc::tmem_wait_ld();
          if (valid < (h + 1) * 64) {
#pragma unroll
            for (int i = 0; i < 64; ++i) s[i] = (h * 64 + i < valid) ? s[i] : -INFINITY;
          }
#pragma unroll
          for (int i = 0; i < 64; i += 2) {
            tc::ffma2(s[i], s[i + 1], s[i], s[i + 1], scale_log2, scale_log2, nm, nm);
            if (((i >> 3) & 3) == 3) {
              tc::ex2_poly2(s[i], s[i + 1]);
            } else {
              s[i] = tc::ex2(s[i]);
              s[i + 1] = tc::ex2(s[i + 1]);
            }
            const int j = (i >> 1) & 3;
            tc::fadd2(a8[2 * j], a8[2 * j + 1], a8[2 * j], a8[2 * j + 1], s[i], s[i + 1]);
          }
          if (h == 0) {
            // the P tile is free once the other tile's previous PV (or, for tile B, this
            // tile-pair's PV_A) has completed; S_t is fully read after the second half's load
            if (t == 0) {
              if (kt > 0) {
                if (hasB) tc::mbar_wait(&bar_o[1], (kt - 1) & 1);
                else tc::mbar_wait(&bar_o[0], (kt - 1) & 1);
              }
            } else {
              tc::mbar_wait(&bar_o[0], kt & 1);
            }
            tc::fence_after();
          }
#pragma unroll
          for (int u = 0; u < 8; ++u) {
            const uint4 v = make_uint4(pack_bf16x2(s[u * 8 + 0], s[u * 8 + 1]),
                                       pack_bf16x2(s[u * 8 + 2], s[u * 8 + 3]),
                                       pack_bf16x2(s[u * 8 + 4], s[u * 8 + 5]),
                                       pack_bf16x2(s[u * 8 + 6], s[u * 8 + 7]));
            *reinterpret_cast<uint4*>(prow + h * CHUNK + ((u ^ sw) << 4)) = v;
          }
        }
        l += ((a8[0] + a8[1]) + (a8[2] + a8[3])) + ((a8[4] + a8[5]) + (a8[6] + a8[7]));
        tc::fence_proxy_async_smem();
        tc::fence_before();
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(&bar_p[t]);
      }
      if (nk > 0) {
        tc::mbar_wait(&bar_o[t], (nk - 1) & 1);
        tc::fence_after();
      }
      const float inv = (l > 0.f) ? 1.0f / l : 0.f;
      const int grow = q0 + t * 128 + row;
      __nv_bfloat16* orow = O + (size_t)grow * ldo + head * D;
#pragma unroll 1
      for (int c = 0; c < D / 32; ++c) {
        uint32_t o[32];
        tc::tmem_ld32(tO + lane_off + c * 32, o);
        tc::tmem_wait_ld();
        if (grow < q_end) {
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            float f[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) f[e] = __uint_as_float(o[g * 8 + e]) * inv;
            *reinterpret_cast<uint4*>(orow + c * 32 + g * 8) = Vec16<__nv_bfloat16>::pack(f);
          }
        }
      }
    }
  done:;
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

// ============================================================================================
// Two query tiles per CTA with P kept in TMEM and a correction warpgroup (default kernel).
//   warp 0      TMA: both Q tiles, then K tiles (2-stage ring)
//   warp 1      MMA: S_A(j), S_B(j), PV_A(j), S_A(j+1), PV_B(j), S_B(j+1), ...  PV takes P from
//               TMEM (A operand "ts" form), V from smem (MN-major); S_t(j+1) is issued right after
//               PV_t(j) into the same columns -- tcgen05.mma executes in issue order
//   warp 2      TMEM allocation
//   warp 3      TMA: V tiles (2-stage ring)
//   warps 4-7   softmax of tile A, 8-11 of tile B: thread = query row, the whole S row in
//               registers (one tcgen05.ld round), P as bf16 pairs back into the upper half of the
//               tile's S columns (tcgen05.st), lazy max with its rescale factor left in smem
//   warps 12-15 correction: rescale O_t in TMEM when a row's max grew (off the softmax critical
//               path; O_t(j-1) is complete by then because S_t(j) was issued after PV_t(j-1)),
//               final O / l to global
// Registers are rebalanced per warpgroup with setmaxnreg (softmax 192, correction 72, rest 56)
// so the 128-float S row fits without spills.  TMEM: S_A/P_A [0,128), S_B/P_B [128,256),
// O_A [256,256+D), O_B [384,384+D).  No smem P tile: the two softmax warpgroups no longer wait
// for each other's PV to free a shared buffer.
// Tuning knobs of the P-in-TMEM kernels (compile-time; defaults are the measured best):
//   FPS_ATTN_POLY  N > 0: every N-th group of 8 exponentials on the FMA pipe (0: all on MUFU)
//   FPS_ATTN_MMA_SPIN  1: the MMA warp spins on the P barriers instead of sleeping in try_wait
#ifndef FPS_ATTN_POLY
#define FPS_ATTN_POLY 4
#endif
#ifndef FPS_ATTN_POLY64          // the same for head_dim 64 (twice the exponentials per MMA FLOP)
#define FPS_ATTN_POLY64 4
#endif
#ifndef FPS_ATTN_PQ               // P release granularity of attn_tc3: 2 halves or 4 quarters
#define FPS_ATTN_PQ 2             // (quarters measured 1030 vs 1047 TF/s at C3's masked shape)
#endif
#ifndef FPS_ATTN_MMA_SPIN
#define FPS_ATTN_MMA_SPIN 0
#endif
#if FPS_ATTN_MMA_SPIN
#define ATTN_MMA_WAIT(bar, par) tc::mbar_wait(bar, par)
#else
#define ATTN_MMA_WAIT(bar, par) tc::mbar_wait_sleep(bar, par)
#endif
// Row max of 128 fp32 scores in C independent FMNMX3 chains.  16 chains (depth 5 + a 3-level
// tree) measured no faster than 4 (tools/scripts/r02z20_max16.sh: 1038 / 1205 vs 1044 / 1211
// TF/s at the C3 masked / dense shapes): the max phase is issue-shared, not latency-bound
#ifndef FPS_ATTN_MAX_CHAINS
#define FPS_ATTN_MAX_CHAINS 4
#endif
__device__ __forceinline__ float row_max128(const float* s) {
  constexpr int C = FPS_ATTN_MAX_CHAINS;
  float m[C];
#pragma unroll
  for (int j = 0; j < C; ++j) m[j] = s[j];
  int k = C;
#pragma unroll
  for (; k + 2 * C <= 128; k += 2 * C)
#pragma unroll
    for (int j = 0; j < C; ++j) m[j] = tc::fmax3(m[j], s[k + j], s[k + C + j]);
#pragma unroll
  for (; k < 128; k += C)
#pragma unroll
    for (int j = 0; j < C; ++j) m[j] = fmaxf(m[j], s[k + j]);
#pragma unroll
  for (int w = C; w > 1; w = (w + 2) / 3) {
#pragma unroll
    for (int j = 0; j < (w + 2) / 3; ++j) {
      const float a = m[3 * j], b = 3 * j + 1 < w ? m[3 * j + 1] : a, c = 3 * j + 2 < w ? m[3 * j + 2] : a;
      m[j] = tc::fmax3(a, b, c);
    }
  }
  return m[0];
}
template <int D>
__device__ __forceinline__ constexpr bool attn_poly(int i) {
  constexpr int N = D == 64 ? FPS_ATTN_POLY64 : FPS_ATTN_POLY;
  return N > 0 && ((i >> 3) % (N > 0 ? N : 1)) == (N > 0 ? N : 1) - 1;
}
#ifdef FPS_ATTN_TRACE
// developer instrumentation (separate build): per-step clock64 stamps of one CTA
__device__ long long g_attn_trace[2][64][8];
#define ATTN_TRACE(t, kt, slot)                                                     \
  do {                                                                              \
    if (blockIdx.x == 3 && blockIdx.y == 2 && (threadIdx.x & 31) == 0 && (kt) < 64) \
      g_attn_trace[t][kt][slot] = clock64();                                        \
  } while (0)
#else
#define ATTN_TRACE(t, kt, slot) do {} while (0)
#endif
template <int D>
struct Attn3Cfg {
  static constexpr int Q_BYTES = 128 * D * 2;
  static constexpr int KV_TILE = 128 * D * 2;
  static constexpr int SMEM = 2 * Q_BYTES + 4 * KV_TILE + 2 * 2 * 128 * 4 + 1024 + 256;
  static constexpr int TMEM_COLS = 512;
};

// Split-KV (gridDim.z = S > 1): CTA z covers key tiles [nk*z/S, nk*(z+1)/S) of its request,
// writes its own normalised output O_z (bf16, [total_q, H] at Opart + z * part_stride) and its
// (running max, row sum) pair to ML[z][row][head]; attn_combine_kernel merges the S partials.
template <int D>
__global__ void __launch_bounds__(512, 1)
    attn_tc3_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmKV,
                    __nv_bfloat16* __restrict__ O, const int32_t* __restrict__ cu_q,
                    const int32_t* __restrict__ cu_k, int n_req, int heads, float scale_log2, int ldo,
                    __nv_bfloat16* __restrict__ Opart, float2* __restrict__ ML, long long part_stride,
                    int total_q, const int32_t* __restrict__ o_map) {
  using Cfg = Attn3Cfg<D>;
  constexpr int CHUNK = 128 * 128;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sQ = smem;                                       // [2 tiles][D/64 chunks]
  uint8_t* sK = sQ + 2 * Cfg::Q_BYTES;                      // [2 stages][D/64 chunks]
  uint8_t* sV = sK + 2 * Cfg::KV_TILE;
  float* sScale = reinterpret_cast<float*>(sV + 2 * Cfg::KV_TILE);   // [tile][row]
  float* sL = sScale + 2 * 128;                                      // [tile][row]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sL + 2 * 128);
  uint64_t* bar_q = bars;
  uint64_t* k_full = bars + 1;
  uint64_t* k_empty = bars + 3;
  uint64_t* v_full = bars + 5;
  uint64_t* v_empty = bars + 7;
  uint64_t* bar_s = bars + 9;       // [tile] S_t(j) in TMEM            (MMA commit)
  uint64_t* bar_p = bars + 11;      // [tile] P_t(j) stored + O_t rescaled (4 softmax + 4 correction warps)
  uint64_t* bar_stat = bars + 13;   // [tile] scale_t(j) in smem             (4 softmax warps)
  uint64_t* bar_o = bars + 15;      // [tile] final PV_t done              (MMA commit)
  uint64_t* bar_fin = bars + 17;    // [tile] row sum l in smem            (4 softmax warps)
  uint64_t* bar_p2 = bars + 19;     // [tile] second half of P_t(j) stored (4 softmax warps)
  // FPS_ATTN_PQ = 4: P released in quarters -- bar_p (keys 0-31, + the correction warps),
  // bar_p2 (32-63), bar_p3 (64-95), bar_p4 (96-127); 2: halves (bar_p 0-63, bar_p2 64-127)
  uint64_t* bar_p3 = bars + 21;
  uint64_t* bar_p4 = bars + 23;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + 25);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // grid (heads, query-tile pairs, splits): heads vary fastest, so the CTAs the block scheduler
  // places last are the highest pair index -- for a single request its odd last tile, a short
  // CTA -- and a grid a few CTAs over the SMs left beside the method-3 gather (sm_budget())
  // costs one short CTA, not a second full-length wave
  const int head = blockIdx.x;
  const int H = heads * D;
  int r = 0, qp = blockIdx.y, ntile = 0;
  for (; r < n_req; ++r) {
    ntile = (__ldg(cu_q + r + 1) - __ldg(cu_q + r) + 127) >> 7;
    const int np = (ntile + 1) >> 1;
    if (qp < np) break;
    qp -= np;
  }
  const bool hasB = 2 * qp + 1 < ntile;
  const int q_end = __ldg(cu_q + r + 1);
  const int q0 = __ldg(cu_q + r) + qp * 256;
  const int Lr = __ldg(cu_k + r + 1) - __ldg(cu_k + r);
  const int nk_all = (Lr + 127) >> 7;
  const int nsplit = gridDim.z, split = blockIdx.z;
  const int kb = (int)(((long long)nk_all * split) / nsplit);       // first key tile of this CTA
  const int nk = (int)(((long long)nk_all * (split + 1)) / nsplit) - kb;
  const int k0 = __ldg(cu_k + r) + kb * 128;                         // its first key row
  const int Lr_rem = Lr - kb * 128;                                  // keys from k0 to the end

  if (threadIdx.x == 0) {
    tc::mbar_init(bar_q, 1);
    for (int s = 0; s < 2; ++s) {
      tc::mbar_init(&k_full[s], 1);
      tc::mbar_init(&k_empty[s], 1);
      tc::mbar_init(&v_full[s], 1);
      tc::mbar_init(&v_empty[s], 1);
      tc::mbar_init(&bar_s[s], 1);
      tc::mbar_init(&bar_p[s], 8);
      tc::mbar_init(&bar_stat[s], 4);
      tc::mbar_init(&bar_o[s], 1);
      tc::mbar_init(&bar_fin[s], 4);
      tc::mbar_init(&bar_p2[s], 4);
      tc::mbar_init(&bar_p3[s], 4);
      tc::mbar_init(&bar_p4[s], 4);
    }
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmQ);
    tc::tma_prefetch_desc(&tmKV);
  }
  if (warp == 2) tc::tmem_alloc<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = *tmem_holder;
  pdl_trigger();
  pdl_wait();

  if (warp < 4) {
    tc::regs_dec<56>();
    if (warp == 0) {
      if (lane == 0 && nk > 0) {
        tc::mbar_expect_tx(bar_q, (hasB ? 2 : 1) * Cfg::Q_BYTES);
        for (int t = 0; t < (hasB ? 2 : 1); ++t)
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tc::tma_load_2d(sQ + t * Cfg::Q_BYTES + c * CHUNK, &tmQ, bar_q, head * D + c * 64,
                            q0 + t * 128);
        for (int kt = 0; kt < nk; ++kt) {
          const int st = kt & 1;
          tc::mbar_wait_sleep(&k_empty[st], ((kt >> 1) & 1) ^ 1);
          tc::mbar_expect_tx(&k_full[st], Cfg::KV_TILE);
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tc::tma_load_2d(sK + st * Cfg::KV_TILE + c * CHUNK, &tmKV, &k_full[st],
                            head * D + c * 64, k0 + kt * 128);
        }
      }
    } else if (warp == 3) {
      if (lane == 0) {
        for (int kt = 0; kt < nk; ++kt) {
          const int st = kt & 1;
          tc::mbar_wait_sleep(&v_empty[st], ((kt >> 1) & 1) ^ 1);
          tc::mbar_expect_tx(&v_full[st], Cfg::KV_TILE);
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tc::tma_load_2d(sV + st * Cfg::KV_TILE + c * CHUNK, &tmKV, &v_full[st],
                            H + head * D + c * 64, k0 + kt * 128);
        }
      }
    } else if (warp == 1) {
      // whole warp: operands stay warp-uniform, one elected lane issues (see mma_bf16_w).  The
      // 512-column allocation is the whole TMEM, so its base is column 0 (a constant here).
      if (nk > 0) {
        constexpr uint32_t idesc_s = tc::idesc_bf16(128, 128);
        constexpr uint32_t idesc_o = tc::idesc_bf16(128, D, /*b_mn_major=*/true);
        tc::mbar_wait_sleep(bar_q, 0);
        const uint64_t dq = tc::sdesc_k_sw128(tc::smem_u32(sQ));
        const uint64_t dk = tc::sdesc_k_sw128(tc::smem_u32(sK));
        const uint64_t dv = tc::sdesc_mn_sw128(tc::smem_u32(sV), CHUNK);
        auto issue_s = [&](int t, int kt) {           // S_t = Q_t K_kt^T
          const uint64_t a = dq + ((t * Cfg::Q_BYTES) >> 4);
          const uint64_t b = dk + (((kt & 1) * Cfg::KV_TILE) >> 4);
          if constexpr (D == 128) tc::mma_ss_k8_commit<CHUNK / 16, CHUNK / 16>(t * 128, a, b, idesc_s, &bar_s[t]);
          else tc::mma_ss_k4_commit(t * 128, a, b, idesc_s, &bar_s[t]);
        };
        // O_t += P_t V_kt, P_t = TMEM cols [64,128): keys 0-63 as soon as the softmax has
        // stored them (bar_p), keys 64-127 after the rest (bar_p2)
        auto issue_pv = [&](int t, int kt) {
          const uint64_t b = dv + (((kt & 1) * Cfg::KV_TILE) >> 4);
          if constexpr (FPS_ATTN_PQ == 4) {
            uint64_t* qb[4] = {&bar_p[t], &bar_p2[t], &bar_p3[t], &bar_p4[t]};
#pragma unroll
            for (int qq = 0; qq < 4; ++qq) {
              ATTN_MMA_WAIT(qb[qq], kt & 1);
              tc::fence_after();
              tc::mma_ts_k2(256 + t * 128, t * 128 + 64 + 16 * qq, b + ((2 * 2048 * qq) >> 4),
                            idesc_o, (kt != 0 || qq != 0) ? 1u : 0u);
            }
          } else {
            ATTN_MMA_WAIT(&bar_p[t], kt & 1);
            tc::fence_after();
            ATTN_TRACE(t, kt, 5);
            tc::mma_ts_k4(256 + t * 128, t * 128 + 64, b, idesc_o, kt != 0);
            ATTN_MMA_WAIT(&bar_p2[t], kt & 1);
            tc::fence_after();
            ATTN_TRACE(t, kt, 6);
            tc::mma_ts_k4(256 + t * 128, t * 128 + 96, b + (4 * 2048 >> 4), idesc_o, 1);
          }
        };
        tc::mbar_wait_sleep(&k_full[0], 0);
        tc::fence_after();
        issue_s(0, 0);
        if (hasB) issue_s(1, 0);
        tc::mma_commit_w(&k_empty[0]);
        for (int kt = 0; kt < nk; ++kt) {
          const bool more = kt + 1 < nk;
          tc::mbar_wait_sleep(&v_full[kt & 1], (kt >> 1) & 1);
          issue_pv(0, kt);
          if (!more) tc::mma_commit_w(&bar_o[0]);
          if (!hasB) tc::mma_commit_w(&v_empty[kt & 1]);
          if (more) {
            tc::mbar_wait_sleep(&k_full[(kt + 1) & 1], ((kt + 1) >> 1) & 1);
            tc::fence_after();
            issue_s(0, kt + 1);
            if (!hasB) tc::mma_commit_w(&k_empty[(kt + 1) & 1]);
          }
          if (hasB) {
            issue_pv(1, kt);
            if (!more) tc::mma_commit_w(&bar_o[1]);
            tc::mma_commit_w(&v_empty[kt & 1]);
            if (more) {
              issue_s(1, kt + 1);
              tc::mma_commit_w(&k_empty[(kt + 1) & 1]);
            }
          }
        }
      }
    }
  } else if (warp < 12) {
    // ---------------- softmax (warps 4-7: tile A, 8-11: tile B) ----------------
    tc::regs_inc<192>();
    const int t = (warp >= 8) ? 1 : 0;
    if (t == 0 || hasB) {
      const int q = warp & 3;
      const int row = q * 32 + lane;
      const uint32_t lane_off = (uint32_t)(q * 32) << 16;
      const uint32_t tS = tmem + t * 128;
      float m_used = -INFINITY, l = 0.f;
      for (int kt = 0; kt < nk; ++kt) {
        tc::mbar_wait(&bar_s[t], kt & 1);
        tc::fence_after();
        ATTN_TRACE(t, kt, 0);
        float s[128];
#pragma unroll
        for (int c = 0; c < 4; ++c)
          tc::tmem_ld32(tS + lane_off + c * 32, reinterpret_cast<uint32_t*>(s + c * 32));
        tc::tmem_wait_ld();
        ATTN_TRACE(t, kt, 1);
        const int valid = Lr_rem - kt * 128;
        if (valid < 128) {                                 // only the request's last key tile
#pragma unroll
          for (int i = 0; i < 128; ++i) s[i] = (i < valid) ? s[i] : -INFINITY;
        }
        const float mx = row_max128(s) * scale_log2;
        float factor = 1.0f;
        if (mx > m_used + 8.0f) {                          // lazy rescale (threshold 2^8)
          factor = tc::ex2(m_used - mx);
          m_used = mx;
        }
        ATTN_TRACE(t, kt, 2);
        sScale[t * 128 + row] = factor;
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(&bar_stat[t]);
        // exponentials (a quarter on the FMA pipe), packed to bf16 pairs and stored into the
        // upper half of this tile's S columns 32 keys at a time
        const float nm = -m_used;
        float a8[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          uint32_t p[16];
#pragma unroll
          for (int i = c * 32; i < c * 32 + 32; i += 2) {
            tc::ffma2(s[i], s[i + 1], s[i], s[i + 1], scale_log2, scale_log2, nm, nm);
            if (attn_poly<D>(i)) {
              tc::ex2_poly2(s[i], s[i + 1]);
            } else {
              s[i] = tc::ex2(s[i]);
              s[i + 1] = tc::ex2(s[i + 1]);
            }
            p[(i - c * 32) >> 1] = tc::pack_bf16x2_rn(s[i], s[i + 1]);
          }
          tc::tmem_st16(tS + lane_off + 64 + c * 16, p);
          if (FPS_ATTN_PQ == 4 || (c & 1)) {               // keys released by halves / quarters
            tc::tmem_wait_st();
            tc::fence_before();
            __syncwarp();
            if (lane == 0) {
              if (FPS_ATTN_PQ == 4)
                tc::mbar_arrive(c == 0 ? &bar_p[t] : c == 1 ? &bar_p2[t] : c == 2 ? &bar_p3[t] : &bar_p4[t]);
              else
                tc::mbar_arrive(c == 1 ? &bar_p[t] : &bar_p2[t]);
            }
            ATTN_TRACE(t, kt, 2 + (c >> 1) + 1);
          }
        }
#pragma unroll
        for (int i = 0; i < 128; i += 2) {
          const int j = (i >> 1) & 3;
          tc::fadd2(a8[2 * j], a8[2 * j + 1], a8[2 * j], a8[2 * j + 1], s[i], s[i + 1]);
        }
        l = l * factor + (((a8[0] + a8[1]) + (a8[2] + a8[3])) + ((a8[4] + a8[5]) + (a8[6] + a8[7])));
      }
      sL[t * 128 + row] = l;
      if (nsplit > 1) {
        const int grow = q0 + t * 128 + row;
        if (grow < q_end) ML[((size_t)split * total_q + grow) * heads + head] = make_float2(m_used, l);
      }
      __syncwarp();
      if (lane == 0) tc::mbar_arrive(&bar_fin[t]);
    }
  } else {
    // ---------------- correction + epilogue (warps 12-15) ----------------
    tc::regs_dec<72>();
    const int q = warp & 3;
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const int ntl = hasB ? 2 : 1;
    for (int kt = 0; kt < nk; ++kt) {
      for (int t = 0; t < ntl; ++t) {
        tc::mbar_wait(&bar_stat[t], kt & 1);
        const float f = sScale[t * 128 + row];
        if (kt > 0 && __any_sync(0xffffffffu, f != 1.0f)) {
          // O_t(kt-1) is complete: softmax saw S_t(kt), issued after PV_t(kt-1)
          tc::fence_after();
          const uint32_t tO = tmem + 256 + t * 128 + lane_off;
#pragma unroll 1
          for (int c = 0; c < D / 32; ++c) {
            uint32_t o[32];
            tc::tmem_ld32(tO + c * 32, o);
            tc::tmem_wait_ld();
#pragma unroll
            for (int e = 0; e < 32; e += 2) {
              float x0 = __uint_as_float(o[e]), x1 = __uint_as_float(o[e + 1]);
              tc::ffma2(x0, x1, x0, x1, f, f, 0.f, 0.f);
              o[e] = __float_as_uint(x0);
              o[e + 1] = __float_as_uint(x1);
            }
            tc::tmem_st32(tO + c * 32, o);
          }
          tc::tmem_wait_st();
        }
        tc::fence_before();
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(&bar_p[t]);
      }
    }
    for (int t = 0; t < ntl; ++t) {
      const int grow = q0 + t * 128 + row;
      const int orow_i = (o_map && grow < q_end) ? __ldg(o_map + grow) : grow;
      __nv_bfloat16* orow = nsplit > 1
          ? Opart + split * part_stride + (size_t)grow * (heads * D) + head * D
          : O + (size_t)orow_i * ldo + head * D;
      if (nk == 0) {                                       // no keys: defined zero output
        if (grow < q_end) {
          for (int c = 0; c < D; c += 8) *reinterpret_cast<uint4*>(orow + c) = make_uint4(0, 0, 0, 0);
          if (nsplit > 1)
            ML[((size_t)split * total_q + grow) * heads + head] = make_float2(-INFINITY, 0.f);
        }
        continue;
      }
      tc::mbar_wait(&bar_fin[t], 0);
      tc::mbar_wait(&bar_o[t], 0);
      tc::fence_after();
      const float l = sL[t * 128 + row];
      const float inv = (l > 0.f) ? 1.0f / l : 0.f;
      const uint32_t tO = tmem + 256 + t * 128 + lane_off;
#pragma unroll 1
      for (int c = 0; c < D / 32; ++c) {
        uint32_t o[32];
        tc::tmem_ld32(tO + c * 32, o);
        tc::tmem_wait_ld();
        if (grow < q_end) {
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            float f[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) f[e] = __uint_as_float(o[g * 8 + e]) * inv;
            *reinterpret_cast<uint4*>(orow + c * 32 + g * 8) = Vec16<__nv_bfloat16>::pack(f);
          }
        }
      }
    }
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

// ============================================================================================
// attn_tc5: head_dim 64, two query tiles per CTA (as attn_tc3) with THREE S buffers in TMEM
// rotating over the two tiles.  At d = 64 the outputs need only 2 x 64 TMEM columns, so the 512
// columns hold S buffers at [0,128), [128,256), [256,384) and O_A [384,448), O_B [448,512).
// S of "index" i = 2 kt + t (tile t, key tile kt) lives in buffer i % 3, its P in that buffer's
// upper half.  The MMA warp issues S(i + 3) right after PV(i) into PV(i)'s buffer (tcgen05 MMAs
// execute in issue order), so the order is
//     S(0) S(1) S(2) | PV(0) S(3) | PV(1) S(4) | PV(2) S(5) | ...
// and S_t(kt+1) is issued after the OTHER tile's PV, not after PV_t(kt): a tile's softmax no
// longer waits for its own PV and next QK^T (attn_tc3's S -> softmax -> PV -> S chain, ~2850
// cycles per key tile at d = 64 against 1024 of MMAs), and the two softmax warpgroups can run
// back to back, bounded by MUFU / issue.
// Because S_t(kt+1) may now be computed before PV_t(kt), the correction warps wait for PV_t(kt)
// to complete (bar_pv) before rescaling O_t for key tile kt+1.  Barriers that a warpgroup may
// reach one key tile ahead of its consumer are double-buffered ([tile][kt & 1], parity
// (kt >> 1) & 1), so no phase can be overtaken.
struct Attn5Cfg {
  static constexpr int D = 64;
  static constexpr int Q_BYTES = 128 * D * 2;
  static constexpr int KV_TILE = 128 * D * 2;
  static constexpr int SMEM = 2 * Q_BYTES + 4 * KV_TILE + 2 * 2 * 128 * 4 + 1024 + 512;
  static constexpr int TMEM_COLS = 512;
  static constexpr int O_COL = 384;                         // O_t at O_COL + 64 t
};

__global__ void __launch_bounds__(512, 1)
    attn_tc5_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmKV,
                    __nv_bfloat16* __restrict__ O, const int32_t* __restrict__ cu_q,
                    const int32_t* __restrict__ cu_k, int n_req, int heads, float scale_log2, int ldo,
                    __nv_bfloat16* __restrict__ Opart, float2* __restrict__ ML, long long part_stride,
                    int total_q, const int32_t* __restrict__ o_map) {
  using Cfg = Attn5Cfg;
  constexpr int D = Cfg::D;
  constexpr int CHUNK = 128 * 128;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sQ = smem;                                       // [2 tiles]
  uint8_t* sK = sQ + 2 * Cfg::Q_BYTES;                      // [2 stages]
  uint8_t* sV = sK + 2 * Cfg::KV_TILE;
  float* sScale = reinterpret_cast<float*>(sV + 2 * Cfg::KV_TILE);   // [tile][row]
  float* sL = sScale + 2 * 128;                                      // [tile][row]
  uint64_t* bars = reinterpret_cast<uint64_t*>(sL + 2 * 128);
  uint64_t* bar_q = bars;
  uint64_t* k_full = bars + 1;      // [stage]
  uint64_t* k_empty = bars + 3;
  uint64_t* v_full = bars + 5;
  uint64_t* v_empty = bars + 7;
  uint64_t* bar_s = bars + 9;       // [buffer 0..2] S(i) in TMEM                 (MMA commit)
  uint64_t* bar_p = bars + 12;      // [tile][kt&1] P half 1 stored + O rescaled  (4 softmax + 4 corr.)
  uint64_t* bar_p2 = bars + 16;     // [tile][kt&1] P half 2 stored               (4 softmax + 4 corr.)
  uint64_t* bar_stat = bars + 20;   // [tile][kt&1] scale in smem                 (4 softmax)
  uint64_t* bar_pv = bars + 24;     // [tile][kt&1] PV_t(kt) complete             (MMA commit)
  uint64_t* bar_o = bars + 28;      // [tile] final PV done                       (MMA commit)
  uint64_t* bar_fin = bars + 30;    // [tile] row sum l in smem                   (4 softmax)
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + 32);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // grid (heads, query-tile pairs, splits) as attn_tc3
  const int head = blockIdx.x;
  const int H = heads * D;
  int r = 0, qp = blockIdx.y, ntile = 0;
  for (; r < n_req; ++r) {
    ntile = (__ldg(cu_q + r + 1) - __ldg(cu_q + r) + 127) >> 7;
    const int np = (ntile + 1) >> 1;
    if (qp < np) break;
    qp -= np;
  }
  const bool hasB = 2 * qp + 1 < ntile;
  const int q_end = __ldg(cu_q + r + 1);
  const int q0 = __ldg(cu_q + r) + qp * 256;
  const int Lr = __ldg(cu_k + r + 1) - __ldg(cu_k + r);
  const int nk_all = (Lr + 127) >> 7;
  const int nsplit = gridDim.z, split = blockIdx.z;
  const int kb = (int)(((long long)nk_all * split) / nsplit);
  const int nk = (int)(((long long)nk_all * (split + 1)) / nsplit) - kb;
  const int k0 = __ldg(cu_k + r) + kb * 128;
  const int Lr_rem = Lr - kb * 128;

  if (threadIdx.x == 0) {
    tc::mbar_init(bar_q, 1);
    for (int s = 0; s < 2; ++s) {
      tc::mbar_init(&k_full[s], 1);
      tc::mbar_init(&k_empty[s], 1);
      tc::mbar_init(&v_full[s], 1);
      tc::mbar_init(&v_empty[s], 1);
      tc::mbar_init(&bar_o[s], 1);
      tc::mbar_init(&bar_fin[s], 4);
    }
    for (int b = 0; b < 3; ++b) tc::mbar_init(&bar_s[b], 1);
    for (int b = 0; b < 4; ++b) {
      tc::mbar_init(&bar_p[b], 8);
      tc::mbar_init(&bar_p2[b], 8);
      tc::mbar_init(&bar_stat[b], 4);
      tc::mbar_init(&bar_pv[b], 1);
    }
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmQ);
    tc::tma_prefetch_desc(&tmKV);
  }
  if (warp == 2) tc::tmem_alloc<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem = *tmem_holder;
  pdl_trigger();
  pdl_wait();

  if (warp < 4) {
    tc::regs_dec<56>();
    if (warp == 0) {
      if (lane == 0 && nk > 0) {
        tc::mbar_expect_tx(bar_q, (hasB ? 2 : 1) * Cfg::Q_BYTES);
        for (int t = 0; t < (hasB ? 2 : 1); ++t)
          tc::tma_load_2d(sQ + t * Cfg::Q_BYTES, &tmQ, bar_q, head * D, q0 + t * 128);
        for (int kt = 0; kt < nk; ++kt) {
          const int st = kt & 1;
          tc::mbar_wait_sleep(&k_empty[st], ((kt >> 1) & 1) ^ 1);
          tc::mbar_expect_tx(&k_full[st], Cfg::KV_TILE);
          tc::tma_load_2d(sK + st * Cfg::KV_TILE, &tmKV, &k_full[st], head * D, k0 + kt * 128);
        }
      }
    } else if (warp == 3) {
      if (lane == 0) {
        for (int kt = 0; kt < nk; ++kt) {
          const int st = kt & 1;
          tc::mbar_wait_sleep(&v_empty[st], ((kt >> 1) & 1) ^ 1);
          tc::mbar_expect_tx(&v_full[st], Cfg::KV_TILE);
          tc::tma_load_2d(sV + st * Cfg::KV_TILE, &tmKV, &v_full[st], H + head * D, k0 + kt * 128);
        }
      }
    } else if (warp == 1) {
      if (nk > 0) {
        constexpr uint32_t idesc_s = tc::idesc_bf16(128, 128);
        constexpr uint32_t idesc_o = tc::idesc_bf16(128, D, /*b_mn_major=*/true);
        tc::mbar_wait_sleep(bar_q, 0);
        const uint64_t dq = tc::sdesc_k_sw128(tc::smem_u32(sQ));
        const uint64_t dk = tc::sdesc_k_sw128(tc::smem_u32(sK));
        const uint64_t dv = tc::sdesc_mn_sw128(tc::smem_u32(sV), CHUNK);
        // S(i) = Q_t K_kt^T into buffer i % 3 (i = 2 kt + t); a K tile is released after the
        // last S that reads it (tile B's, or tile A's when the CTA has one tile)
        auto issue_s = [&](int i) {
          const int t = i & 1, kt = i >> 1;
          const uint64_t a = dq + ((t * Cfg::Q_BYTES) >> 4);
          const uint64_t b = dk + (((kt & 1) * Cfg::KV_TILE) >> 4);
          tc::mma_ss_k4_commit((uint32_t)((i % 3) * 128), a, b, idesc_s, &bar_s[i % 3]);
          if (t == 1 || !hasB) tc::mma_commit_w(&k_empty[kt & 1]);
        };
        auto wait_k = [&](int kt) {
          tc::mbar_wait_sleep(&k_full[kt & 1], (kt >> 1) & 1);
          tc::fence_after();
        };
        // O_t += P_t V_kt: keys 0-63 once bar_p, keys 64-127 once bar_p2
        auto issue_pv = [&](int i) {
          const int t = i & 1, kt = i >> 1, pb = t * 2 + (kt & 1);
          const uint32_t ph = (kt >> 1) & 1;
          const uint64_t b = dv + (((kt & 1) * Cfg::KV_TILE) >> 4);
          const uint32_t p = (uint32_t)((i % 3) * 128);
          ATTN_MMA_WAIT(&bar_p[pb], ph);
          tc::fence_after();
          tc::mma_ts_k4(Cfg::O_COL + t * 64, p + 64, b, idesc_o, kt != 0);
          ATTN_MMA_WAIT(&bar_p2[pb], ph);
          tc::fence_after();
          tc::mma_ts_k4(Cfg::O_COL + t * 64, p + 96, b + (4 * 2048 >> 4), idesc_o, 1);
          tc::mma_commit_w(&bar_pv[pb]);
          if (kt + 1 == nk) tc::mma_commit_w(&bar_o[t]);
          if (t == 1 || !hasB) tc::mma_commit_w(&v_empty[kt & 1]);
        };
        // prologue: S(0), S(1), S(2) (indices of a missing tile B are skipped)
        wait_k(0);
        issue_s(0);
        if (hasB) issue_s(1);
        if (nk > 1) {
          wait_k(1);
          issue_s(2);
        }
        for (int kt = 0; kt < nk; ++kt) {
          tc::mbar_wait_sleep(&v_full[kt & 1], (kt >> 1) & 1);
          issue_pv(2 * kt);                                  // PV_A(kt)
          if (kt + 1 < nk && hasB) issue_s(2 * kt + 3);      // S_B(kt+1) into PV_A(kt)'s buffer
          if (hasB) issue_pv(2 * kt + 1);                    // PV_B(kt)
          if (kt + 2 < nk) {                                 // S_A(kt+2) into PV_B(kt)'s buffer
            wait_k(kt + 2);
            issue_s(2 * kt + 4);
          }
        }
      }
    }
  } else if (warp < 12) {
    // ---------------- softmax (warps 4-7: tile A, 8-11: tile B), as attn_tc3 ----------------
    tc::regs_inc<192>();
    const int t = (warp >= 8) ? 1 : 0;
    if (t == 0 || hasB) {
      const int q = warp & 3;
      const int row = q * 32 + lane;
      const uint32_t lane_off = (uint32_t)(q * 32) << 16;
      float m_used = -INFINITY, l = 0.f;
      for (int kt = 0; kt < nk; ++kt) {
        const int i = 2 * kt + t, pb = t * 2 + (kt & 1);
        // how many times buffer i % 3 was filled before: with two tiles every index is used
        // (buffer b holds indices b, b + 3, b + 6, ...: use i / 3); with one tile only the even
        // indices 2 kt are (buffer (2 kt) % 3 cycles with period 3 in kt: use kt / 3)
        const int n_use = hasB ? i / 3 : kt / 3;
        tc::mbar_wait(&bar_s[i % 3], (uint32_t)(n_use & 1));
        tc::fence_after();
        const uint32_t tS = tmem + (uint32_t)((i % 3) * 128);
        float s[128];
#pragma unroll
        for (int c = 0; c < 4; ++c)
          tc::tmem_ld32(tS + lane_off + c * 32, reinterpret_cast<uint32_t*>(s + c * 32));
        tc::tmem_wait_ld();
        const int valid = Lr_rem - kt * 128;
        if (valid < 128) {
#pragma unroll
          for (int k = 0; k < 128; ++k) s[k] = (k < valid) ? s[k] : -INFINITY;
        }
        const float mx = row_max128(s) * scale_log2;
        float factor = 1.0f;
        if (mx > m_used + 8.0f) {
          factor = tc::ex2(m_used - mx);
          m_used = mx;
        }
        sScale[t * 128 + row] = factor;
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(&bar_stat[pb]);
        const float nm = -m_used;
        float a8[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          uint32_t p[16];
#pragma unroll
          for (int k = c * 32; k < c * 32 + 32; k += 2) {
            tc::ffma2(s[k], s[k + 1], s[k], s[k + 1], scale_log2, scale_log2, nm, nm);
            if (attn_poly<D>(k)) {
              tc::ex2_poly2(s[k], s[k + 1]);
            } else {
              s[k] = tc::ex2(s[k]);
              s[k + 1] = tc::ex2(s[k + 1]);
            }
            p[(k - c * 32) >> 1] = tc::pack_bf16x2_rn(s[k], s[k + 1]);
          }
          tc::tmem_st16(tS + lane_off + 64 + c * 16, p);
          if (c & 1) {
            tc::tmem_wait_st();
            tc::fence_before();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(c == 1 ? &bar_p[pb] : &bar_p2[pb]);
          }
        }
#pragma unroll
        for (int k = 0; k < 128; k += 2) {
          const int j = (k >> 1) & 3;
          tc::fadd2(a8[2 * j], a8[2 * j + 1], a8[2 * j], a8[2 * j + 1], s[k], s[k + 1]);
        }
        l = l * factor + (((a8[0] + a8[1]) + (a8[2] + a8[3])) + ((a8[4] + a8[5]) + (a8[6] + a8[7])));
      }
      sL[t * 128 + row] = l;
      if (nsplit > 1) {
        const int grow = q0 + t * 128 + row;
        if (grow < q_end) ML[((size_t)split * total_q + grow) * heads + head] = make_float2(m_used, l);
      }
      __syncwarp();
      if (lane == 0) tc::mbar_arrive(&bar_fin[t]);
    }
  } else {
    // ---------------- correction + epilogue (warps 12-15) ----------------
    tc::regs_dec<72>();
    const int q = warp & 3;
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const int ntl = hasB ? 2 : 1;
    for (int kt = 0; kt < nk; ++kt) {
      for (int t = 0; t < ntl; ++t) {
        const int pb = t * 2 + (kt & 1);
        tc::mbar_wait(&bar_stat[pb], (uint32_t)((kt >> 1) & 1));
        if (kt > 0) {
          // PV_t(kt-1) must be complete before O_t is rescaled for key tile kt (its S may have
          // been computed first) -- and before this warp's arrival for kt can complete a phase
          const int pp = t * 2 + ((kt - 1) & 1);
          tc::mbar_wait(&bar_pv[pp], (uint32_t)(((kt - 1) >> 1) & 1));
        }
        const float f = sScale[t * 128 + row];
        if (kt > 0 && __any_sync(0xffffffffu, f != 1.0f)) {
          tc::fence_after();
          const uint32_t tO = tmem + Cfg::O_COL + t * 64 + lane_off;
#pragma unroll 1
          for (int c = 0; c < D / 32; ++c) {
            uint32_t o[32];
            tc::tmem_ld32(tO + c * 32, o);
            tc::tmem_wait_ld();
#pragma unroll
            for (int e = 0; e < 32; e += 2) {
              float x0 = __uint_as_float(o[e]), x1 = __uint_as_float(o[e + 1]);
              tc::ffma2(x0, x1, x0, x1, f, f, 0.f, 0.f);
              o[e] = __float_as_uint(x0);
              o[e + 1] = __float_as_uint(x1);
            }
            tc::tmem_st32(tO + c * 32, o);
          }
          tc::tmem_wait_st();
        }
        tc::fence_before();
        __syncwarp();
        if (lane == 0) {
          tc::mbar_arrive(&bar_p[pb]);
          tc::mbar_arrive(&bar_p2[pb]);
        }
      }
    }
    for (int t = 0; t < ntl; ++t) {
      const int grow = q0 + t * 128 + row;
      const int orow_i = (o_map && grow < q_end) ? __ldg(o_map + grow) : grow;
      __nv_bfloat16* orow = nsplit > 1
          ? Opart + split * part_stride + (size_t)grow * (heads * D) + head * D
          : O + (size_t)orow_i * ldo + head * D;
      if (nk == 0) {
        if (grow < q_end) {
          for (int c = 0; c < D; c += 8) *reinterpret_cast<uint4*>(orow + c) = make_uint4(0, 0, 0, 0);
          if (nsplit > 1)
            ML[((size_t)split * total_q + grow) * heads + head] = make_float2(-INFINITY, 0.f);
        }
        continue;
      }
      tc::mbar_wait(&bar_fin[t], 0);
      tc::mbar_wait(&bar_o[t], 0);
      tc::fence_after();
      const float l = sL[t * 128 + row];
      const float inv = (l > 0.f) ? 1.0f / l : 0.f;
      const uint32_t tO = tmem + Cfg::O_COL + t * 64 + lane_off;
#pragma unroll 1
      for (int c = 0; c < D / 32; ++c) {
        uint32_t o[32];
        tc::tmem_ld32(tO + c * 32, o);
        tc::tmem_wait_ld();
        if (grow < q_end) {
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            float f[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) f[e] = __uint_as_float(o[g * 8 + e]) * inv;
            *reinterpret_cast<uint4*>(orow + c * 32 + g * 8) = Vec16<__nv_bfloat16>::pack(f);
          }
        }
      }
    }
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc<Cfg::TMEM_COLS>(tmem);
  }
}

// ============================================================================================
// attn_tc4: CTA-pair (cta_group::2) attention, head_dim 128.  A cluster of two CTAs on two SMs
// takes two query tiles of one request (128 rows each, one per CTA); every MMA is issued by the
// leader for both:
//   S  = Q K^T   M = 256 (both tiles), N = 128 keys: each CTA stages its Q tile and HALF of the
//                key tile (64 keys) -- per SM half the K bytes of the 1-SM kernel, both from TMA
//                and from the smem port the MMA reads operands through;
//   O += P V     M = 256, N = 128: each CTA stages half of V's columns, P from each CTA's TMEM.
// S is double-buffered in TMEM (cols 0-127 / 128-255, O at 256-383), so S(j+1) is computed
// while the softmax works on S(j): the tensor pipe no longer waits for the exponentials of the
// tile it has just produced (attn_tc3's chain S -> softmax -> PV -> next S, measured 3066 cycles
// per key tile for two query tiles against 2048 of MMAs, tools/attn_trace.py).
// Warps: 0 K/Q producer, 1 MMA issuer (leader CTA), 2 TMEM allocator, 3 V producer,
// 4-11 softmax (two warps per TMEM lane quarter, 64 key columns each; the row max is exchanged
// through shared memory with a 64-thread named barrier), 12-15 correction + epilogue.
// Barriers on the leader count both CTAs' arrivals (P stored: softmax + correction warps of
// the two CTAs); MMA completions are multicast to both CTAs.
#ifndef FPS_ATTN4_POLY
#define FPS_ATTN4_POLY 4
#endif
// the leader's MMA warp waits for P (arrivals from both CTAs) spinning (1) or in the
// suspend-hinted try_wait (0)
#ifndef FPS_ATTN4_SPIN
#define FPS_ATTN4_SPIN 0
#endif
// MMA issue split over two warps on two SM sub-partitions (S: warp 1, PV: warp 2) instead of
// one: a tcgen05.mma issue occupies its sub-partition's dispatch, which the trace showed as the
// two softmax warps sharing the MMA warp's sub-partition running ~1000 cycles late per tile
#ifndef FPS_ATTN4_SPLIT
#define FPS_ATTN4_SPLIT 1
#endif
#ifndef FPS_ATTN4_CLUSTER_RELEASE
#define FPS_ATTN4_CLUSTER_RELEASE 0
#endif
#if FPS_ATTN4_CLUSTER_RELEASE
#define ATTN4_ARRIVE(a) tc::mbar_arrive_cluster(a)
#else
#define ATTN4_ARRIVE(a) tc::mbar_arrive_remote(a)
#endif
#if FPS_ATTN4_SPIN
#define ATTN4_MMA_WAIT(bar, par) tc::mbar_wait(bar, par)
#else
#define ATTN4_MMA_WAIT(bar, par) tc::mbar_wait_sleep(bar, par)
#endif
struct Attn4Cfg {
  static constexpr int D = 128;
  static constexpr int KS = 3, VS = 3;                      // K / V ring depths
  static constexpr int Q_BYTES = 128 * D * 2;               // this CTA's query tile
  static constexpr int K_HALF = 64 * D * 2;                 // 64 keys x 128 (2 chunks of 8 KB)
  static constexpr int V_HALF = 128 * 64 * 2;               // 128 keys x 64 columns
  static constexpr int SMEM = Q_BYTES + KS * K_HALF + VS * V_HALF + (4 + 2 + 2 + 1) * 128 * 4 + 1024 + 512;
  static constexpr int TMEM_COLS = 512;
};

#ifdef FPS_ATTN_TRACE
__device__ long long g_attn4_trace[4][64][8];
#define ATTN4_TRACE(t, kt, slot)                                                    \
  do {                                                                              \
    if (blockIdx.x == 2 && blockIdx.y == 3 && (threadIdx.x & 31) == 0 && (kt) < 64) \
      g_attn4_trace[t][kt][slot] = clock64();                                       \
  } while (0)
// every warp of both CTAs of pair 1 / head 3: [rank][warp][kt][slot], %globaltimer-free clock64
// of each SM (the two SMs' clocks are not aligned: compare within a rank)
__device__ long long g_attn4_warps[2][16][64][2];
#define ATTN4_WTRACE(kt, slot)                                                                 \
  do {                                                                                         \
    if ((blockIdx.x >> 1) == 1 && blockIdx.y == 3 && (threadIdx.x & 31) == 0 && (kt) < 64)     \
      g_attn4_warps[blockIdx.x & 1][threadIdx.x >> 5][kt][slot] = clock64();                   \
  } while (0)
#else
#define ATTN4_TRACE(t, kt, slot) do {} while (0)
#define ATTN4_WTRACE(kt, slot) do {} while (0)
#endif
__device__ __forceinline__ void named_bar_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(512, 1)
    attn_tc4_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                    const __grid_constant__ CUtensorMap tmV, __nv_bfloat16* __restrict__ O,
                    const int32_t* __restrict__ cu_q, const int32_t* __restrict__ cu_k, int n_req,
                    int heads, float scale_log2, int ldo, __nv_bfloat16* __restrict__ Opart,
                    float2* __restrict__ ML, long long part_stride, int total_q,
                    const int32_t* __restrict__ o_map) {
  using Cfg = Attn4Cfg;
  constexpr int D = Cfg::D;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + Cfg::Q_BYTES;
  uint8_t* sV = sK + Cfg::KS * Cfg::K_HALF;
  float* sMax = reinterpret_cast<float*>(sV + Cfg::VS * Cfg::V_HALF);   // [buf][half][row]
  float* sScale = sMax + 4 * 128;                                        // [buf][row]
  float* sL = sScale + 2 * 128;                                          // [half][row]
  float* sM = sL + 2 * 128;                                              // [row] final max
  uint64_t* bars = reinterpret_cast<uint64_t*>(sM + 128);
  uint64_t* bar_q = bars;                  // leader: both Q tiles landed
  uint64_t* k_full = bars + 1;             // [KS] leader: both K halves landed
  uint64_t* k_empty = bars + 4;            // [KS] both: S MMA done with the stage (multicast)
  uint64_t* v_full = bars + 7;             // [VS] leader
  uint64_t* v_empty = bars + 10;           // [VS] both (multicast)
  uint64_t* bar_s = bars + 13;             // [buf] both: S(j) in TMEM (multicast)
  uint64_t* bar_p = bars + 15;             // [buf] leader: keys 0-63 of P + O rescaled (2 x 8 warps)
  uint64_t* bar_p2 = bars + 17;            // [buf] leader: keys 64-127 of P (2 x 4 warps)
  uint64_t* bar_stat = bars + 19;          // [buf] local: scale of step j in smem (4 warps)
  uint64_t* bar_pv = bars + 21;            // both: PV(j) complete (multicast)
  uint64_t* bar_o = bars + 22;             // both: last PV complete (multicast)
  uint64_t* bar_fin = bars + 23;           // local: row-sum halves in smem (8 warps)
  uint64_t* pv_iss = bars + 24;            // [buf] leader: PV(j) issued (split issue: S warp waits)
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + 26);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = tc::cluster_ctarank();
  const int head = blockIdx.y;
  const int H = heads * D;
  int r = 0, qp = blockIdx.x >> 1, ntile = 0;
  for (; r < n_req; ++r) {
    ntile = (__ldg(cu_q + r + 1) - __ldg(cu_q + r) + 127) >> 7;
    const int np = (ntile + 1) >> 1;
    if (qp < np) break;
    qp -= np;
  }
  const int q_end = __ldg(cu_q + r + 1);
  const int q0 = __ldg(cu_q + r) + qp * 256 + (int)rank * 128;   // this CTA's first query row
  const int Lr = __ldg(cu_k + r + 1) - __ldg(cu_k + r);
  const int nk_all = (Lr + 127) >> 7;
  const int nsplit = gridDim.z, split = blockIdx.z;
  const int kb = (int)(((long long)nk_all * split) / nsplit);
  const int nk = (int)(((long long)nk_all * (split + 1)) / nsplit) - kb;
  const int k0 = __ldg(cu_k + r) + kb * 128;
  const int Lr_rem = Lr - kb * 128;

  if (threadIdx.x == 0) {
    tc::mbar_init(bar_q, 1);
    for (int s = 0; s < Cfg::KS; ++s) {
      tc::mbar_init(&k_full[s], 1);
      tc::mbar_init(&k_empty[s], 1);
    }
    for (int s = 0; s < Cfg::VS; ++s) {
      tc::mbar_init(&v_full[s], 1);
      tc::mbar_init(&v_empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      tc::mbar_init(&bar_s[b], 1);
      tc::mbar_init(&bar_p[b], 16);
      tc::mbar_init(&bar_p2[b], 8);
      tc::mbar_init(&bar_stat[b], 4);
    }
    tc::mbar_init(bar_pv, 1);
    tc::mbar_init(bar_o, 1);
    tc::mbar_init(bar_fin, 8);
    tc::mbar_init(&pv_iss[0], 1);
    tc::mbar_init(&pv_iss[1], 1);
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmQ);
    tc::tma_prefetch_desc(&tmK);
    tc::tma_prefetch_desc(&tmV);
  }
  if (warp == 2) tc::tmem_alloc_2sm<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::cluster_sync();                                      // peer barriers initialised
  tc::fence_after();
  const uint32_t tmem = *tmem_holder;
  pdl_trigger();
  pdl_wait();

  if (warp < 4) {
    tc::regs_dec<88>();
    if (warp == 0) {
      if (lane == 0 && nk > 0) {
        if (rank == 0) tc::mbar_expect_tx(bar_q, 2 * Cfg::Q_BYTES);
#pragma unroll
        for (int c = 0; c < D / 64; ++c)
          tc::tma_load_2d_2sm(sQ + c * (Cfg::Q_BYTES / 2), &tmQ, bar_q, head * D + c * 64, q0);
        for (int kt = 0; kt < nk; ++kt) {
          const int st = kt % Cfg::KS;
          tc::mbar_wait_sleep(&k_empty[st], ((kt / Cfg::KS) & 1) ^ 1);
          if (rank == 0) tc::mbar_expect_tx(&k_full[st], 2 * Cfg::K_HALF);
#pragma unroll
          for (int c = 0; c < D / 64; ++c)
            tc::tma_load_2d_2sm(sK + st * Cfg::K_HALF + c * (Cfg::K_HALF / 2), &tmK, &k_full[st],
                                head * D + c * 64, k0 + kt * 128 + (int)rank * 64);
        }
      }
    } else if (warp == 3) {
      if (lane == 0) {
        for (int kt = 0; kt < nk; ++kt) {
          const int st = kt % Cfg::VS;
          tc::mbar_wait_sleep(&v_empty[st], ((kt / Cfg::VS) & 1) ^ 1);
          if (rank == 0) tc::mbar_expect_tx(&v_full[st], 2 * Cfg::V_HALF);
          tc::tma_load_2d_2sm(sV + st * Cfg::V_HALF, &tmV, &v_full[st], H + head * D + (int)rank * 64,
                              k0 + kt * 128);
        }
      }
    } else if (warp == 1 || (FPS_ATTN4_SPLIT && warp == 2)) {
      if (rank == 0 && nk > 0) {
        constexpr uint32_t idesc_s = tc::idesc_bf16(256, 128);
        constexpr uint32_t idesc_o = tc::idesc_bf16(256, 128, /*b_mn_major=*/true);
        const uint64_t dq = tc::sdesc_k_sw128(tc::smem_u32(sQ));
        const uint64_t dk = tc::sdesc_k_sw128(tc::smem_u32(sK));
        const uint64_t dv = tc::sdesc_mn_sw128(tc::smem_u32(sV), Cfg::V_HALF);
        auto issue_s = [&](int j) {                        // S(j) -> TMEM buffer j & 1
          const int st = j % Cfg::KS;
          tc::mbar_wait_sleep(&k_full[st], (j / Cfg::KS) & 1);
          tc::fence_after();
          tc::mma2_ss_k8<(Cfg::Q_BYTES / 2) / 16, (Cfg::K_HALF / 2) / 16>(
              (j & 1) * 128, dq, dk + ((st * Cfg::K_HALF) >> 4), idesc_s);
          tc::mma2_commit_w(&k_empty[st]);
          tc::mma2_commit_w(&bar_s[j & 1]);
        };
        auto issue_pv = [&](int kt) {                      // O += P(kt) V(kt), both halves
          const int b = kt & 1, st = kt % Cfg::VS;
          const uint64_t v = dv + ((st * Cfg::V_HALF) >> 4);
          tc::mbar_wait_sleep(&v_full[st], (kt / Cfg::VS) & 1);
          ATTN4_TRACE(2, kt, 0);
          ATTN4_MMA_WAIT(&bar_p[b], (kt >> 1) & 1);
          tc::fence_after();
          ATTN4_TRACE(2, kt, 1);
          ATTN4_WTRACE(kt, 0);
          tc::mma2_ts_k4(256, b * 128 + 64, v, idesc_o, kt != 0);
          ATTN4_MMA_WAIT(&bar_p2[b], (kt >> 1) & 1);
          tc::fence_after();
          ATTN4_TRACE(2, kt, 2);
          ATTN4_WTRACE(kt, 1);
          tc::mma2_ts_k4(256, b * 128 + 96, v + (4 * 2048 >> 4), idesc_o, 1);
          tc::mma2_commit_w(&v_empty[st]);
          tc::mma2_commit_w(bar_pv);
          if (kt + 1 == nk) tc::mma2_commit_w(bar_o);
        };
        if (!FPS_ATTN4_SPLIT) {                            // one issuing warp: program order
          tc::mbar_wait_sleep(bar_q, 0);
          issue_s(0);
          if (nk > 1) issue_s(1);
          for (int kt = 0; kt < nk; ++kt) {
            issue_pv(kt);
            if (kt + 2 < nk) issue_s(kt + 2);              // into buffer b: after PV(kt) in order
            ATTN4_TRACE(2, kt, 3);
          }
        } else if (warp == 1) {                            // S issuer
          tc::mbar_wait_sleep(bar_q, 0);
          issue_s(0);
          if (nk > 1) issue_s(1);
          for (int j = 2; j < nk; ++j) {
            // buffer j & 1 still holds P(j - 2): issue after PV(j - 2) (same tensor-pipe queue)
            tc::mbar_wait_sleep(&pv_iss[j & 1], ((j - 2) >> 1) & 1);
            tc::fence_after();
            issue_s(j);
            ATTN4_TRACE(2, j - 2, 3);
          }
        } else {                                           // PV issuer (warp 2)
          for (int kt = 0; kt < nk; ++kt) {
            issue_pv(kt);
            tc::fence_before();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&pv_iss[kt & 1]);
          }
        }
      }
    }
  } else if (warp < 12) {
    // ---------------- softmax: warps 4-7 keys 0-63, 8-11 keys 64-127 of each S tile ----------
    tc::regs_inc<168>();
    const int q = warp & 3, h = (warp - 4) >> 2;
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const uint32_t leader_p = tc::mapa(tc::smem_u32(h == 0 ? bar_p : bar_p2), 0);
    float m_used = -INFINITY, l = 0.f;
    for (int kt = 0; kt < nk; ++kt) {
      const int b = kt & 1;
      const uint32_t tS = tmem + lane_off + b * 128;
      tc::mbar_wait(&bar_s[b], (kt >> 1) & 1);
      tc::fence_after();
      if (q == 0) ATTN4_TRACE(h, kt, 0);
      float s[64];
      tc::tmem_ld32(tS + h * 64, reinterpret_cast<uint32_t*>(s));
      tc::tmem_ld32(tS + h * 64 + 32, reinterpret_cast<uint32_t*>(s + 32));
      tc::tmem_wait_ld();
      if (q == 0) ATTN4_TRACE(h, kt, 1);
      const int valid = Lr_rem - kt * 128 - h * 64;
      if (valid < 64) {
#pragma unroll
        for (int i = 0; i < 64; ++i) s[i] = (i < valid) ? s[i] : -INFINITY;
      }
      float m4[4] = {s[0], s[1], s[2], s[3]};
#pragma unroll
      for (int i = 4; i < 60; i += 8)
#pragma unroll
        for (int j = 0; j < 4; ++j) m4[j] = tc::fmax3(m4[j], s[i + j], s[i + 4 + j]);
#pragma unroll
      for (int j = 0; j < 4; ++j) m4[j] = fmaxf(m4[j], s[60 + j]);
      const float pm = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3]));
      sMax[(b * 2 + h) * 128 + row] = pm;
      named_bar_sync(1 + q, 64);                           // both halves' S loaded, maxima out
      if (q == 0) ATTN4_TRACE(h, kt, 2);
      ATTN4_WTRACE(kt, 0);
      const float mx = fmaxf(pm, sMax[(b * 2 + (h ^ 1)) * 128 + row]) * scale_log2;
      float factor = 1.0f;
      if (mx > m_used + 8.0f) {                            // lazy rescale (threshold 2^8)
        factor = tc::ex2(m_used - mx);
        m_used = mx;
      }
      if (h == 0) {
        sScale[b * 128 + row] = factor;
        __syncwarp();
        if (lane == 0) tc::mbar_arrive(&bar_stat[b]);
      }
      // the exponentials below are plain (non-volatile) arithmetic the compiler may hoist above
      // the arrive, which then only issues near the end of the tile and holds the correction
      // warps (and PV) back by ~1000 cycles: make them depend on a volatile move after it
      float nm;
      asm volatile("mov.b32 %0, %1;" : "=f"(nm) : "f"(-m_used));
      float a8[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
#pragma unroll
      for (int c = 0; c < 2; ++c) {
        uint32_t p[16];
#pragma unroll
        for (int i = c * 32; i < c * 32 + 32; i += 2) {
          tc::ffma2(s[i], s[i + 1], s[i], s[i + 1], scale_log2, scale_log2, nm, nm);
          if (FPS_ATTN4_POLY > 0 && ((i >> 3) % (FPS_ATTN4_POLY > 0 ? FPS_ATTN4_POLY : 1)) ==
                                        (FPS_ATTN4_POLY > 0 ? FPS_ATTN4_POLY : 1) - 1) {
            tc::ex2_poly2(s[i], s[i + 1]);
          } else {
            s[i] = tc::ex2(s[i]);
            s[i + 1] = tc::ex2(s[i + 1]);
          }
          p[(i - c * 32) >> 1] = tc::pack_bf16x2_rn(s[i], s[i + 1]);
        }
        if (c == 1 && q == 0) ATTN4_TRACE(h, kt, 3);
        tc::tmem_st16(tS + 64 + h * 32 + c * 16, p);
      }
      tc::tmem_wait_st();
      if (q == 0) ATTN4_TRACE(h, kt, 4);
      tc::fence_before();
      __syncwarp();
      if (q == 0) ATTN4_TRACE(h, kt, 5);
      if (lane == 0) ATTN4_ARRIVE(leader_p + b * 8);
      if (q == 0) ATTN4_TRACE(h, kt, 6);
      ATTN4_WTRACE(kt, 1);
#pragma unroll
      for (int i = 0; i < 64; i += 2) {
        const int j = (i >> 1) & 3;
        tc::fadd2(a8[2 * j], a8[2 * j + 1], a8[2 * j], a8[2 * j + 1], s[i], s[i + 1]);
      }
      l = l * factor + (((a8[0] + a8[1]) + (a8[2] + a8[3])) + ((a8[4] + a8[5]) + (a8[6] + a8[7])));
    }
    sL[h * 128 + row] = l;
    if (nsplit > 1 && h == 0) sM[row] = m_used;            // final statistics: m for ML below
    __syncwarp();
    if (lane == 0) tc::mbar_arrive(bar_fin);
  } else {
    // ---------------- correction + epilogue (warps 12-15) ----------------
    tc::regs_dec<88>();
    const int q = warp & 3;
    const int row = q * 32 + lane;
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    const uint32_t leader_p = tc::mapa(tc::smem_u32(bar_p), 0);
    const uint32_t tO = tmem + 256 + lane_off;
    for (int kt = 0; kt < nk; ++kt) {
      const int b = kt & 1;
      tc::mbar_wait_sleep(&bar_stat[b], (kt >> 1) & 1);   // off the softmax warps' issue slots
      if (q == 0) ATTN4_TRACE(3, kt, 0);
      ATTN4_WTRACE(kt, 0);
      const float f = sScale[b * 128 + row];
      if (kt > 0 && __any_sync(0xffffffffu, f != 1.0f)) {
        tc::mbar_wait(bar_pv, (kt - 1) & 1);               // O(kt-1) complete
        tc::fence_after();
#pragma unroll 1
        for (int c = 0; c < D / 32; ++c) {
          uint32_t o[32];
          tc::tmem_ld32(tO + c * 32, o);
          tc::tmem_wait_ld();
#pragma unroll
          for (int e = 0; e < 32; e += 2) {
            float x0 = __uint_as_float(o[e]), x1 = __uint_as_float(o[e + 1]);
            tc::ffma2(x0, x1, x0, x1, f, f, 0.f, 0.f);
            o[e] = __float_as_uint(x0);
            o[e + 1] = __float_as_uint(x1);
          }
          tc::tmem_st32(tO + c * 32, o);
        }
        tc::tmem_wait_st();
      }
      tc::fence_before();
      __syncwarp();
      if (lane == 0) ATTN4_ARRIVE(leader_p + b * 8);
      if (q == 0) ATTN4_TRACE(3, kt, 1);
      ATTN4_WTRACE(kt, 1);
    }
    const int grow = q0 + row;
    const int orow_i = (o_map && grow < q_end) ? __ldg(o_map + grow) : grow;
    __nv_bfloat16* orow = nsplit > 1 ? Opart + split * part_stride + (size_t)grow * (heads * D) + head * D
                                     : O + (size_t)orow_i * ldo + head * D;
    if (nk == 0) {
      if (grow < q_end) {
        for (int c = 0; c < D; c += 8) *reinterpret_cast<uint4*>(orow + c) = make_uint4(0, 0, 0, 0);
        if (nsplit > 1) ML[((size_t)split * total_q + grow) * heads + head] = make_float2(-INFINITY, 0.f);
      }
    } else {
      tc::mbar_wait(bar_fin, 0);
      tc::mbar_wait(bar_o, 0);
      tc::fence_after();
      const float l = sL[row] + sL[128 + row];
      if (nsplit > 1 && grow < q_end)
        ML[((size_t)split * total_q + grow) * heads + head] = make_float2(sM[row], l);
      const float inv = (l > 0.f) ? 1.0f / l : 0.f;
#pragma unroll 1
      for (int c = 0; c < D / 32; ++c) {
        uint32_t o[32];
        tc::tmem_ld32(tO + c * 32, o);
        tc::tmem_wait_ld();
        if (grow < q_end) {
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            float f[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) f[e] = __uint_as_float(o[g * 8 + e]) * inv;
            *reinterpret_cast<uint4*>(orow + c * 32 + g * 8) = Vec16<__nv_bfloat16>::pack(f);
          }
        }
      }
    }
  }
  tc::fence_before();
  __syncthreads();
  tc::cluster_sync();                                      // both CTAs done with TMEM / barriers
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc_2sm<Cfg::TMEM_COLS>(tmem);
  }
}

// Merge of the split-KV partials: out = sum_z w_z O_z / sum_z w_z, w_z = l_z 2^(m_z - max m).
// One thread per 8 output columns of one (row, head).
template <int D>
__global__ void __launch_bounds__(256) attn_combine_kernel(const __nv_bfloat16* __restrict__ Opart,
                                                           const float2* __restrict__ ML,
                                                           long long part_stride, int nsplit,
                                                           int total_q, int heads,
                                                           __nv_bfloat16* __restrict__ O, int ldo,
                                                           const int32_t* __restrict__ o_map) {
  pdl_trigger();
  pdl_wait();
  constexpr int C8 = D / 8;
  const long long n = (long long)total_q * heads * C8;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (long long)gridDim.x * blockDim.x) {
    const int c8 = (int)(i % C8);
    const long long rh = i / C8;                       // row * heads + head
    const int row = (int)(rh / heads), head = (int)(rh - (long long)row * heads);
    float m = -INFINITY;
    for (int z = 0; z < nsplit; ++z) {
      const float2 v = __ldg(ML + (size_t)z * total_q * heads + rh);
      if (v.y > 0.f) m = fmaxf(m, v.x);
    }
    float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f}, wsum = 0.f;
    const size_t col = (size_t)row * heads * D + (size_t)head * D + c8 * 8;
    for (int z = 0; z < nsplit; ++z) {
      const float2 v = __ldg(ML + (size_t)z * total_q * heads + rh);
      if (!(v.y > 0.f)) continue;
      const float wz = v.y * exp2f(v.x - m);
      float f[8];
      Vec16<__nv_bfloat16>::unpack(__ldg(reinterpret_cast<const uint4*>(Opart + z * part_stride + col)), f);
#pragma unroll
      for (int e = 0; e < 8; ++e) acc[e] += wz * f[e];
      wsum += wz;
    }
    const float inv = wsum > 0.f ? 1.0f / wsum : 0.f;
#pragma unroll
    for (int e = 0; e < 8; ++e) acc[e] *= inv;
    const int orow = o_map ? __ldg(o_map + row) : row;
    *reinterpret_cast<uint4*>(O + (size_t)orow * ldo + head * D + c8 * 8) = Vec16<__nv_bfloat16>::pack(acc);
  }
}

int g_attn_force = 0;   // tests: 1 = one-tile kernel, 2 = two-tile smem-P kernel, 3 = P-in-TMEM
int g_attn_split = 0;   // tests: 0 = choose the split-KV factor, S > 0 = force S (when scratch fits)

bool attention_tc_supported(int dtype, int head_dim) {
  return dtype == FPS_BF16 && (head_dim == 64 || head_dim == 128);
}

template <int D>
static fps_status launch_d(const void* q, const void* kv, void* o, int heads,
                           const int32_t* d_cu_q, const int32_t* d_cu_k, const int32_t* h_cu_q,
                           const int32_t* h_cu_k, int n_req, cudaStream_t s, int ldo) {
  using Cfg = AttnCfg<D>;
  const int H = heads * D;
  int tiles = 0;
  for (int r = 0; r < n_req; ++r) tiles += (h_cu_q[r + 1] - h_cu_q[r] + 127) / 128;
  if (tiles == 0) return FPS_OK;
  // rows past a request's own keys (next request, or past the end: TMA zero fill) are masked
  // in-kernel; past-the-end query rows are never stored
  CUtensorMap tq, tkv;
  if (!make_tmap_2d_bf16(&tq, q, (uint64_t)h_cu_q[n_req], H, (uint64_t)H * 2, 64, 128))
    return fail(FPS_ECUDA, "attention_tc: Q tensor map");
  if (!make_tmap_2d_bf16(&tkv, kv, (uint64_t)h_cu_k[n_req], 2 * H, (uint64_t)H * 4, 64, 128))
    return fail(FPS_ECUDA, "attention_tc: KV tensor map");
  FPS_SMEM_ATTR((attn_tc_kernel<D>), Cfg::SMEM);
  const float scale_log2 = 1.4426950408889634f / sqrtf((float)D);
  FPS_CUDA_TRY(launch_k(attn_tc_kernel<D>, dim3(tiles, heads), dim3(256), Cfg::SMEM, s, tq, tkv,
                        reinterpret_cast<__nv_bfloat16*>(o), d_cu_q, d_cu_k, n_req, heads,
                        scale_log2, ldo));
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

template <int D>
static fps_status launch_d2(const void* q, const void* kv, void* o, int heads,
                            const int32_t* d_cu_q, const int32_t* d_cu_k, const int32_t* h_cu_q,
                            const int32_t* h_cu_k, int n_req, cudaStream_t s, int ldo) {
  using Cfg = Attn2Cfg<D>;
  const int H = heads * D;
  int pairs = 0;
  for (int r = 0; r < n_req; ++r) pairs += ((h_cu_q[r + 1] - h_cu_q[r] + 127) / 128 + 1) / 2;
  if (pairs == 0) return FPS_OK;
  CUtensorMap tq, tkv;
  if (!make_tmap_2d_bf16(&tq, q, (uint64_t)h_cu_q[n_req], H, (uint64_t)H * 2, 64, 128))
    return fail(FPS_ECUDA, "attention_tc2: Q tensor map");
  if (!make_tmap_2d_bf16(&tkv, kv, (uint64_t)h_cu_k[n_req], 2 * H, (uint64_t)H * 4, 64, 128))
    return fail(FPS_ECUDA, "attention_tc2: KV tensor map");
  FPS_SMEM_ATTR((attn_tc2_kernel<D>), Cfg::SMEM);
  const float scale_log2 = 1.4426950408889634f / sqrtf((float)D);
  FPS_CUDA_TRY(launch_k(attn_tc2_kernel<D>, dim3(pairs, heads), dim3(384), Cfg::SMEM, s, tq, tkv,
                        reinterpret_cast<__nv_bfloat16*>(o), d_cu_q, d_cu_k, n_req, heads,
                        scale_log2, ldo));
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

// Split-KV factor: the grid of `pairs x heads` CTAs (one per SM) often leaves the last wave
// mostly empty (C2A: 200 CTAs on 148 SMs -> 2 waves at 68 %); splitting every CTA's key range in
// S parts fills the waves better at the cost of a combine pass.  Chosen by wave efficiency
// (CTAs / (waves x 148)), S <= 4, at least 8 key tiles per part (measured with
// tools/block_probe.py: C2A, 32 key tiles, S = 2 cuts the block's attention 0.130 -> 0.119 ms,
// S = 3 / 4 lose; C2B, 8 key tiles, S = 2 loses 0.036 -> 0.044 ms), S > 1 only if it gains
// > 8 % and the scratch (partial outputs + statistics) fits.
static int choose_split(int ctas, int min_nk, int total_q, int H, int heads,
                        const AttnScratch* sc) {
  auto fits = [&](int S) {
    return sc && (size_t)S * total_q * H * 2 <= sc->part_bytes &&
           (size_t)S * total_q * heads * 8 <= sc->ml_bytes;
  };
  if (g_attn_split > 0) return fits(g_attn_split) && min_nk >= g_attn_split ? g_attn_split : 1;
  auto eff = [&](int S) {
    const long long c = (long long)ctas * S;
    const long long nb = sm_budget();
    return (double)c / (double)(((c + nb - 1) / nb) * nb);
  };
  int best = 1;
  double be = eff(1);
  for (int S = 2; S <= 4; ++S)
    if (min_nk >= 8 * S && fits(S) && eff(S) > be + 0.08) {
      best = S;
      be = eff(S);
    }
  return best;
}

template <int D>
static fps_status launch_d3(const void* q, const void* kv, void* o, int heads,
                            const int32_t* d_cu_q, const int32_t* d_cu_k, const int32_t* h_cu_q,
                            const int32_t* h_cu_k, int n_req, cudaStream_t s, int ldo,
                            const AttnScratch* sc, const int32_t* o_map) {
  using Cfg = Attn3Cfg<D>;
  const int H = heads * D;
  int pairs = 0, min_nk = 1 << 30;
  for (int r = 0; r < n_req; ++r) {
    const int pr = ((h_cu_q[r + 1] - h_cu_q[r] + 127) / 128 + 1) / 2;
    pairs += pr;
    if (pr > 0) min_nk = std::min(min_nk, (h_cu_k[r + 1] - h_cu_k[r] + 127) / 128);
  }
  if (pairs == 0) return FPS_OK;
  const int total_q = h_cu_q[n_req];
  const int S = choose_split(pairs * heads, min_nk, total_q, H, heads, sc);
  CUtensorMap tq, tkv;
  if (!make_tmap_2d_bf16(&tq, q, (uint64_t)h_cu_q[n_req], H, (uint64_t)H * 2, 64, 128))
    return fail(FPS_ECUDA, "attention_tc3: Q tensor map");
  if (!make_tmap_2d_bf16(&tkv, kv, (uint64_t)h_cu_k[n_req], 2 * H, (uint64_t)H * 4, 64, 128))
    return fail(FPS_ECUDA, "attention_tc3: KV tensor map");
  FPS_SMEM_ATTR((attn_tc3_kernel<D>), Cfg::SMEM);
  const float scale_log2 = 1.4426950408889634f / sqrtf((float)D);
  const long long part_stride = (long long)total_q * H;
  auto* Opart = S > 1 ? reinterpret_cast<__nv_bfloat16*>(sc->part) : nullptr;
  auto* ML = S > 1 ? reinterpret_cast<float2*>(sc->ml) : nullptr;
  FPS_CUDA_TRY(launch_k(attn_tc3_kernel<D>, dim3(heads, pairs, S), dim3(512), Cfg::SMEM, s, tq, tkv,
                        reinterpret_cast<__nv_bfloat16*>(o), d_cu_q, d_cu_k, n_req, heads,
                        scale_log2, ldo, Opart, ML, part_stride, total_q, o_map));
  if (S > 1) {
    count_launch();
    const long long n = (long long)total_q * heads * (D / 8);
    const int grid = (int)std::min<long long>((n + 255) / 256, kNumSMs * 8LL);
    FPS_CUDA_TRY(launch_k(attn_combine_kernel<D>, dim3(grid), dim3(256), 0, s,
                          (const __nv_bfloat16*)Opart, (const float2*)ML, part_stride, S, total_q,
                          heads, reinterpret_cast<__nv_bfloat16*>(o), ldo, o_map));
  }
#ifdef FPS_ATTN_TRACE
  {
    static long long h[2][64][8];
    cudaStreamSynchronize(s);
    cudaMemcpyFromSymbol(h, g_attn_trace, sizeof(h));
    const long long base = h[0][0][0];
    for (int kt = 0; kt < 12; ++kt)
      for (int t = 0; t < 2; ++t)
        fprintf(stderr, "trace t%d kt%2d: S %7lld ld %5lld max %5lld Plo %5lld Phi %5lld | mmaPV %7lld %7lld\n", t, kt,
                h[t][kt][0] - base, h[t][kt][1] - h[t][kt][0], h[t][kt][2] - h[t][kt][0],
                h[t][kt][3] - h[t][kt][0], h[t][kt][4] - h[t][kt][0], h[t][kt][5] - base,
                h[t][kt][6] - base);
  }
#endif
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

int g_attn_rot = 1;     // 1 = attn_tc5 (three rotating S buffers) for head_dim 64; 0 = attn_tc3

static fps_status launch_d5(const void* q, const void* kv, void* o, int heads,
                            const int32_t* d_cu_q, const int32_t* d_cu_k, const int32_t* h_cu_q,
                            const int32_t* h_cu_k, int n_req, cudaStream_t s, int ldo,
                            const AttnScratch* sc, const int32_t* o_map) {
  using Cfg = Attn5Cfg;
  constexpr int D = Cfg::D;
  const int H = heads * D;
  int pairs = 0, min_nk = 1 << 30;
  for (int r = 0; r < n_req; ++r) {
    const int pr = ((h_cu_q[r + 1] - h_cu_q[r] + 127) / 128 + 1) / 2;
    pairs += pr;
    if (pr > 0) min_nk = std::min(min_nk, (h_cu_k[r + 1] - h_cu_k[r] + 127) / 128);
  }
  if (pairs == 0) return FPS_OK;
  const int total_q = h_cu_q[n_req];
  const int S = choose_split(pairs * heads, min_nk, total_q, H, heads, sc);
  CUtensorMap tq, tkv;
  if (!make_tmap_2d_bf16(&tq, q, (uint64_t)h_cu_q[n_req], H, (uint64_t)H * 2, 64, 128))
    return fail(FPS_ECUDA, "attention_tc5: Q tensor map");
  if (!make_tmap_2d_bf16(&tkv, kv, (uint64_t)h_cu_k[n_req], 2 * H, (uint64_t)H * 4, 64, 128))
    return fail(FPS_ECUDA, "attention_tc5: KV tensor map");
  FPS_SMEM_ATTR(attn_tc5_kernel, Cfg::SMEM);
  const float scale_log2 = 1.4426950408889634f / sqrtf((float)D);
  const long long part_stride = (long long)total_q * H;
  auto* Opart = S > 1 ? reinterpret_cast<__nv_bfloat16*>(sc->part) : nullptr;
  auto* ML = S > 1 ? reinterpret_cast<float2*>(sc->ml) : nullptr;
  FPS_CUDA_TRY(launch_k(attn_tc5_kernel, dim3(heads, pairs, S), dim3(512), Cfg::SMEM, s, tq, tkv,
                        reinterpret_cast<__nv_bfloat16*>(o), d_cu_q, d_cu_k, n_req, heads,
                        scale_log2, ldo, Opart, ML, part_stride, total_q, o_map));
  if (S > 1) {
    count_launch();
    const long long n = (long long)total_q * heads * (D / 8);
    const int grid = (int)std::min<long long>((n + 255) / 256, kNumSMs * 8LL);
    FPS_CUDA_TRY(launch_k(attn_combine_kernel<D>, dim3(grid), dim3(256), 0, s,
                          (const __nv_bfloat16*)Opart, (const float2*)ML, part_stride, S, total_q,
                          heads, reinterpret_cast<__nv_bfloat16*>(o), ldo, o_map));
  }
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

int g_attn_pair = 0;    // 1 = the CTA-pair kernel (attn_tc4) for head_dim 128

static fps_status launch_d4(const void* q, const void* kv, void* o, int heads,
                            const int32_t* d_cu_q, const int32_t* d_cu_k, const int32_t* h_cu_q,
                            const int32_t* h_cu_k, int n_req, cudaStream_t s, int ldo,
                            const AttnScratch* sc, const int32_t* o_map) {
  using Cfg = Attn4Cfg;
  constexpr int D = Cfg::D;
  const int H = heads * D;
  int pairs = 0, min_nk = 1 << 30;
  for (int r = 0; r < n_req; ++r) {
    const int pr = ((h_cu_q[r + 1] - h_cu_q[r] + 127) / 128 + 1) / 2;
    pairs += pr;
    if (pr > 0) min_nk = std::min(min_nk, (h_cu_k[r + 1] - h_cu_k[r] + 127) / 128);
  }
  if (pairs == 0) return FPS_OK;
  const int total_q = h_cu_q[n_req];
  const int S = choose_split(2 * pairs * heads, min_nk, total_q, H, heads, sc);
  CUtensorMap tq, tk, tv;
  if (!make_tmap_2d_bf16(&tq, q, (uint64_t)h_cu_q[n_req], H, (uint64_t)H * 2, 64, 128))
    return fail(FPS_ECUDA, "attention_tc4: Q tensor map");
  if (!make_tmap_2d_bf16(&tk, kv, (uint64_t)h_cu_k[n_req], 2 * H, (uint64_t)H * 4, 64, 64) ||
      !make_tmap_2d_bf16(&tv, kv, (uint64_t)h_cu_k[n_req], 2 * H, (uint64_t)H * 4, 64, 128))
    return fail(FPS_ECUDA, "attention_tc4: KV tensor maps");
  FPS_SMEM_ATTR(attn_tc4_kernel, Cfg::SMEM);
  const float scale_log2 = 1.4426950408889634f / sqrtf((float)D);
  const long long part_stride = (long long)total_q * H;
  auto* Opart = S > 1 ? reinterpret_cast<__nv_bfloat16*>(sc->part) : nullptr;
  auto* ML = S > 1 ? reinterpret_cast<float2*>(sc->ml) : nullptr;
  FPS_CUDA_TRY(launch_k(attn_tc4_kernel, dim3(2 * pairs, heads, S), dim3(512), Cfg::SMEM, s, tq, tk,
                        tv, reinterpret_cast<__nv_bfloat16*>(o), d_cu_q, d_cu_k, n_req, heads,
                        scale_log2, ldo, Opart, ML, part_stride, total_q, o_map));
  if (S > 1) {
    count_launch();
    const long long n = (long long)total_q * heads * (D / 8);
    const int grid = (int)std::min<long long>((n + 255) / 256, kNumSMs * 8LL);
    FPS_CUDA_TRY(launch_k(attn_combine_kernel<D>, dim3(grid), dim3(256), 0, s,
                          (const __nv_bfloat16*)Opart, (const float2*)ML, part_stride, S, total_q,
                          heads, reinterpret_cast<__nv_bfloat16*>(o), ldo, o_map));
  }
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

fps_status launch_attention_tc(const void* q, const void* kv, void* o, int heads, int head_dim,
                               const int32_t* d_cu_q, const int32_t* d_cu_k, const int32_t* h_cu_q,
                               const int32_t* h_cu_k, int n_req, cudaStream_t s, int ldo,
                               const AttnScratch* sc, const int32_t* o_map) {
  if (ldo == 0) ldo = heads * head_dim;
  if (ldo < heads * head_dim || ldo % 8 != 0)
    return fail(FPS_EINVAL, "attention_tc: output row stride %d", ldo);
  if (!h_cu_q || !h_cu_k) return fail(FPS_EINVAL, "attention_tc needs host cu_q / cu_k");
  if (!aligned16(q) || !aligned16(kv) || !aligned16(o))
    return fail(FPS_EINVAL, "attention_tc: unaligned operand");
  // Default: P in TMEM + correction warpgroup (attn_tc3).  Measured on B200 (tools/attn_probe.py,
  // TFLOP/s at 16 x 1800 / 4 x 4608 query rows over 4608 keys): 1085 / 1200 vs 930 / 1004 for the
  // smem-P two-tile kernel and ~800 / 900 for the one-tile kernel.  A 64-key-step variant with S
  // double-buffered per tile (no S -> softmax -> PV -> S chain) measured 1113 at best: M=128 N=64
  // SS MMAs run at 66% of the tensor rate (48.6 instead of 32 cycles each, tools/micro/mma_rate:
  // A+B operand reads exceed the 128 B/clk smem port), which ate the latency it saved.
  if (g_attn_force == 0 && g_attn_pair && head_dim == 128)
    return launch_d4(q, kv, o, heads, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s, ldo, sc, o_map);
  if (g_attn_force == 0 || g_attn_force == 3) {
    if (head_dim == 128)
      return launch_d3<128>(q, kv, o, heads, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s, ldo, sc,
                            o_map);
    if (g_attn_force == 0 && g_attn_rot)
      return launch_d5(q, kv, o, heads, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s, ldo, sc, o_map);
    return launch_d3<64>(q, kv, o, heads, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s, ldo, sc, o_map);
  }
  if (o_map) return fail(FPS_EUNSUPPORTED, "attention: output row map needs the default kernel");
  if (g_attn_force == 2) {
    if (head_dim == 128)
      return launch_d2<128>(q, kv, o, heads, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s, ldo);
    return launch_d2<64>(q, kv, o, heads, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s, ldo);
  }
  if (head_dim == 128)
    return launch_d<128>(q, kv, o, heads, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s, ldo);
  return launch_d<64>(q, kv, o, heads, d_cu_q, d_cu_k, h_cu_q, h_cu_k, n_req, s, ldo);
}

}  // namespace fps

#ifdef FPS_ATTN_TRACE
extern "C" int fps_debug_attn_trace(long long* out) {
  return (int)cudaMemcpyFromSymbol(out, fps::g_attn_trace, sizeof(fps::g_attn_trace));
}
extern "C" int fps_debug_attn4_trace(long long* out) {
  return (int)cudaMemcpyFromSymbol(out, fps::g_attn4_trace, sizeof(fps::g_attn4_trace));
}
extern "C" int fps_debug_attn4_warps(long long* out) {
  return (int)cudaMemcpyFromSymbol(out, fps::g_attn4_warps, sizeof(fps::g_attn4_warps));
}
#endif
