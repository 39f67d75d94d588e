// a5/a7/a8: the masked-row projections and MLP as persistent, warp-specialised tcgen05 GEMMs.
// C[M, N] = A[M, K] . B[N, K]^T, bf16 in, fp32 accumulate in TMEM, fused epilogue (bias, GELU,
// gated residual, K/V row scatter into the merged key buffer -- PAPER.md L157/L161).
//
//   warp 0      TMA producer: A tile 128 x 64 and B tile BN x 64 per k-block, 128-B swizzle,
//               STAGES-deep smem ring (full/empty mbarriers)
//   warp 1      MMA issuer: one thread issues 4 x tcgen05.mma (M=128, N=BN, K=16) per k-block
//               into one of two TMEM accumulators; tcgen05.commit frees the smem stage
//   warp 2      TMEM allocator (2 x BN columns)
//   warps 4-7   epilogue: tcgen05.ld 32 columns at a time (thread = output row), fused ops,
//               16-B stores; the second accumulator lets tile i's epilogue overlap tile i+1's MMAs
// Tiles are visited n-major so the CTAs working at the same time share one weight tile (L2).
#include "epilogue.cuh"
#include "kernels.h"
#include "tc_util.cuh"

namespace fps {

template <int BN, int STAGES>
struct GemmCfg {
  static constexpr int BM = 128, BK = 64;
  static constexpr int A_BYTES = BM * BK * 2;
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int TMEM_COLS = 2 * BN;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 256;
};

template <int BN, int STAGES>
__global__ void __launch_bounds__(256, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   int M, int N, int K, Epilogue ep) {
  using Cfg = GemmCfg<BN, STAGES>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * Cfg::A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * Cfg::STAGE_BYTES);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int num_m = (M + Cfg::BM - 1) / Cfg::BM;
  const int num_n = (N + BN - 1) / BN;
  const int num_tiles = num_m * num_n;
  const int num_k = K / Cfg::BK;

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      tc::mbar_init(&full[s], 1);
      tc::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      tc::mbar_init(&tfull[a], 1);
      tc::mbar_init(&tempty[a], 4);
    }
    tc::fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tc::tma_prefetch_desc(&tmA);
    tc::tma_prefetch_desc(&tmB);
  }
  if (warp == 2) tc::tmem_alloc<Cfg::TMEM_COLS>(tmem_holder);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem_base = *tmem_holder;

  if (warp == 0) {
    if (lane == 0) {
      int stage = 0;
      uint32_t phase = 0;
      for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x) {
        const int m_blk = tile % num_m, n_blk = tile / num_m;
        for (int kb = 0; kb < num_k; ++kb) {
          tc::mbar_wait(&empty[stage], phase ^ 1);
          tc::mbar_expect_tx(&full[stage], Cfg::STAGE_BYTES);
          tc::tma_load_2d(sA + stage * Cfg::A_BYTES, &tmA, &full[stage], kb * Cfg::BK,
                          m_blk * Cfg::BM);
          tc::tma_load_2d(sB + stage * Cfg::B_BYTES, &tmB, &full[stage], kb * Cfg::BK, n_blk * BN);
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
        const uint32_t aphase = (it >> 1) & 1;
        tc::mbar_wait(&tempty[acc], aphase ^ 1);
        tc::fence_after();
        const uint32_t d = tmem_base + acc * BN;
        for (int kb = 0; kb < num_k; ++kb) {
          tc::mbar_wait(&full[stage], phase);
          tc::fence_after();
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
      }
    }
  } else if (warp >= 4) {
    const int q = warp & 3;
    int it = 0;
    const __nv_bfloat16* __restrict__ bias = reinterpret_cast<const __nv_bfloat16*>(ep.bias);
    const __nv_bfloat16* __restrict__ resid = reinterpret_cast<const __nv_bfloat16*>(ep.resid);
    for (int tile = blockIdx.x; tile < num_tiles; tile += gridDim.x, ++it) {
      const int m_blk = tile % num_m, n_blk = tile / num_m;
      const int acc = it & 1;
      const int row = m_blk * Cfg::BM + q * 32 + lane;
      const bool row_ok = row < M;
      // per-row epilogue state, looked up once per tile (not per column group)
      const __nv_bfloat16* gate = nullptr;
      int orow0 = row, orow1 = row;
      if (row_ok) {
        if (ep.gate)
          gate = reinterpret_cast<const __nv_bfloat16*>(ep.gate) +
                 (size_t)find_req(ep.cu, ep.n_req, row) * ep.gate_stride;
        if (ep.map0) orow0 = __ldg(ep.map0 + row);
        if (ep.map1) orow1 = __ldg(ep.map1 + row);
      }
      tc::mbar_wait(&tfull[acc], (it >> 1) & 1);
      tc::fence_after();
#pragma unroll 1
      for (int c = 0; c < BN / 32; ++c) {
        uint32_t r[32];
        tc::tmem_ld32(tmem_base + ((uint32_t)(q * 32) << 16) + acc * BN + c * 32, r);
        // issue every global load of this 32-column chunk before using any of them
        const int col0 = n_blk * BN + c * 32;
        uint4 bv[4], rv[4], gv[4];
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          const int c0 = col0 + g * 8;
          const bool ok = row_ok && c0 < N;
          bv[g] = (bias && ok) ? __ldg(reinterpret_cast<const uint4*>(bias + c0)) : make_uint4(0, 0, 0, 0);
          rv[g] = (resid && ok) ? __ldg(reinterpret_cast<const uint4*>(resid + (size_t)row * ep.ld_resid + c0))
                                : make_uint4(0, 0, 0, 0);
          gv[g] = (gate && ok) ? __ldg(reinterpret_cast<const uint4*>(gate + c0)) : make_uint4(0, 0, 0, 0);
        }
        tc::tmem_wait_ld();
        if (row_ok) {
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            const int c0 = col0 + g * 8;
            if (c0 < N) {
              float v[8], t[8];
#pragma unroll
              for (int e = 0; e < 8; ++e) v[e] = __uint_as_float(r[g * 8 + e]);
              if (bias) {
                Vec16<__nv_bfloat16>::unpack(bv[g], t);
#pragma unroll
                for (int e = 0; e < 8; ++e) v[e] += t[e];
              }
              if (ep.act == 1) {
#pragma unroll
                for (int e = 0; e < 8; ++e) v[e] = gelu_tanh(v[e]);
              }
              if (resid) {
                float rr[8];
                Vec16<__nv_bfloat16>::unpack(rv[g], rr);
                if (gate) {
                  Vec16<__nv_bfloat16>::unpack(gv[g], t);
#pragma unroll
                  for (int e = 0; e < 8; ++e) v[e] = rr[e] + t[e] * v[e];
                } else {
#pragma unroll
                  for (int e = 0; e < 8; ++e) v[e] = rr[e] + v[e];
                }
              }
              __nv_bfloat16* dst =
                  c0 < ep.split
                      ? reinterpret_cast<__nv_bfloat16*>(ep.out0) + (size_t)orow0 * ep.ld0 + c0
                      : reinterpret_cast<__nv_bfloat16*>(ep.out1) + (size_t)orow1 * ep.ld1 +
                            (c0 - ep.split);
              *reinterpret_cast<uint4*>(dst) = Vec16<__nv_bfloat16>::pack(v);
            }
          }
        }
      }
      tc::fence_before();
      __syncwarp();
      if (lane == 0) tc::mbar_arrive(&tempty[acc]);
    }
  }
  __syncthreads();
  if (warp == 2) {
    tc::fence_after();
    tc::tmem_dealloc<Cfg::TMEM_COLS>(tmem_base);
  }
}

bool gemm_tc_supported(int dtype, int M, int N, int K) {
  return dtype == FPS_BF16 && M > 0 && K >= 64 && K % 64 == 0 && N % 8 == 0;
}

template <int BN, int STAGES>
static fps_status launch_cfg(const void* A, const void* B, int M, int N, int K,
                             const Epilogue& ep, cudaStream_t s) {
  using Cfg = GemmCfg<BN, STAGES>;
  CUtensorMap ta, tb;
  if (!make_tmap_2d_bf16(&ta, A, M, K, (uint64_t)K * 2, Cfg::BK, Cfg::BM) ||
      !make_tmap_2d_bf16(&tb, B, N, K, (uint64_t)K * 2, Cfg::BK, BN))
    return fail(FPS_ECUDA, "gemm_tc: cuTensorMapEncodeTiled failed (M=%d N=%d K=%d)", M, N, K);
  static bool attr_set = false;
  if (!attr_set) {
    FPS_CUDA_TRY(cudaFuncSetAttribute(gemm_tc_kernel<BN, STAGES>,
                                      cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr_set = true;
  }
  const int tiles = ceil_div(M, Cfg::BM) * ceil_div(N, BN);
  const int grid = tiles < kNumSMs ? tiles : kNumSMs;
  gemm_tc_kernel<BN, STAGES><<<grid, 256, Cfg::SMEM, s>>>(ta, tb, M, N, K, ep);
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

fps_status launch_gemm_tc(const void* A, const void* B, int M, int N, int K, const Epilogue& ep,
                          cudaStream_t s) {
  if (!aligned16(A) || !aligned16(B)) return fail(FPS_EINVAL, "gemm_tc: unaligned operand");
  // pick the N tile that minimises (waves x tile width); ties -> the wider tile (less L2 traffic)
  const int m_blocks = ceil_div(M, 128);
  const long t256 = (long)m_blocks * ceil_div(N, 256), t128 = (long)m_blocks * ceil_div(N, 128);
  const long c256 = ((t256 + kNumSMs - 1) / kNumSMs) * 256;
  const long c128 = ((t128 + kNumSMs - 1) / kNumSMs) * 128;
  if (c256 <= c128) return launch_cfg<256, 4>(A, B, M, N, K, ep, s);
  return launch_cfg<128, 6>(A, B, M, N, K, ep, s);
}

}  // namespace fps
