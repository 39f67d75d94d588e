// sm_100a PTX helpers: mbarrier, TMA (cp.async.bulk.tensor), tcgen05 MMA / TMEM.
// Descriptor bit layouts follow the PTX ISA "tcgen05 matrix descriptors" and "instruction
// descriptor" tables (K-major operands, 128-byte swizzle, bf16 inputs, fp32 accumulate).
#pragma once
#include <cuda.h>

#include "common.cuh"

namespace fps {
namespace tc {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ---- mbarrier ------------------------------------------------------------------------------
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
// FPS_HANG_WATCH builds (debugging only): a wait still unsatisfied after 4 s of wall time
// reports the kernel shape, block, thread, barrier and parity, then traps.
#ifdef FPS_HANG_WATCH
__device__ __forceinline__ unsigned long long global_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define FPS_WATCH_DECL unsigned long long _t0 = 0, _spins = 0;
#define FPS_WATCH_STEP(a, parity)                                                              \
  if ((++_spins & 1023) == 0) {                                                                \
    const unsigned long long _now = global_ns();                                              \
    if (_t0 == 0) _t0 = _now;                                                                  \
    else if (_now - _t0 > 4000000000ull) {                                                     \
      printf("HANG grid(%d,%d) block(%d) cta(%d,%d) thr %d bar 0x%x parity %u\n", gridDim.x,  \
             gridDim.y, blockDim.x, blockIdx.x, blockIdx.y, threadIdx.x, a, parity);           \
      __trap();                                                                                \
    }                                                                                          \
  }
#else
#define FPS_WATCH_DECL
#define FPS_WATCH_STEP(a, parity)
#endif
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  uint32_t done;
  FPS_WATCH_DECL
  do {
    FPS_WATCH_STEP(a, parity)
    asm volatile(
        "{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
        "selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(a), "r"(parity)
        : "memory");
  } while (!done);
}
// try_wait with a suspend-time hint: the waiting warp sleeps in hardware until the phase
// completes instead of re-issuing try_wait in a tight loop.  Used by the attention's producer and
// MMA warps, whose spinning otherwise steals issue slots from the softmax warps sharing their SM
// sub-partition (measured: 2.3M try_wait issues per launch; 537 -> 564 TFLOP/s at n = 1331).
// Not used in the GEMM: there the later wake-up cost more than the issue slots it saved.
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  uint32_t done;
  FPS_WATCH_DECL
  do {
    FPS_WATCH_STEP(a, parity)
    asm volatile(
        "{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n"
        "selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(a), "r"(parity), "r"(10000000u)
        : "memory");
  } while (!done);
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

// ---- TMA -----------------------------------------------------------------------------------
__device__ __forceinline__ void tma_prefetch_desc(const void* desc) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(desc)) : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* smem_dst, const void* desc, uint64_t* bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3}], [%4];" ::"r"(smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(desc)), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_load_3d(void* smem_dst, const void* desc, uint64_t* bar,
                                            int c0, int c1, int c2) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(desc)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_u32(bar))
      : "memory");
}

// ---- clusters (CTA pairs) ------------------------------------------------------------------
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::
                   : "memory");
}
// shared::cluster address of the same smem offset in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t mapa(uint32_t smem_addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_addr), "r"(rank));
  return r;
}
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr)
               : "memory");
}
// remote arrive with the default (.release.cta) semantics, as CUTLASS's ClusterBarrier::arrive:
// the payload it publishes (tcgen05 stores, ordered by tcgen05.fence::before_thread_sync) is read
// by the tensor core, not by the peer's threads, so no cluster-scope release is needed
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
// 2-SM TMA: data lands in the issuing CTA, the transaction bytes count on CTA 0's barrier
constexpr uint32_t kPeerBitMask = 0xFEFFFFFFu;
__device__ __forceinline__ void tma_load_2d_2sm(void* smem_dst, const void* desc, uint64_t* bar,
                                                int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3}], [%4];" ::"r"(smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(desc)), "r"(c0), "r"(c1),
      "r"(smem_u32(bar) & kPeerBitMask)
      : "memory");
}
__device__ __forceinline__ void mma_bf16_2sm(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc,
                                             uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}
// commit the leader's MMAs to the barrier at this offset in both CTAs of the pair
__device__ __forceinline__ void mma_commit_2sm(uint64_t* bar) {
  asm volatile(
      "{\n.reg .b16 m;\nmov.b16 m, 3;\n"
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64"
      " [%0], m;\n}\n" ::"r"(smem_u32(bar))
      : "memory");
}
template <int NCOLS>
__device__ __forceinline__ void tmem_alloc_2sm(uint32_t* smem_holder) {
  asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                   smem_u32(smem_holder)),
               "n"(NCOLS)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
template <int NCOLS>
__device__ __forceinline__ void tmem_dealloc_2sm(uint32_t base) {
  asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(base), "n"(NCOLS)
               : "memory");
}

// ---- tcgen05 -------------------------------------------------------------------------------
// Shared-memory matrix descriptor, K-major, SWIZZLE_128B: rows of 128 B, 8-row core groups
// 1024 B apart (SBO), LBO unused (1), version 1 (sm_100), layout type 2 (128B swizzle).
__device__ __forceinline__ uint64_t sdesc_k_sw128(uint32_t smem_addr) {
  uint64_t d = 0;
  d |= (uint64_t)((smem_addr >> 4) & 0x3FFFu);
  d |= (uint64_t)1u << 16;                 // LBO (ignored for swizzled K-major)
  d |= (uint64_t)(1024u >> 4) << 32;       // SBO = 1024 B
  d |= (uint64_t)1u << 46;                 // descriptor version (sm_100)
  d |= (uint64_t)2u << 61;                 // SWIZZLE_128B
  return d;
}
// MN-major (e.g. V as the B operand of P.V: rows = keys (K dim), 128 B = 64 values of the N dim
// contiguous), SWIZZLE_128B: LBO = byte distance between 64-wide N chunks, SBO = 1024 B between
// 8-row K groups.
__device__ __forceinline__ uint64_t sdesc_mn_sw128(uint32_t smem_addr, uint32_t lbo_bytes) {
  uint64_t d = 0;
  d |= (uint64_t)((smem_addr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo_bytes >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)(1024u >> 4) << 32;
  d |= (uint64_t)1u << 46;
  d |= (uint64_t)2u << 61;
  return d;
}
// Instruction descriptor kind::f16: D f32, A/B bf16, K-major (or MN-major B), M x N.
__host__ __device__ constexpr uint32_t idesc_bf16(int M, int N, bool b_mn_major = false) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((b_mn_major ? 1u : 0u) << 16) |
         ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ void mma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc,
                                         uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}
// A operand from TMEM (the "ts" form): D += A[tmem] * B[smem]
__device__ __forceinline__ void mma_bf16_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc,
                                            uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(bdesc), "r"(idesc), "r"(accumulate));
}
// Warp-wide variants: executed by all 32 lanes with warp-uniform operands, one lane elected inside
// the asm issues.  Keeps the operands in uniform registers (no per-MMA R2UR / waterfall loop that
// a single-lane branch costs), which matters for the 64-cycle 128x128x16 MMAs of the attention.
__device__ __forceinline__ void mma_bf16_w(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc,
                                          uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n.reg .pred p, e;\nelect.sync _|e, 0xffffffff;\nsetp.ne.b32 p, %4, 0;\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}
__device__ __forceinline__ void mma_bf16_ts_w(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc,
                                              uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n.reg .pred p, e;\nelect.sync _|e, 0xffffffff;\nsetp.ne.b32 p, %4, 0;\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(bdesc), "r"(idesc), "r"(accumulate));
}
__device__ __forceinline__ void mma_commit_w(uint64_t* bar) {
  asm volatile(
      "{\n.reg .pred e;\nelect.sync _|e, 0xffffffff;\n"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n}\n" ::"r"(
          smem_u32(bar))
      : "memory");
}
// Whole MMA groups in one asm block (one elect.sync per group, descriptor low words advanced with
// 32-bit immediates): the per-MMA wrapper above still cost ~20 SASS instructions per 64-cycle
// MMA (collective elect + R2UR of every operand), which made the attention's MMA warp the
// bottleneck.  Descriptor addresses stay below 2^14 (smem < 256 KB) so the low-word adds never
// carry into the high word.
// SS group, K-major SW128 A and B, 8 x K=16 (d = 128): k-steps 0-3 advance 32 B inside the 128 B
// swizzle row, k-steps 4-7 start at the next 64-column chunk (A_CH / B_CH, in 16-B units).
// Commits the group to `bar`.
template <int A_CH, int B_CH>
__device__ __forceinline__ void mma_ss_k8_commit(uint32_t d, uint64_t adesc, uint64_t bdesc,
                                                 uint32_t idesc, uint64_t* bar) {
  const uint32_t alo = (uint32_t)adesc, ahi = (uint32_t)(adesc >> 32);
  const uint32_t blo = (uint32_t)bdesc, bhi = (uint32_t)(bdesc >> 32);
  asm volatile(
      "{\n.reg .pred e;\n.reg .b32 al, bl;\n.reg .b64 ad, bd;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "mov.b64 ad, {%1, %2};\nmov.b64 bd, {%3, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 0;\n"
      "add.s32 al, %1, 2;\nadd.s32 bl, %3, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, %1, 4;\nadd.s32 bl, %3, 4;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, %1, 6;\nadd.s32 bl, %3, 6;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, %1, %7;\nadd.s32 bl, %3, %8;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, al, 2;\nadd.s32 bl, bl, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, al, 2;\nadd.s32 bl, bl, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, al, 2;\nadd.s32 bl, bl, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%6];\n"
      "}\n" ::"r"(d),
      "r"(alo), "r"(ahi), "r"(blo), "r"(bhi), "r"(idesc), "r"(smem_u32(bar)), "n"(A_CH), "n"(B_CH)
      : "memory");
}
// SS group with 4 x K=16 (d = 64): one 64-column chunk.
__device__ __forceinline__ void mma_ss_k4_commit(uint32_t d, uint64_t adesc, uint64_t bdesc,
                                                 uint32_t idesc, uint64_t* bar) {
  const uint32_t alo = (uint32_t)adesc, ahi = (uint32_t)(adesc >> 32);
  const uint32_t blo = (uint32_t)bdesc, bhi = (uint32_t)(bdesc >> 32);
  asm volatile(
      "{\n.reg .pred e;\n.reg .b32 al, bl;\n.reg .b64 ad, bd;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "mov.b64 ad, {%1, %2};\nmov.b64 bd, {%3, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 0;\n"
      "add.s32 al, %1, 2;\nadd.s32 bl, %3, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, %1, 4;\nadd.s32 bl, %3, 4;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, %1, 6;\nadd.s32 bl, %3, 6;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], ad, bd, %5, 1;\n"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%6];\n"
      "}\n" ::"r"(d),
      "r"(alo), "r"(ahi), "r"(blo), "r"(bhi), "r"(idesc), "r"(smem_u32(bar))
      : "memory");
}
// TS group (A = P from TMEM, 8 columns per K=16 step; B = V MN-major, 2048 B per 16 keys),
// 4 steps (64 keys); `acc` = 0 only for the first group of the output.
__device__ __forceinline__ void mma_ts_k4(uint32_t d, uint32_t a_tmem, uint64_t bdesc,
                                          uint32_t idesc, uint32_t acc) {
  const uint32_t blo = (uint32_t)bdesc, bhi = (uint32_t)(bdesc >> 32);
  asm volatile(
      "{\n.reg .pred e, p;\n.reg .b32 ta, bl;\n.reg .b64 bd;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "setp.ne.b32 p, %5, 0;\n"
      "mov.b64 bd, {%2, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], bd, %4, p;\n"
      "add.s32 ta, %1, 8;\nadd.s32 bl, %2, 128;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 16;\nadd.s32 bl, %2, 256;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 24;\nadd.s32 bl, %2, 384;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "}\n" ::"r"(d),
      "r"(a_tmem), "r"(blo), "r"(bhi), "r"(idesc), "r"(acc)
      : "memory");
}
// TS group of 2 steps (32 keys): as mma_ts_k4, half the keys
__device__ __forceinline__ void mma_ts_k2(uint32_t d, uint32_t a_tmem, uint64_t bdesc,
                                          uint32_t idesc, uint32_t acc) {
  const uint32_t blo = (uint32_t)bdesc, bhi = (uint32_t)(bdesc >> 32);
  asm volatile(
      "{\n.reg .pred e, p;\n.reg .b32 ta, bl;\n.reg .b64 bd;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "setp.ne.b32 p, %5, 0;\n"
      "mov.b64 bd, {%2, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], bd, %4, p;\n"
      "add.s32 ta, %1, 8;\nadd.s32 bl, %2, 128;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "}\n" ::"r"(d),
      "r"(a_tmem), "r"(blo), "r"(bhi), "r"(idesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void mma_ts_k4_commit(uint32_t d, uint32_t a_tmem, uint64_t bdesc,
                                                 uint32_t idesc, uint32_t acc, uint64_t* bar) {
  mma_ts_k4(d, a_tmem, bdesc, idesc, acc);
  mma_commit_w(bar);
}
// TS group, 8 steps (128 keys), no commit (callers commit once per tile).
__device__ __forceinline__ void mma_ts_k8(uint32_t d, uint32_t a_tmem, uint64_t bdesc,
                                          uint32_t idesc, uint32_t acc) {
  const uint32_t blo = (uint32_t)bdesc, bhi = (uint32_t)(bdesc >> 32);
  asm volatile(
      "{\n.reg .pred e, p;\n.reg .b32 ta, bl;\n.reg .b64 bd;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "setp.ne.b32 p, %5, 0;\n"
      "mov.b64 bd, {%2, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], bd, %4, p;\n"
      "add.s32 ta, %1, 8;\nadd.s32 bl, %2, 128;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 16;\nadd.s32 bl, %2, 256;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 24;\nadd.s32 bl, %2, 384;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 32;\nadd.s32 bl, %2, 512;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 40;\nadd.s32 bl, %2, 640;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 48;\nadd.s32 bl, %2, 768;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 56;\nadd.s32 bl, %2, 896;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::1.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "}\n" ::"r"(d),
      "r"(a_tmem), "r"(blo), "r"(bhi), "r"(idesc), "r"(acc)
      : "memory");
}
// ---- CTA-pair (cta_group::2) groups for the attention: issued by the leader CTA's MMA warp
// (warp-wide, one elected lane), M = 256 rows = 128 per CTA, B operand split along N between the
// two CTAs (same smem offset in each), A from smem (S = Q K^T) or from TMEM (O += P V).
// SS group, 8 x K=16 (d = 128), no commit; A_CH / B_CH = 64-column chunk strides (16-B units).
template <int A_CH, int B_CH>
__device__ __forceinline__ void mma2_ss_k8(uint32_t d, uint64_t adesc, uint64_t bdesc,
                                           uint32_t idesc) {
  const uint32_t alo = (uint32_t)adesc, ahi = (uint32_t)(adesc >> 32);
  const uint32_t blo = (uint32_t)bdesc, bhi = (uint32_t)(bdesc >> 32);
  asm volatile(
      "{\n.reg .pred e;\n.reg .b32 al, bl;\n.reg .b64 ad, bd;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "mov.b64 ad, {%1, %2};\nmov.b64 bd, {%3, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], ad, bd, %5, 0;\n"
      "add.s32 al, %1, 2;\nadd.s32 bl, %3, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, %1, 4;\nadd.s32 bl, %3, 4;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, %1, 6;\nadd.s32 bl, %3, 6;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, %1, %6;\nadd.s32 bl, %3, %7;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, al, 2;\nadd.s32 bl, bl, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, al, 2;\nadd.s32 bl, bl, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], ad, bd, %5, 1;\n"
      "add.s32 al, al, 2;\nadd.s32 bl, bl, 2;\nmov.b64 ad, {al, %2};\nmov.b64 bd, {bl, %4};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], ad, bd, %5, 1;\n"
      "}\n" ::"r"(d),
      "r"(alo), "r"(ahi), "r"(blo), "r"(bhi), "r"(idesc), "n"(A_CH), "n"(B_CH)
      : "memory");
}
// TS group, 4 x K=16 (64 keys): A = P from TMEM (8 columns per step, both CTAs' TMEM at the same
// address), B = V MN-major SW128 (2048 B per 16 keys); acc = 0 only for the first group.
__device__ __forceinline__ void mma2_ts_k4(uint32_t d, uint32_t a_tmem, uint64_t bdesc,
                                           uint32_t idesc, uint32_t acc) {
  const uint32_t blo = (uint32_t)bdesc, bhi = (uint32_t)(bdesc >> 32);
  asm volatile(
      "{\n.reg .pred e, p;\n.reg .b32 ta, bl;\n.reg .b64 bd;\n"
      "elect.sync _|e, 0xffffffff;\n"
      "setp.ne.b32 p, %5, 0;\n"
      "mov.b64 bd, {%2, %3};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], [%1], bd, %4, p;\n"
      "add.s32 ta, %1, 8;\nadd.s32 bl, %2, 128;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 16;\nadd.s32 bl, %2, 256;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "add.s32 ta, %1, 24;\nadd.s32 bl, %2, 384;\nmov.b64 bd, {bl, %3};\n"
      "@e tcgen05.mma.cta_group::2.kind::f16 [%0], [ta], bd, %4, 1;\n"
      "}\n" ::"r"(d),
      "r"(a_tmem), "r"(blo), "r"(bhi), "r"(idesc), "r"(acc)
      : "memory");
}
// warp-wide commit of the leader's MMAs to the barrier at this offset in both CTAs
__device__ __forceinline__ void mma2_commit_w(uint64_t* bar) {
  asm volatile(
      "{\n.reg .pred e;\n.reg .b16 m;\nmov.b16 m, 3;\nelect.sync _|e, 0xffffffff;\n"
      "@e tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64"
      " [%0], m;\n}\n" ::"r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
template <int NCOLS>
__device__ __forceinline__ void tmem_alloc(uint32_t* smem_holder) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                   smem_u32(smem_holder)),
               "n"(NCOLS)
               : "memory");
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
template <int NCOLS>
__device__ __forceinline__ void tmem_dealloc(uint32_t base) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(base), "n"(NCOLS)
               : "memory");
}
__device__ __forceinline__ void tmem_wait_ld() {
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_wait_st() {
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}
// 32 lanes x 32 consecutive 32-bit columns: thread i of the warp gets lane (base lane + i).
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,"
      "%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]),
        "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]),
        "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,"
      "%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t* r) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,"
      "%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
      "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]),
      "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]),
      "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]),
      "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// Packed fp32 pair ops (sm_100 FFMA2 / FADD2): half the issue slots of two scalar ops.
__device__ __forceinline__ void ffma2(float& d0, float& d1, float a0, float a1, float b0, float b1,
                                      float c0, float c1) {
  asm("{\n.reg .b64 a, b, c, d;\nmov.b64 a, {%2, %3};\nmov.b64 b, {%4, %5};\nmov.b64 c, {%6, %7};\n"
      "fma.rn.f32x2 d, a, b, c;\nmov.b64 {%0, %1}, d;\n}\n"
      : "=f"(d0), "=f"(d1)
      : "f"(a0), "f"(a1), "f"(b0), "f"(b1), "f"(c0), "f"(c1));
}
__device__ __forceinline__ void fadd2(float& d0, float& d1, float a0, float a1, float b0, float b1) {
  asm("{\n.reg .b64 a, b, d;\nmov.b64 a, {%2, %3};\nmov.b64 b, {%4, %5};\n"
      "add.rn.f32x2 d, a, b;\nmov.b64 {%0, %1}, d;\n}\n"
      : "=f"(d0), "=f"(d1)
      : "f"(a0), "f"(a1), "f"(b0), "f"(b1));
}
// 2^x for a pair on the FMA pipe (offloads the MUFU unit, FA4-style): x = n + f, n = round(x),
// f in [-0.5, 0.5], 2^f by a degree-3 polynomial fitted for relative error on [-0.5, 0.5]
// (max 7.5e-5, far below the 2^-9 rounding of the bf16 P it feeds), then n is added to the
// exponent field.  x is clamped to >= -126 (results below 2^-126 flush towards 0; they are far
// below bf16 P resolution relative to the row max, which is >= 1).
__device__ __forceinline__ void ex2_poly2(float& x0, float& x1) {
  const float magic = 12582912.0f;                          // 1.5 * 2^23: round-to-nearest trick
  x0 = fmaxf(x0, -126.0f);
  x1 = fmaxf(x1, -126.0f);
  float r0, r1, n0, n1, f0, f1;
  fadd2(r0, r1, x0, x1, magic, magic);
  fadd2(n0, n1, r0, r1, -magic, -magic);
  fadd2(f0, f1, x0, x1, -n0, -n1);
  float p0 = 5.5171650e-2f, p1 = 5.5171650e-2f;
  ffma2(p0, p1, p0, p1, f0, f1, 2.4261113e-1f, 2.4261113e-1f);
  ffma2(p0, p1, p0, p1, f0, f1, 6.9326097e-1f, 6.9326097e-1f);
  ffma2(p0, p1, p0, p1, f0, f1, 9.9992806e-1f, 9.9992806e-1f);
  x0 = __int_as_float(__float_as_int(p0) + (__float_as_int(r0) << 23));
  x1 = __int_as_float(__float_as_int(p1) + (__float_as_int(r1) << 23));
}
// three-input max (one FMNMX3 on sm_100)
__device__ __forceinline__ float fmax3(float a, float b, float c) {
  float r;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
  return r;
}
// per-warpgroup register budget (all four warps of a warpgroup execute the same one)
template <int N>
__device__ __forceinline__ void regs_inc() {
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(N));
}
template <int N>
__device__ __forceinline__ void regs_dec() {
  asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(N));
}
__device__ __forceinline__ uint32_t pack_bf16x2_rn(float lo, float hi) {
  uint32_t r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t* r) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,"
      "%14,%15,%16};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
      "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]),
      "r"(r[15])
      : "memory");
}

}  // namespace tc

// Host: encode a 2-D bf16 tensor map (rows x cols, row pitch in bytes), box box_cols x box_rows,
// 128-byte swizzle.  Defined in tma_host.cu.
bool make_tmap_2d_bf16(CUtensorMap* map, const void* base, uint64_t rows, uint64_t cols,
                       uint64_t row_pitch_bytes, uint32_t box_cols, uint32_t box_rows);

}  // namespace fps
