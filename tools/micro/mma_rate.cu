// Microbenchmark: back-to-back tcgen05.mma issue rate from one warp for several N (M = 128,
// K = 16 bf16 per instruction, operands in smem, accumulator in TMEM).  Developer tool.
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_eurosys_jianglyfdlzllyl26_b200/csrc/tc_util.cuh"
using namespace fps;

template <int N, int GROUPS, int GROUPED>
__global__ void k_rate(long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* base = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  uint64_t* bar = reinterpret_cast<uint64_t*>(base + 96 * 1024);
  uint32_t* holder = reinterpret_cast<uint32_t*>(bar + 2);
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) { tc::mbar_init(bar, 1); tc::fence_mbar_init(); }
  if (warp == 0) tc::tmem_alloc<512>(holder);
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  if (warp == 1) {
    constexpr uint32_t idesc = tc::idesc_bf16(128, N);
    const uint64_t da = tc::sdesc_k_sw128(tc::smem_u32(base));
    const uint64_t db = tc::sdesc_k_sw128(tc::smem_u32(base + 32768));
    long long t0 = clock64();
    for (int g = 0; g < GROUPS; ++g) {
      if (GROUPED == 2) {
        constexpr uint32_t idesc_mn = tc::idesc_bf16(128, N, true);
        tc::mma_ts_k8(256, 0, tc::sdesc_mn_sw128(tc::smem_u32(base + 32768), 16384), idesc_mn, g > 0);
        tc::mma_commit_w(bar);
      } else if (GROUPED) {
        tc::mma_ss_k8_commit<1024, 1024>((g & 1) * 256, da, db, idesc, bar);
      } else {
        for (int ks = 0; ks < 8; ++ks)
          tc::mma_bf16_w((g & 1) * 256, da + ks * 2, db + ks * 2, idesc, ks > 0);
        tc::mma_commit_w(bar);
      }
    }
    long long t1 = clock64();
    tc::mbar_wait(bar, (GROUPS - 1) & 1);
    long long t2 = clock64();
    if ((threadIdx.x & 31) == 0 && blockIdx.x == 0) { out[0] = t1 - t0; out[1] = t2 - t0; }
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 0) { tc::fence_after(); tc::tmem_dealloc<512>(0); }
}

template <int N, int G>
void run(long long* d) {
  constexpr int GR = 64;
  cudaFuncSetAttribute(k_rate<N, GR, G>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  long long h[2];
  for (int it = 0; it < 3; ++it) {
    k_rate<N, GR, G><<<148, 128, 100 * 1024>>>(d);
    cudaDeviceSynchronize();
  }
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  const double ideal = GR * 8.0 * 128 * N * 16 / 4096.0;   // cycles at 4096 MAC/clk
  printf("N=%3d grouped=%d: issue %lld cyc, done %lld cyc for %d MMAs -> %.1f cyc/MMA (ideal %.1f), %.0f%% of peak\n",
         N, G, h[0], h[1], GR * 8, (double)h[1] / (GR * 8), ideal / (GR * 8), 100.0 * ideal / h[1]);
}

int main() {
  long long* d;
  cudaMalloc(&d, 64);
  run<64, 1>(d); run<128, 1>(d); run<256, 1>(d);
  run<64, 0>(d); run<128, 0>(d); run<256, 0>(d);
  run<64, 2>(d); run<128, 2>(d); run<256, 2>(d);
  printf("%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
