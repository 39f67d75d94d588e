// Throughput of ex2.approx.f32 vs ex2.approx.f16x2 on one B200 (exponentials per clock per SM).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ex2_rate ex2_rate.cu && ./ex2_rate
#include <cuda_fp16.h>
#include <cstdio>

__global__ void k_f32(float* out, int iters) {
  float v[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = -0.001f * (threadIdx.x + i);
  for (int it = 0; it < iters; ++it)
#pragma unroll
    for (int i = 0; i < 8; ++i) asm volatile("ex2.approx.ftz.f32 %0, %0;" : "+f"(v[i]));
  float s = 0.f;
  for (int i = 0; i < 8; ++i) s += v[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_f16x2(float* out, int iters) {
  unsigned v[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    __half2 h = __floats2half2_rn(-0.001f * (threadIdx.x + i), -0.002f * i);
    v[i] = *reinterpret_cast<unsigned*>(&h);
  }
  for (int it = 0; it < iters; ++it)
#pragma unroll
    for (int i = 0; i < 8; ++i) asm volatile("ex2.approx.f16x2 %0, %0;" : "+r"(v[i]));
  float s = 0.f;
  for (int i = 0; i < 8; ++i) s += __half2float(reinterpret_cast<__half2*>(&v[i])->x);
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

int main() {
  int sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  float* out;
  cudaMalloc(&out, sms * 8 * 256 * sizeof(float));
  const int iters = 4096;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int kind = 0; kind < 2; ++kind) {
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(a);
      if (kind == 0) k_f32<<<sms * 8, 256>>>(out, iters);
      else k_f16x2<<<sms * 8, 256>>>(out, iters);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
    }
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    const double ops = (double)sms * 8 * 256 * iters * 8 * (kind ? 2 : 1);   // exponentials
    printf("%s: %.3f ms, %.1f exp/clk/SM (at %.0f MHz nominal max)\n", kind ? "ex2.f16x2" : "ex2.f32",
           ms, ops / (ms * 1e-3) / sms / (clk * 1e3), clk / 1e3);
  }
  return 0;
}
