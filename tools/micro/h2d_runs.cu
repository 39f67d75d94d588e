// Microbenchmark: host->device copy of the unmasked rows of KV cache entries (C3 shapes: 4096
// rows x 12288 B per entry, a disc-shaped mask of 819 tokens on the 64x64 grid) by
//   whole   one DMA per entry (masked rows copied too)
//   runs    one cudaMemcpyAsync per run of unmasked rows
//   batch   cudaMemcpyBatchAsync of all runs of an entry
// Reports host API time, device time and the bytes moved; verifies the batch copy.  Dev tool.
#include <chrono>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

int main() {
  const int R = 4096, RB = 12288, NE = 8, ITER = 40;
  const size_t EB = (size_t)R * RB;
  char *h, *d;
  CK(cudaHostAlloc(&h, EB * NE, cudaHostAllocMapped));
  CK(cudaMalloc(&d, EB * NE));
  for (size_t i = 0; i < EB * NE; i += 4096) h[i] = (char)(i / 4096 * 7 + 1);
  std::vector<char> masked(R, 0);
  int nm = 0;
  for (int y = 0; y < 64; ++y)
    for (int x = 0; x < 64; ++x) {
      const float dx = x - 30.5f, dy = y - 33.5f;
      if (dx * dx + dy * dy < 16.15f * 16.15f) { masked[y * 64 + x] = 1; ++nm; }
    }
  std::vector<std::pair<int, int>> runs;   // (start row, rows)
  for (int i = 0; i < R;) {
    if (masked[i]) { ++i; continue; }
    int j = i;
    while (j < R && !masked[j]) ++j;
    runs.push_back({i, j - i});
    i = j;
  }
  printf("masked %d rows, %zu unmasked runs\n", nm, runs.size());
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  std::vector<void*> dsts, srcs;
  std::vector<size_t> sizes;
  for (int mode = 0; mode < 3; ++mode) {
    if (getenv("ONLY_VERIFY")) break;
    for (int rep = 0; rep < 2; ++rep) {
      double host_us = 0, bytes = 0;
      CK(cudaStreamSynchronize(s));
      cudaEventRecord(e0, s);
      for (int it = 0; it < ITER; ++it) {
        const int e = it % NE;
        char* hs = h + e * EB;
        char* dd = d + e * EB;
        auto t0 = std::chrono::steady_clock::now();
        if (mode == 0) {
          CK(cudaMemcpyAsync(dd, hs, EB, cudaMemcpyHostToDevice, s));
          bytes += EB;
        } else if (mode == 1) {
          for (auto& r : runs) {
            CK(cudaMemcpyAsync(dd + (size_t)r.first * RB, hs + (size_t)r.first * RB,
                               (size_t)r.second * RB, cudaMemcpyHostToDevice, s));
            bytes += (double)r.second * RB;
          }
        } else {
          dsts.clear(); srcs.clear(); sizes.clear();
          for (auto& r : runs) {
            dsts.push_back(dd + (size_t)r.first * RB);
            srcs.push_back(hs + (size_t)r.first * RB);
            sizes.push_back((size_t)r.second * RB);
            bytes += (double)r.second * RB;
          }
          cudaMemcpyAttributes a{};
          a.srcAccessOrder = cudaMemcpySrcAccessOrderStream;
          a.srcLocHint.type = cudaMemLocationTypeHost;
          a.dstLocHint.type = cudaMemLocationTypeDevice;
          a.dstLocHint.id = 0;
          a.flags = cudaMemcpyFlagPreferOverlapWithCompute;
          size_t idx = 0, fail = ~size_t(0);
          CK(cudaMemcpyBatchAsync(dsts.data(), srcs.data(), sizes.data(), dsts.size(), &a, &idx, 1,
                                  &fail, s));
        }
        host_us += std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count();
      }
      cudaEventRecord(e1, s);
      CK(cudaStreamSynchronize(s));
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      printf("%-5s: %6.2f ms per entry (device), host %7.1f us per entry, %5.1f GB/s of copied bytes, "
             "%5.1f GB/s of unmasked bytes\n",
             mode == 0 ? "whole" : mode == 1 ? "runs" : "batch", ms / ITER, host_us / ITER,
             bytes / (ms * 1e6), (double)(R - nm) * RB * ITER / (ms * 1e6));
    }
  }
  // verify: clear device, batch-copy entry 3, compare unmasked rows
  CK(cudaMemset(d, 0, EB * NE));
  CK(cudaDeviceSynchronize());
  {
    dsts.clear(); srcs.clear(); sizes.clear();
    for (auto& r : runs) {
      dsts.push_back(d + 3 * EB + (size_t)r.first * RB);
      srcs.push_back(h + 3 * EB + (size_t)r.first * RB);
      sizes.push_back((size_t)r.second * RB);
    }
    cudaMemcpyAttributes a{};
    a.srcAccessOrder = cudaMemcpySrcAccessOrderStream;
    a.flags = cudaMemcpyFlagPreferOverlapWithCompute;
    size_t idx = 0, fail = ~size_t(0);
    CK(cudaMemcpyBatchAsync(dsts.data(), srcs.data(), sizes.data(), dsts.size(), &a, &idx, 1, &fail, s));
    CK(cudaStreamSynchronize(s));
    std::vector<char> back(EB);
    CK(cudaMemcpy(back.data(), d + 3 * EB, EB, cudaMemcpyDeviceToHost));
    long bad = 0;
    for (int i = 0; i < R; ++i)
      if (!masked[i] && memcmp(back.data() + (size_t)i * RB, h + 3 * EB + (size_t)i * RB, RB)) ++bad;
    printf("batch verify: %ld bad rows of %d\n", bad, R - nm);
  }
  return 0;
}
