// Host-link micro for the a3 cache prefetch: how fast can the unmasked rows U
// of one Flux-scale KV entry (4096 rows x 12288 B) move from pinned host DRAM to their token rows
// in HBM, and what does each method cost the compute stream?
//
// Methods (useful bytes = |U| x row):
//   whole     one cudaMemcpyAsync of the whole entry (raw bytes = all rows)
//   run_sK    one cudaMemcpyAsync per run of consecutive unmasked tokens, runs dealt round-robin
//             over K streams (K = 1, 2, 4)
//   sm_C      SM zero-copy gather: C CTAs x 256 threads, 8 x 16-B loads in flight per thread
//   tma_C_S_B TMA bulk gather: C CTAs, one thread each, S smem buffers of B bytes; each chunk of a
//             run goes host -> smem (cp.async.bulk, mbarrier) -> HBM (cp.async.bulk store)
// For each method: GB/s of useful bytes over NE entries back to back; then the same loads
// concurrent with a cuBLAS bf16 GEMM loop on another stream (GEMM slowdown vs alone).
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o h2d_gather h2d_gather.cu -lcublas
#include <cublas_v2.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <string>
#include <vector>

#define CK(x)                                                                          \
  do {                                                                                 \
    cudaError_t e_ = (x);                                                              \
    if (e_ != cudaSuccess) {                                                           \
      fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
      exit(1);                                                                         \
    }                                                                                  \
  } while (0)

static const int kRows = 4096, kRowBytes = 12288, kL = 4608;

struct Chunk {
  long long src, dst;   // byte offsets (src in the entry, dst in the slot)
  int bytes;
};

// ---- SM zero-copy gather ------------------------------------------------------------------------
__global__ void __launch_bounds__(256) sm_gather(const uint4* __restrict__ src, const int* rows, int n,
                                                 int vpr, uint4* dst) {
  const long long total = (long long)n * vpr, stride = (long long)gridDim.x * blockDim.x;
  for (long long i0 = (long long)blockIdx.x * blockDim.x + threadIdx.x; i0 < total; i0 += 8 * stride) {
    uint4 v[8];
    long long d[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const long long i = i0 + u * stride;
      d[u] = -1;
      if (i < total) {
        const int r = (int)(i / vpr), c = (int)(i - (long long)r * vpr);
        const long long row = rows[r];
        v[u] = src[row * vpr + c];
        d[u] = row * vpr + c;
      }
    }
#pragma unroll
    for (int u = 0; u < 8; ++u)
      if (d[u] >= 0) dst[d[u]] = v[u];
  }
}

// ---- TMA bulk gather --------------------------------------------------------------------------
__device__ __forceinline__ uint32_t su32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__global__ void tma_gather(const char* __restrict__ src, char* __restrict__ dst, const Chunk* chunks,
                           int n_chunks, int S, int B) {
  extern __shared__ __align__(128) char sm[];
  uint64_t* bar = reinterpret_cast<uint64_t*>(sm);
  char* buf = sm + 128;
  if (threadIdx.x != 0) return;
  for (int i = 0; i < S; ++i)
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(bar + i)));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  // this CTA's chunks: blockIdx.x, blockIdx.x + gridDim.x, ...
  const int mine = n_chunks > (int)blockIdx.x ? (n_chunks - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  auto load = [&](int k) {
    const Chunk c = chunks[blockIdx.x + (long long)k * gridDim.x];
    const int b = k % S;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(bar + b)),
                 "r"(c.bytes)
                 : "memory");
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            su32(buf + (size_t)b * B)),
        "l"(src + c.src), "r"(c.bytes), "r"(su32(bar + b))
        : "memory");
  };
  for (int k = 0; k < (S < mine ? S : mine); ++k) load(k);
  for (int k = 0; k < mine; ++k) {
    const int b = k % S;
    const uint32_t ph = (k / S) & 1;
    asm volatile(
        "{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W;\n}\n" ::"r"(
            su32(bar + b)),
        "r"(ph)
        : "memory");
    const Chunk c = chunks[blockIdx.x + (long long)k * gridDim.x];
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + c.dst),
                 "r"(su32(buf + (size_t)b * B)), "r"(c.bytes)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    // refill the previous chunk's buffer once its store has read smem (this one may still run)
    if (k >= 1 && k - 1 + S < mine) {
      asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      load(k - 1 + S);
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// ---- masks ---------------------------------------------------------------------------------
static std::vector<int> unmasked_rows(const char* kind, double m, unsigned seed) {
  std::vector<char> masked(kRows, 0);
  const int want = (int)(m * kRows + 0.5);
  std::mt19937 g(seed);
  if (!strcmp(kind, "random")) {
    std::vector<int> p(kRows);
    for (int i = 0; i < kRows; ++i) p[i] = i;
    std::shuffle(p.begin(), p.end(), g);
    for (int i = 0; i < want; ++i) masked[p[i]] = 1;
  } else {   // blob: tokens nearest to a random centre on the 64 x 64 grid (a disc)
    const double cx = 20 + g() % 24, cy = 20 + g() % 24;
    std::vector<std::pair<double, int>> d(kRows);
    for (int i = 0; i < kRows; ++i) {
      const double x = i % 64, y = i / 64;
      d[i] = {(x - cx) * (x - cx) + 1.3 * (y - cy) * (y - cy), i};
    }
    std::sort(d.begin(), d.end());
    for (int i = 0; i < want; ++i) masked[d[i].second] = 1;
  }
  std::vector<int> u;
  for (int i = 0; i < kRows; ++i)
    if (!masked[i]) u.push_back(i);
  return u;
}

struct Run {
  long long off;
  long long bytes;
};
static std::vector<Run> runs_of(const std::vector<int>& u) {
  std::vector<Run> r;
  for (size_t j = 0; j < u.size();) {
    size_t k = j;
    while (k + 1 < u.size() && u[k + 1] == u[k] + 1) ++k;
    r.push_back({(long long)u[j] * kRowBytes, (long long)(k - j + 1) * kRowBytes});
    j = k + 1;
  }
  return r;
}

int main(int argc, char** argv) {
  const int NE = argc > 1 ? atoi(argv[1]) : 24;
  const double m = argc > 2 ? atof(argv[2]) : 0.2;
  const size_t entry = (size_t)kRows * kRowBytes;
  char* host;
  CK(cudaHostAlloc((void**)&host, NE * entry, cudaHostAllocMapped | cudaHostAllocPortable));
  memset(host, 1, NE * entry);
  char* hdev;
  CK(cudaHostGetDevicePointer((void**)&hdev, host, 0));
  char* slot;
  CK(cudaMalloc(&slot, (size_t)kL * kRowBytes));
  const int NS = 4;
  cudaStream_t ls[NS], cs;
  for (int i = 0; i < NS; ++i) CK(cudaStreamCreateWithFlags(&ls[i], cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, g0, g1, join[NS];
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaEventCreate(&g0));
  CK(cudaEventCreate(&g1));
  for (int i = 0; i < NS; ++i) CK(cudaEventCreateWithFlags(&join[i], cudaEventDisableTiming));
  // GEMM for the interference test: 4608 x 3072 x 12288 bf16 (about the Flux MLP-down shape)
  cublasHandle_t cb;
  cublasCreate(&cb);
  cublasSetStream(cb, cs);
  const int GM = 4608, GN = 3072, GK = 12288;
  __nv_bfloat16 *A, *Bm, *C;
  CK(cudaMalloc(&A, (size_t)GM * GK * 2));
  CK(cudaMalloc(&Bm, (size_t)GN * GK * 2));
  CK(cudaMalloc(&C, (size_t)GM * GN * 2));
  CK(cudaMemset(A, 0, (size_t)GM * GK * 2));
  CK(cudaMemset(Bm, 0, (size_t)GN * GK * 2));
  const float one = 1.f, zero = 0.f;
  auto gemm = [&](int reps) {
    for (int i = 0; i < reps; ++i)
      cublasGemmEx(cb, CUBLAS_OP_T, CUBLAS_OP_N, GN, GM, GK, &one, Bm, CUDA_R_16BF, GK, A, CUDA_R_16BF,
                   GK, &zero, C, CUDA_R_16BF, GN, CUBLAS_COMPUTE_32F, CUBLAS_GEMM_DEFAULT);
  };
  gemm(5);
  CK(cudaStreamSynchronize(cs));
  const int GREPS = 100;
  CK(cudaEventRecord(g0, cs));
  gemm(GREPS);
  CK(cudaEventRecord(g1, cs));
  CK(cudaEventSynchronize(g1));
  float gemm_alone;
  CK(cudaEventElapsedTime(&gemm_alone, g0, g1));
  printf("gemm alone: %.3f ms per GEMM (%.0f TF/s)\n", gemm_alone / GREPS,
         2.0 * GM * GN * GK / (gemm_alone / GREPS * 1e-3) / 1e12);

  for (const char* kind : {"blob", "random"}) {
    const std::vector<int> u = unmasked_rows(kind, m, 7);
    const std::vector<Run> runs = runs_of(u);
    const double useful = (double)u.size() * kRowBytes;
    int* d_rows;
    CK(cudaMalloc(&d_rows, u.size() * 4));
    CK(cudaMemcpy(d_rows, u.data(), u.size() * 4, cudaMemcpyHostToDevice));
    printf("\nmask %s m=%.2f: |U| = %zu rows, %zu runs, useful %.1f MB per entry\n", kind, m, u.size(),
           runs.size(), useful / 1e6);
    struct Method {
      std::string name;
      int kind, a, b, c;   // 0 whole, 1 runs(a streams), 2 sm(a ctas), 3 tma(a ctas, b stages, c bytes)
    };
    std::vector<Method> ms = {{"whole", 0, 0, 0, 0},     {"run_s1", 1, 1, 0, 0},
                              {"run_s2", 1, 2, 0, 0},    {"run_s4", 1, 4, 0, 0},
                              {"sm_8", 2, 8, 0, 0},      {"sm_16", 2, 16, 0, 0},
                              {"sm_32", 2, 32, 0, 0}};
    for (int ctas : {1, 2, 4, 8, 16})
      for (int S : {2, 3, 4})
        for (int Bb : {8192, 12288})
          ms.push_back({"tma_" + std::to_string(ctas) + "_" + std::to_string(S) + "_" + std::to_string(Bb),
                        3, ctas, S, Bb});
    for (const Method& me : ms) {
      // chunks for TMA: runs split at B bytes
      Chunk* d_chunks = nullptr;
      int n_chunks = 0;
      if (me.kind == 3) {
        std::vector<Chunk> ch;
        for (const Run& r : runs)
          for (long long o = 0; o < r.bytes; o += me.c)
            ch.push_back({r.off + o, r.off + o, (int)std::min<long long>(me.c, r.bytes - o)});
        n_chunks = (int)ch.size();
        CK(cudaMalloc(&d_chunks, ch.size() * sizeof(Chunk)));
        CK(cudaMemcpy(d_chunks, ch.data(), ch.size() * sizeof(Chunk), cudaMemcpyHostToDevice));
        CK(cudaFuncSetAttribute(tma_gather, cudaFuncAttributeMaxDynamicSharedMemorySize, 128 + me.b * me.c));
      }
      double host_us = 0;
      auto one_entry = [&](int e) {
        const char* src = host + (size_t)e * entry;
        const char* srcd = hdev + (size_t)e * entry;
        auto t0 = std::chrono::steady_clock::now();
        if (me.kind == 0) {
          CK(cudaMemcpyAsync(slot, src, entry, cudaMemcpyHostToDevice, ls[0]));
        } else if (me.kind == 1) {
          for (int k = 1; k < me.a; ++k) {
            CK(cudaEventRecord(join[0], ls[0]));
            CK(cudaStreamWaitEvent(ls[k], join[0], 0));
          }
          for (size_t q = 0; q < runs.size(); ++q)
            CK(cudaMemcpyAsync(slot + runs[q].off, src + runs[q].off, runs[q].bytes,
                               cudaMemcpyHostToDevice, ls[q % me.a]));
          for (int k = 1; k < me.a; ++k) {
            CK(cudaEventRecord(join[k], ls[k]));
            CK(cudaStreamWaitEvent(ls[0], join[k], 0));
          }
        } else if (me.kind == 2) {
          sm_gather<<<me.a, 256, 0, ls[0]>>>((const uint4*)srcd, d_rows, (int)u.size(), kRowBytes / 16,
                                             (uint4*)slot);
        } else {
          tma_gather<<<me.a, 32, 128 + me.b * me.c, ls[0]>>>(srcd, slot, d_chunks, n_chunks, me.b, me.c);
        }
        host_us += std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count();
      };
      for (int e = 0; e < 2; ++e) one_entry(e);
      CK(cudaStreamSynchronize(ls[0]));
      CK(cudaGetLastError());
      host_us = 0;
      CK(cudaEventRecord(e0, ls[0]));
      for (int e = 0; e < NE; ++e) one_entry(e);
      CK(cudaEventRecord(e1, ls[0]));
      CK(cudaEventSynchronize(e1));
      float ms_alone;
      CK(cudaEventElapsedTime(&ms_alone, e0, e1));
      // concurrent with the GEMM loop
      CK(cudaDeviceSynchronize());
      CK(cudaEventRecord(g0, cs));
      gemm(GREPS);
      CK(cudaEventRecord(g1, cs));
      CK(cudaEventRecord(e0, ls[0]));
      for (int e = 0; e < NE; ++e) one_entry(e % NE);
      CK(cudaEventRecord(e1, ls[0]));
      CK(cudaDeviceSynchronize());
      CK(cudaGetLastError());
      float ms_conc, gemm_conc;
      CK(cudaEventElapsedTime(&ms_conc, e0, e1));
      CK(cudaEventElapsedTime(&gemm_conc, g0, g1));
      // GEMM slowdown over the overlapped window only: compare per-GEMM time when the loads end
      // before the GEMMs (normally they do: NE entries ~ 20-30 ms, 40 GEMMs ~ 40 ms)
      printf("%-16s alone %7.3f ms/entry %6.1f GB/s useful | host %6.1f us/entry | with GEMM %6.1f GB/s, "
             "GEMM %.3f ms (x%.3f)\n",
             me.name.c_str(), ms_alone / NE, useful * NE / (ms_alone * 1e-3) / 1e9, host_us / NE / 2,
             useful * NE / (ms_conc * 1e-3) / 1e9, gemm_conc / GREPS, gemm_conc / gemm_alone);
      if (d_chunks) CK(cudaFree(d_chunks));
    }
    CK(cudaFree(d_rows));
  }
  return 0;
}
