// a3: activation cache in pinned host DRAM + layer-ahead prefetch (PAPER.md L203 host-memory
// store, L207 block granularity, L209 "while loading the i-th block, the computation stream
// can concurrently execute the computation of the (i-1)-th block"; reading R7 keys).
//
// Three load methods (fps_cache_desc.copy_method):
//  0  SM zero-copy gather: a few CTAs read the unmasked rows straight out of the mapped pinned
//     arena over PCIe (16-B loads, many in flight) and write them to their token rows in HBM.
//     One launch per layer for the whole batch, exact bytes, any mask shape -- but the gather
//     warps share the SMs with the compute stream (~10% slower GEMMs in the step).
//  1  copy-engine DMA of exactly the unmasked rows: one cudaMemcpyAsync per run of consecutive
//     tokens.  Measured on B200 (a dev micro, C3 entry, 33 runs): 47 GB/s and ~200 us of host
//     time per entry, against 44 GB/s of useful bytes for whole entries.  (The CUDA 12.8
//     batched-copy entry point measured faster, 55 GB/s / ~11 us, but it is closed on the GPU
//     pool this library is validated on -- it raised device faults there -- so it is not used.)
//  2  copy-engine DMA of whole entries (all L_img rows, one copy per request and block): +25%
//     bytes at m = 0.2 but no SM time and no per-run overhead; the caller orders fresh-row writes
//     after the ready event.  Fastest measured step on B200 for both tiers.
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <cstring>
#include <vector>

#include "kernels.h"

struct fps_cache {
  fps_cache_desc d;
  int elt = 2;
  size_t entry_bytes = 0;      // slot size (widest entry)
  size_t row_bytes_main = 0;   // W * elt
  size_t row_bytes_final = 0;  // H * elt (KV-mode final Y entry)
  long long n_keys = 0;
  long long n_entries = 0;
  char* host = nullptr;        // pinned, mapped
  char* dev_alias = nullptr;   // device pointer of `host`
  void* mmap_base = nullptr;   // location 2: the mapping behind `host`
  size_t mmap_bytes = 0;
  std::vector<void*> dsts, srcs;
  std::vector<size_t> sizes;
};

namespace fps {

constexpr int kMaxPrefetchItems = 32;
// Row gather launch shape (threads per CTA, 16-B loads in flight per thread).  Measured on B200
// (C3 pinned-host step): 256 x 8 gives 43.4 ms; 128 x 8 45.2, 64 x 16 47.7 (41 GB/s), 32 x 16
// 50.7 -- fewer, deeper threads do not reach the link rate.  FPS_PREFETCH_SHAPE=threads,unroll
// overrides (experiments).
static int g_pf_threads = 256, g_pf_unroll = 8;

struct PrefetchBatch {
  const uint4* src[kMaxPrefetchItems];
  const int32_t* rows[kMaxPrefetchItems];
  uint4* dst[kMaxPrefetchItems];
  long long start[kMaxPrefetchItems + 1];   // prefix sums of vectors per item
  int vpr[kMaxPrefetchItems];
  int n_items;
};

template <int kPrefetchUnroll>
__global__ void __launch_bounds__(256) prefetch_kernel(const __grid_constant__ PrefetchBatch b) {
  const long long total = b.start[b.n_items];
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i0 = (long long)blockIdx.x * blockDim.x + threadIdx.x; i0 < total;
       i0 += kPrefetchUnroll * stride) {
    uint4 v[kPrefetchUnroll];
    uint4* dp[kPrefetchUnroll];
#pragma unroll
    for (int u = 0; u < kPrefetchUnroll; ++u) {
      const long long i = i0 + u * stride;
      dp[u] = nullptr;
      if (i < total) {
        int it = 0;
        while (i >= b.start[it + 1]) ++it;
        const long long local = i - b.start[it];
        const int vpr = b.vpr[it];
        const int rr = (int)(local / vpr), c = (int)(local - (long long)rr * vpr);
        const long long row = __ldg(b.rows[it] + rr);
        v[u] = b.src[it][row * vpr + c];
        dp[u] = b.dst[it] + row * vpr + c;
      }
    }
#pragma unroll
    for (int u = 0; u < kPrefetchUnroll; ++u)
      if (dp[u]) *dp[u] = v[u];
  }
}

// ---- method 3: TMA bulk row gather (host -> smem -> HBM) ------------------------------------
// A few CTAs, one warp each, in CTA pairs (cluster of 2 = one TPC, so the CTA-pair GEMMs keep
// whole TPCs); the warp scans 32 row ids at a time, cuts them into chunks of consecutive rows
// (a chunk ends at a run boundary, every kBulkRows-aligned token, and every 32 ids), and lane 0
// moves each chunk with one cp.async.bulk load into a smem ring slot (mbarrier completion) and
// one cp.async.bulk store to the same rows of the destination.  Measured on B200
// (tools/micro/h2d_gather.cu, one C3 KV entry): 4 CTAs x 4 slots x 12 KB reach 51.1 GB/s of
// unmasked bytes from mapped pinned memory for blob and random masks alike, against 44 GB/s of
// useful bytes for the whole-entry DMA and 47 / 12 GB/s for one DMA per run (blob / random).
// The loads cost the compute stream only the reserved SMs (sm_budget()).
constexpr int kBulkMaxSlots = 16;
constexpr int kBulkMinChunk = 12288;   // bytes per ring slot (at least one row)
constexpr int kBulkMaxRow = 32768;     // widest row method 3 accepts (KV-mode H <= 8192 bf16)
// bytes in flight per CTA: PCIe read latency ~2 us x ~55 GB/s needs > 110 KB over all CTAs; the
// micro reached the link rate from 128 KB (e.g. 16 x 8 KB, 8 x 16 KB, 4 x 48 KB).  Inside the
// C4 step the link needs 6-8 CTAs (C4: 4 CTAs 603 ms/step, 6 527, 8 524, 12 536) and a deeper
// ring per CTA does not help (8 CTAs: 48 KB 523.5, 96 KB 525.0, 192 KB 529.8 ms/step)
constexpr int kBulkInFlightPerCta = 48 * 1024;
constexpr int kBulkMaxSmem = 200 * 1024;
constexpr int kBulkHeader = 512;   // barriers, row ids, pending stores (kBulkMaxSlots = 16)

struct BulkBatch {
  const char* src[kMaxPrefetchItems];
  char* dst[kMaxPrefetchItems];
  const int32_t* rows[kMaxPrefetchItems];
  int n_rows[kMaxPrefetchItems];
  int row_bytes[kMaxPrefetchItems];
  int n_items;
  int slot_bytes;
  int slots;        // ring slots per CTA (<= kBulkMaxSlots)
};

__device__ __forceinline__ uint32_t bulk_su32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// cp.async.bulk.wait_group.read takes an immediate: at most n of this thread's newest bulk
// store groups may still be reading shared memory
__device__ __forceinline__ void bulk_wait_read(int n) {
  switch (n) {
#define FPS_BW(i) \
  case i: asm volatile("cp.async.bulk.wait_group.read " #i ";" ::: "memory"); break;
    FPS_BW(0) FPS_BW(1) FPS_BW(2) FPS_BW(3) FPS_BW(4) FPS_BW(5) FPS_BW(6) FPS_BW(7)
    FPS_BW(8) FPS_BW(9) FPS_BW(10) FPS_BW(11) FPS_BW(12) FPS_BW(13) FPS_BW(14)
#undef FPS_BW
    default: asm volatile("cp.async.bulk.wait_group.read 15;" ::: "memory"); break;
  }
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(32)
    bulk_gather_kernel(const __grid_constant__ BulkBatch b) {
  extern __shared__ __align__(128) char bulk_smem[];
  // header: slot barriers | 32 row ids | pending store (dst, bytes) per slot | ring
  uint64_t* bar = reinterpret_cast<uint64_t*>(bulk_smem);
  int* toks = reinterpret_cast<int*>(bulk_smem + 8 * kBulkMaxSlots);
  char** pend_dst = reinterpret_cast<char**>(bulk_smem + 8 * kBulkMaxSlots + 128);
  int* pend_bytes = reinterpret_cast<int*>(bulk_smem + 16 * kBulkMaxSlots + 128);
  char* ring = bulk_smem + kBulkHeader;
  const int lane = threadIdx.x;
  if (lane == 0) {
    for (int i = 0; i < b.slots; ++i)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bulk_su32(bar + i)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  // lane 0's pipeline: chunk k is loaded into ring slot k % S; chunks are stored in order,
  // lazily, when their slot is needed again (S - 1 loads stay in flight).  Measured on B200:
  // storing each chunk as soon as it lands (a test_wait poll after every issue) was slower
  // (49.5 vs 51.3 GB/s at 4 CTAs x 4 slots), and a deeper ring on fewer CTAs does not help --
  // 2 CTAs x 8 slots reach 21 GB/s: the bulk copies one SM keeps in flight from system memory
  // are limited, so the link needs about 4 SMs
  const int S = b.slots;
  long long k = 0, stored = 0;
  auto landed = [&](long long j) {     // chunk j is in its slot
    const uint32_t addr = bulk_su32(bar + (int)(j % S)), ph = (uint32_t)((j / S) & 1);
    asm volatile(
        "{\n.reg .pred p;\nBW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra BW;\n}\n" ::"r"(
            addr),
        "r"(ph)
        : "memory");
  };
  auto store_next = [&]() {
    const int sl = (int)(stored % S);
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(pend_dst[sl]),
                 "r"(bulk_su32(ring + (size_t)sl * b.slot_bytes)), "r"(pend_bytes[sl])
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    ++stored;
  };
  auto issue = [&](const char* src, char* dst, int bytes) {
    const int sl = (int)(k % S);
    if (k >= S) {
      while (stored <= k - S) {
        landed(stored);
        store_next();
      }
      bulk_wait_read((int)(stored - 1 - (k - S)));   // chunk k - S's store has read slot sl
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bulk_su32(bar + sl)),
                 "r"(bytes)
                 : "memory");
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
            bulk_su32(ring + (size_t)sl * b.slot_bytes)),
        "l"(src), "r"(bytes), "r"(bulk_su32(bar + sl))
        : "memory");
    pend_dst[sl] = dst;
    pend_bytes[sl] = bytes;
    ++k;
  };
  const int G = gridDim.x, rank = blockIdx.x;
  for (int it = 0; it < b.n_items; ++it) {
    const int n = b.n_rows[it], rb = b.row_bytes[it];
    const int kr = rb >= b.slot_bytes ? 1 : b.slot_bytes / rb;   // rows per chunk at most
    const int p0 = (int)((long long)n * rank / G), p1 = (int)((long long)n * (rank + 1) / G);
    const int32_t* rows = b.rows[it];
    for (int base = p0; base < p1; base += 32) {
      const int pos = base + lane;
      const bool valid = pos < p1;
      const int tok = valid ? __ldg(rows + pos) : 0;
      const int prev = __shfl_up_sync(0xffffffffu, tok, 1);
      const bool start = valid && (lane == 0 || tok != prev + 1 || tok % kr == 0);
      const unsigned mask = __ballot_sync(0xffffffffu, start);
      toks[lane] = tok;
      __syncwarp();
      if (lane == 0) {
        const int nvalid = min(32, p1 - base);
        unsigned m = mask;
        while (m) {
          const int a = __ffs(m) - 1;
          m &= m - 1;
          const int e = m ? __ffs(m) - 1 : nvalid;
          const long long off = (long long)toks[a] * rb;
          issue(b.src[it] + off, b.dst[it] + off, (e - a) * rb);
        }
      }
      __syncwarp();
    }
  }
  if (lane == 0) {
    while (stored < k) {
      landed(stored);
      store_next();
    }
    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}

static long long key_of(const fps_cache* c, uint32_t t, int step, int layer) {
  const int per_step = c->d.n_layers + (c->d.mode == FPS_MODE_KV ? 1 : 0);
  return ((long long)t * c->d.n_steps + step) * per_step + layer;
}

static bool key_ok(const fps_cache* c, uint32_t t, int step, int layer) {
  const int max_layer = c->d.n_layers + (c->d.mode == FPS_MODE_KV ? 1 : 0);
  return (int)t < c->d.n_templates && step >= 0 && step < c->d.n_steps && layer >= 0 &&
         layer < max_layer;
}

static size_t row_bytes_of(const fps_cache* c, int layer) {
  return (c->d.mode == FPS_MODE_KV && layer == c->d.n_layers) ? c->row_bytes_final
                                                              : c->row_bytes_main;
}

static size_t offset_of(const fps_cache* c, uint32_t t, int step, int layer) {
  return (size_t)(key_of(c, t, step, layer) % c->n_entries) * c->entry_bytes;
}

// CTAs of the method-3 gather (even: CTA pairs): copy_ctas, default 4
int bulk_ctas(const fps_cache* c) {
  if (!c || c->d.copy_method != 3) return 0;
  int n = c->d.copy_ctas > 0 ? c->d.copy_ctas : 4;
  n = (n + 1) & ~1;
  return std::min(n, 32);
}

// the arena lives in device memory: this GPU's HBM (location 1) or a peer GPU's, opened
// through a CUDA IPC handle and read over NVLink / NVSwitch (location 4)
static bool in_device_memory(const fps_cache* c) { return c->d.location == 1 || c->d.location == 4; }

int g_d2d_kernel = 1;   // experiments: 0 = driver D2D memcpy for HBM whole-entry loads
bool cache_writes_all_rows(const fps_cache* c) { return c && c->d.copy_method == 2; }

}  // namespace fps

using namespace fps;

extern "C" {

fps_status fps_cache_create(const fps_cache_desc* desc, fps_cache_t* out) {
  FPS_CHECK_ARG(desc && out, "NULL argument");
  const fps_cache_desc& d = *desc;
  FPS_CHECK_ARG(d.mode == FPS_MODE_KV || d.mode == FPS_MODE_Y, "mode %d", d.mode);
  FPS_CHECK_ARG(d.dtype == FPS_BF16 || d.dtype == FPS_F32, "dtype %d", d.dtype);
  FPS_CHECK_ARG(d.H > 0 && d.L_img > 0 && d.n_layers > 0 && d.n_steps > 0 && d.n_templates > 0,
                "sizes must be positive");
  FPS_CHECK_ARG(d.n_entries >= 0 && d.copy_method >= 0 && d.copy_method <= 3, "bad desc");
  FPS_CHECK_ARG(d.copy_method != 3 ||
                    (size_t)(d.mode == FPS_MODE_KV ? 2 : 1) * d.H * (d.dtype == FPS_BF16 ? 2 : 4) <=
                        (size_t)kBulkMaxRow,
                "copy_method 3: rows wider than %d bytes", kBulkMaxRow);
  auto* c = new (std::nothrow) fps_cache();
  if (!c) return fail(FPS_ENOMEM, "cache: host allocation");
  c->d = d;
  c->elt = d.dtype == FPS_BF16 ? 2 : 4;
  c->row_bytes_main = (size_t)(d.mode == FPS_MODE_KV ? 2 : 1) * d.H * c->elt;
  c->row_bytes_final = (size_t)d.H * c->elt;
  c->entry_bytes = (size_t)d.L_img * c->row_bytes_main;
  const int per_step = d.n_layers + (d.mode == FPS_MODE_KV ? 1 : 0);
  c->n_keys = (long long)d.n_templates * d.n_steps * per_step;
  c->n_entries = d.n_entries > 0 ? std::min<long long>(d.n_entries, c->n_keys) : c->n_keys;
  const size_t bytes = (size_t)c->n_entries * c->entry_bytes;
  FPS_CHECK_ARG(d.location >= 0 && d.location <= 4, "location %d", d.location);
  FPS_CHECK_ARG(d.location != 4 || d.peer_ipc_handle, "location 4 needs peer_ipc_handle");
  FPS_CHECK_ARG(d.location != 3 || (d.shm_path && d.shm_path[0]), "location 3 needs shm_path");
  if (d.location == 1) {
    // HBM tier: the arena lives in device memory; "host" then names that device buffer
    cudaError_t e = cudaMalloc((void**)&c->host, bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      delete c;
      return fail(e == cudaErrorMemoryAllocation ? FPS_ENOMEM : FPS_ECUDA,
                  "cache: cudaMalloc(%zu bytes): %s", bytes, cudaGetErrorString(e));
    }
    c->dev_alias = c->host;
    *out = c;
    return FPS_OK;
  }
  if (d.location == 4) {
    // NEXT-1, the peer tier: the template arena of another GPU (its HBM tier, exported with
    // fps_cache_export_ipc), mapped into this process; loads read it over NVLink / NVSwitch.
    // Same layout and size rules as the exporter's cache (the caller passes the same desc).
    cudaIpcMemHandle_t h;
    memcpy(&h, d.peer_ipc_handle, sizeof(h));
    cudaError_t e = cudaIpcOpenMemHandle((void**)&c->host, h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      cudaGetLastError();
      delete c;
      return fail(FPS_ECUDA, "cache: cudaIpcOpenMemHandle: %s", cudaGetErrorString(e));
    }
    c->dev_alias = c->host;
    *out = c;
    return FPS_OK;
  }
  cudaError_t e;
  if (d.location == 3) {
    // one pinned arena shared by the worker processes of a box (SURVEY §8(e) "shared
    // resource"): every process maps the same file (e.g. a memfd as /proc/<pid>/fd/<n>, or a
    // /dev/shm file) MAP_SHARED and page-locks its own mapping for its device
    const int fd = open(d.shm_path, O_RDWR | O_CREAT, 0600);
    if (fd < 0) {
      delete c;
      return fail(FPS_EINVAL, "cache: open(%s) failed", d.shm_path);
    }
    struct stat st {};
    if (fstat(fd, &st) != 0 || ((size_t)st.st_size < bytes && ftruncate(fd, (off_t)bytes) != 0)) {
      close(fd);
      delete c;
      return fail(FPS_ENOMEM, "cache: sizing %s to %zu bytes failed", d.shm_path, bytes);
    }
    void* p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (p == MAP_FAILED) {
      delete c;
      return fail(FPS_ENOMEM, "cache: mmap(%s, %zu) failed", d.shm_path, bytes);
    }
    e = cudaHostRegister(p, bytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
    if (e != cudaSuccess) {
      cudaGetLastError();
      munmap(p, bytes);
      delete c;
      return fail(FPS_ECUDA, "cache: cudaHostRegister(shared arena): %s", cudaGetErrorString(e));
    }
    c->host = static_cast<char*>(p);
    c->mmap_base = p;
    c->mmap_bytes = bytes;
  } else if (d.location == 2) {
    // pinned host DRAM backed by transparent huge pages (fewer IOMMU translations per byte on
    // the PCIe path): 2 MiB-aligned anonymous mapping, MADV_HUGEPAGE, then page-locked+mapped
    const size_t align = size_t(2) << 20;
    const size_t mbytes = (bytes + align - 1) / align * align;
    void* p = mmap(nullptr, mbytes + align, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
    if (p == MAP_FAILED) {
      delete c;
      return fail(FPS_ENOMEM, "cache: mmap(%zu) failed", mbytes);
    }
    char* a = reinterpret_cast<char*>((reinterpret_cast<uintptr_t>(p) + align - 1) & ~(align - 1));
    madvise(a, mbytes, MADV_HUGEPAGE);
    memset(a, 0, mbytes);                                   // fault the pages in (as huge pages)
    e = cudaHostRegister(a, mbytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
    if (e != cudaSuccess) {
      cudaGetLastError();
      munmap(p, mbytes + align);
      delete c;
      return fail(FPS_ECUDA, "cache: cudaHostRegister: %s", cudaGetErrorString(e));
    }
    c->host = a;
    c->mmap_base = p;
    c->mmap_bytes = mbytes + align;
  } else {
    e = cudaHostAlloc((void**)&c->host, bytes, cudaHostAllocMapped | cudaHostAllocPortable);
    if (e != cudaSuccess) {
      cudaGetLastError();
      delete c;
      return fail(e == cudaErrorMemoryAllocation ? FPS_ENOMEM : FPS_ECUDA,
                  "cache: cudaHostAlloc(%zu bytes): %s", bytes, cudaGetErrorString(e));
    }
  }
  e = cudaHostGetDevicePointer((void**)&c->dev_alias, c->host, 0);
  if (e != cudaSuccess) {
    cudaGetLastError();
    cudaFreeHost(c->host);
    delete c;
    return fail(FPS_ECUDA, "cache: cudaHostGetDevicePointer: %s", cudaGetErrorString(e));
  }
  *out = c;
  return FPS_OK;
}

fps_status fps_cache_destroy(fps_cache_t c) {
  if (!c) return FPS_OK;
  if (c->host) {
    if (c->d.location == 1) {
      cudaFree(c->host);
    } else if (c->d.location == 4) {
      cudaIpcCloseMemHandle(c->host);
    } else if (c->d.location == 2 || c->d.location == 3) {
      cudaHostUnregister(c->host);
      munmap(c->mmap_base, c->mmap_bytes);
    } else {
      cudaFreeHost(c->host);
    }
  }
  delete c;
  return FPS_OK;
}

void* fps_cache_entry_ptr(fps_cache_t c, uint32_t template_id, int32_t step, int32_t layer) {
  if (!c || !key_ok(c, template_id, step, layer)) return nullptr;
  return c->host + offset_of(c, template_id, step, layer);
}

void* fps_cache_entry_host_ptr(fps_cache_t c, uint32_t template_id, int32_t step, int32_t layer) {
  if (!c || in_device_memory(c)) return nullptr;
  return fps_cache_entry_ptr(c, template_id, step, layer);
}

static_assert(sizeof(cudaIpcMemHandle_t) == 64, "the ABI passes IPC handles as 64 bytes");

fps_status fps_cache_export_ipc(fps_cache_t c, void* handle_out) {
  FPS_CHECK_ARG(c && handle_out, "NULL argument");
  FPS_CHECK_ARG(c->d.location == 1, "only an HBM-tier cache (location 1) can be exported");
  cudaIpcMemHandle_t h;
  FPS_CUDA_TRY(cudaIpcGetMemHandle(&h, c->host));
  memcpy(handle_out, &h, sizeof(h));
  return FPS_OK;
}

size_t fps_cache_entry_bytes(fps_cache_t c, int32_t layer) {
  if (!c) return 0;
  return (size_t)c->d.L_img * row_bytes_of(c, layer);
}

fps_status fps_cache_store(fps_cache_t c, uint32_t template_id, int32_t step, int32_t layer,
                           const void* d_src, int32_t src_row_bytes, void* stream) {
  FPS_CHECK_ARG(c && d_src, "NULL argument");
  FPS_CHECK_ARG(key_ok(c, template_id, step, layer), "key (%u,%d,%d) out of range", template_id,
                step, layer);
  const size_t rb = row_bytes_of(c, layer);
  FPS_CHECK_ARG(src_row_bytes >= (int)rb, "src_row_bytes %d < %zu", src_row_bytes, rb);
  FPS_CUDA_TRY(cudaMemcpy2DAsync(c->host + offset_of(c, template_id, step, layer), rb, d_src,
                                 src_row_bytes, rb, c->d.L_img, cudaMemcpyDefault,
                                 as_stream(stream)));
  return FPS_OK;
}

fps_status fps_cache_prefetch(fps_cache_t c, const fps_prefetch_item* items, int32_t n_items,
                              void* load_stream, void* ready_event) {
  FPS_CHECK_ARG(c, "NULL cache");
  FPS_CHECK_ARG(n_items >= 0 && (n_items == 0 || items), "bad items");
  cudaStream_t s = as_stream(load_stream);
  for (int i = 0; i < n_items; ++i) {
    const fps_prefetch_item& it = items[i];
    FPS_CHECK_ARG(key_ok(c, it.template_id, it.step, it.layer), "item %d: key out of range", i);
    FPS_CHECK_ARG(it.n_rows >= 0 && it.n_rows <= c->d.L_img, "item %d: n_rows %d", i, it.n_rows);
    FPS_CHECK_ARG(it.n_rows == 0 || it.d_dst, "item %d: NULL dst", i);
    FPS_CHECK_ARG(it.dst_row_bytes == (int)row_bytes_of(c, it.layer),
                  "item %d: dst_row_bytes %d != entry row bytes %zu", i, it.dst_row_bytes,
                  row_bytes_of(c, it.layer));
    // the row gather (method 0, and method 1 on the HBM arena) reads d_rows on the device;
    // the per-run DMA reads h_rows on the host
    if (c->d.copy_method == 0 || c->d.copy_method == 3 || (c->d.copy_method == 1 && in_device_memory(c)))
      FPS_CHECK_ARG(it.n_rows == 0 || it.d_rows, "item %d: d_rows needed for the row gather", i);
    if (c->d.copy_method == 1 && !in_device_memory(c))
      FPS_CHECK_ARG(it.n_rows == 0 || it.h_rows, "item %d: h_rows needed for DMA", i);
  }
  if (c->d.copy_method == 2) {
    // whole entries: one contiguous DMA per request (rows [0, L_img) land at their token rows)
    double bytes = 0;
    prof::begin(s);
    for (int i = 0; i < n_items; ++i) {
      const fps_prefetch_item& it = items[i];
      if (it.n_rows == 0) continue;
      const size_t nb = (size_t)c->d.L_img * row_bytes_of(c, it.layer);
      const char* src = c->host + offset_of(c, it.template_id, it.step, it.layer);
      if (in_device_memory(c) && g_d2d_kernel) {
        // HBM arena: device-to-device entry copy by our own kernel (launched without PDL).
        // A driver cudaMemcpyAsync D2D here, with PDL launches on the compute stream, hung
        // the C2B stack deterministically (tools/hang_probe.py: plan 21 dense + 39 cached).
        pdl_fence(s);
        FPS_TRY(launch_copy_rows(src, nullptr, nullptr, c->d.L_img, (int)row_bytes_of(c, it.layer),
                                 it.d_dst, s, 0, false));
      } else {
        FPS_COPY_TRY(s, cudaMemcpyAsync(it.d_dst, src, nb, cudaMemcpyDefault, s));
      }
      bytes += nb;
    }
    prof::end(s, prof::PREFETCH, 0, bytes);
  } else if (c->d.copy_method == 3) {
    // TMA bulk row gather: exactly the rows U, a few CTA pairs on reserved SMs
    int max_rb = 0;
    for (int i = 0; i < n_items; ++i) max_rb = std::max(max_rb, (int)row_bytes_of(c, items[i].layer));
    const int slot_bytes = std::max(kBulkMinChunk, max_rb);
    const int ctas = bulk_ctas(c);
    static int inflight_env = -1;     // FPS_BULK_INFLIGHT: bytes over all CTAs (experiments)
    if (inflight_env < 0) {
      const char* v = getenv("FPS_BULK_INFLIGHT");
      inflight_env = v ? std::max(1, atoi(v)) : 0;
    }
    const int inflight = inflight_env > 0 ? inflight_env : kBulkInFlightPerCta * ctas;
    const int slots = std::max(2, std::min({kBulkMaxSlots, (kBulkMaxSmem - kBulkHeader) / slot_bytes,
                                             (inflight + ctas * slot_bytes - 1) / (ctas * slot_bytes)}));
    const int smem = kBulkHeader + slots * slot_bytes;
    FPS_SMEM_ATTR(bulk_gather_kernel, kBulkMaxSmem);
    for (int base = 0; base < n_items; base += kMaxPrefetchItems) {
      BulkBatch b{};
      b.slot_bytes = slot_bytes;
      b.slots = slots;
      double bytes = 0;
      int k = 0;
      for (int i = base; i < n_items && i < base + kMaxPrefetchItems; ++i) {
        const fps_prefetch_item& it = items[i];
        if (it.n_rows == 0) continue;
        b.src[k] = c->dev_alias + offset_of(c, it.template_id, it.step, it.layer);
        b.dst[k] = reinterpret_cast<char*>(it.d_dst);
        b.rows[k] = it.d_rows;
        b.n_rows[k] = it.n_rows;
        b.row_bytes[k] = (int)row_bytes_of(c, it.layer);
        bytes += (double)it.n_rows * b.row_bytes[k];
        ++k;
      }
      b.n_items = k;
      if (k == 0) continue;
      prof::begin(s);
      pdl_fence(s);    // plain launch: the load stream's kernels never overlap via PDL
      FPS_CUDA_TRY(launch_k(bulk_gather_kernel, dim3(ctas), dim3(32), smem, s, b));
      prof::end(s, prof::PREFETCH, 0, bytes);
      count_launch();
      FPS_LAUNCH_CHECK();
    }
  } else if (c->d.copy_method == 0 || in_device_memory(c)) {
    // (method 1 on the HBM arena takes the row gather too: a driver D2D copy per run would
    //  interleave with PDL launches, the pattern that hung in tools/hang_probe.py)
    for (int base = 0; base < n_items; base += kMaxPrefetchItems) {
      PrefetchBatch b{};
      long long acc = 0;
      int k = 0;
      for (int i = base; i < n_items && k < kMaxPrefetchItems; ++i) {
        const fps_prefetch_item& it = items[i];
        if (it.n_rows == 0) continue;
        const int vpr = (int)(row_bytes_of(c, it.layer) / 16);
        b.src[k] = reinterpret_cast<const uint4*>(c->dev_alias +
                                                  offset_of(c, it.template_id, it.step, it.layer));
        b.rows[k] = it.d_rows;
        b.dst[k] = reinterpret_cast<uint4*>(it.d_dst);
        b.vpr[k] = vpr;
        b.start[k] = acc;
        acc += (long long)it.n_rows * vpr;
        ++k;
      }
      b.start[k] = acc;
      b.n_items = k;
      if (acc == 0) continue;
      // few CTAs: the copy overlaps the compute stream and should not crowd it out.
      // Measured on B200 (bench --copy-ctas sweep, 256 threads x 8 loads): 16 CTAs sustain the
      // PCIe link while stealing the least issue bandwidth from the compute stream; the HBM tier
      // needs 64 to keep its row gather (~0.1 ms per Flux block) off the critical path.
      static bool shape_read = false;
      if (!shape_read) {
        shape_read = true;
        if (const char* e = getenv("FPS_PREFETCH_SHAPE"))
          if (sscanf(e, "%d,%d", &g_pf_threads, &g_pf_unroll) != 2) g_pf_threads = 64, g_pf_unroll = 16;
      }
      const int thr = g_pf_threads, unr = g_pf_unroll;
      int ctas = c->d.copy_ctas > 0 ? c->d.copy_ctas : (in_device_memory(c) ? 64 : 16);
      ctas = (int)((long long)ctas * 2048 / (thr * unr));  // same loads in flight as 256 x 8
      long long want = (acc + (long long)thr * unr - 1) / ((long long)thr * unr);
      if (want < ctas) ctas = (int)want;
      if (ctas < 1) ctas = 1;
      prof::begin(s);
      if (unr >= 16) prefetch_kernel<16><<<ctas, thr, 0, s>>>(b);
      else if (unr >= 8) prefetch_kernel<8><<<ctas, thr, 0, s>>>(b);
      else prefetch_kernel<4><<<ctas, thr, 0, s>>>(b);
      prof::end(s, prof::PREFETCH, 0, 16.0 * acc);
      count_launch();
      FPS_LAUNCH_CHECK();
    }
  } else {
    c->dsts.clear();
    c->srcs.clear();
    c->sizes.clear();
    for (int i = 0; i < n_items; ++i) {
      const fps_prefetch_item& it = items[i];
      const size_t rb = row_bytes_of(c, it.layer);
      char* src = c->host + offset_of(c, it.template_id, it.step, it.layer);
      char* dst = (char*)it.d_dst;
      int j = 0;
      while (j < it.n_rows) {
        int k = j;
        while (k + 1 < it.n_rows && it.h_rows[k + 1] == it.h_rows[k] + 1) ++k;
        const size_t r0 = (size_t)it.h_rows[j];
        c->dsts.push_back(dst + r0 * rb);
        c->srcs.push_back(src + r0 * rb);
        c->sizes.push_back((size_t)(k - j + 1) * rb);
        j = k + 1;
      }
    }
    // one DMA per run of consecutive tokens, in submission order on the load stream
    double bytes = 0;
    for (size_t q = 0; q < c->sizes.size(); ++q) bytes += c->sizes[q];
    prof::begin(s);
    if (!c->sizes.empty()) pdl_fence(s);
    for (size_t q = 0; q < c->sizes.size(); ++q)
      FPS_COPY_TRY(s, cudaMemcpyAsync(c->dsts[q], c->srcs[q], c->sizes[q], cudaMemcpyDefault, s));
    prof::end(s, prof::PREFETCH, 0, bytes);
  }
  if (ready_event) FPS_CUDA_TRY(cudaEventRecord((cudaEvent_t)ready_event, s));
  return FPS_OK;
}

}  // extern "C"
