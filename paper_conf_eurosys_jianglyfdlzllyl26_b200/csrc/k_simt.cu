// SIMT kernels: fp32 path (C1, no TF32 -- reading R17) and the generic fallback for shapes the
// tensor-core kernels do not take.  GEMM C = A[M,K] B[N,K]^T (nn.Linear layout) with the fused
// epilogue; varlen merged-key attention (queries from active rows only).
#include "epilogue.cuh"
#include "kernels.h"

namespace fps {

constexpr int SBM = 64, SBN = 64, SBK = 16;

template <typename T>
__global__ void __launch_bounds__(256) gemm_simt_kernel(const T* __restrict__ A,
                                                        const T* __restrict__ B, int M, int N,
                                                        int K, Epilogue ep) {
  __shared__ float As[SBK][SBM + 4];
  __shared__ float Bs[SBK][SBN + 4];
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int m0 = blockIdx.y * SBM, n0 = blockIdx.x * SBN;
  float acc[4][4] = {};
  const int lr = tid >> 2, lk = (tid & 3) * 4;
  for (int k0 = 0; k0 < K; k0 += SBK) {
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int k = k0 + lk + e;
      const int ra = m0 + lr, rb = n0 + lr;
      As[lk + e][lr] = (ra < M && k < K) ? to_f(A[(size_t)ra * K + k]) : 0.f;
      Bs[lk + e][lr] = (rb < N && k < K) ? to_f(B[(size_t)rb * K + k]) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < SBK; ++k) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[k][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[k][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
  const int c0 = n0 + tx * 4;
  if (c0 >= N) return;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int r = m0 + ty * 4 + i;
    if (r < M) epilogue_store<T, 4>(ep, r, c0, acc[i]);
  }
}

fps_status launch_gemm_simt(int dtype, const void* A, const void* B, int M, int N, int K,
                            const Epilogue& ep, cudaStream_t s) {
  if (M <= 0) return FPS_OK;
  if (ep.act == 2 || ep.out0_f32 || ep.resid_f32)
    return fail(FPS_EUNSUPPORTED, "gemm_simt: GEGLU / fp32-residual epilogues are tcgen05-only");
  if (N % 4 != 0 || ep.split % 4 != 0 || ep.split2 % 4 != 0 || ep.act_from % 4 != 0)
    return fail(FPS_EUNSUPPORTED, "gemm_simt: N=%d and the epilogue splits must be multiples of 4", N);
  dim3 grid(ceil_div(N, SBN), ceil_div(M, SBM));
  if (dtype == FPS_BF16)
    gemm_simt_kernel<__nv_bfloat16><<<grid, 256, 0, s>>>(
        (const __nv_bfloat16*)A, (const __nv_bfloat16*)B, M, N, K, ep);
  else
    gemm_simt_kernel<float><<<grid, 256, 0, s>>>((const float*)A, (const float*)B, M, N, K, ep);
  count_launch();
  FPS_LAUNCH_CHECK();
  return FPS_OK;
}

// One warp per (active row, head); online softmax over the request's merged keys in token
// order; exact expf (fp32 path parity 1e-5).  q: [total_q, H]; kv: [total_k, 2H] rows K|V.
template <typename T, int DPL>
__global__ void __launch_bounds__(128) attn_simt_kernel(const T* __restrict__ q,
                                                        const T* __restrict__ kv,
                                                        T* __restrict__ o, int heads, int total_q,
                                                        const int32_t* __restrict__ cu_q,
                                                        const int32_t* __restrict__ cu_k,
                                                        int n_req, int ldo,
                                                        const int32_t* __restrict__ o_map) {
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  const int i = gw / heads, j = gw - (gw / heads) * heads;
  if (i >= total_q) return;
  const int d = DPL * 32, H = heads * d;
  const int r = find_req(cu_q, n_req, i);
  const int k0 = __ldg(cu_k + r), k1 = __ldg(cu_k + r + 1);
  float qv[DPL], acc[DPL];
  const T* qp = q + (size_t)i * H + j * d + lane * DPL;
#pragma unroll
  for (int e = 0; e < DPL; ++e) {
    qv[e] = to_f(qp[e]);
    acc[e] = 0.f;
  }
  const float scale = 1.0f / sqrtf((float)d);
  float m = -INFINITY, l = 0.f;
  for (int t = k0; t < k1; ++t) {
    const T* kr = kv + (size_t)t * 2 * H + j * d + lane * DPL;
    const T* vr = kr + H;
    float s = 0.f;
#pragma unroll
    for (int e = 0; e < DPL; ++e) s = fmaf(qv[e], to_f(kr[e]), s);
    s = warp_sum(s) * scale;
    const float mn = fmaxf(m, s);
    const float c = expf(m - mn), p = expf(s - mn);
    l = l * c + p;
#pragma unroll
    for (int e = 0; e < DPL; ++e) acc[e] = acc[e] * c + p * to_f(vr[e]);
    m = mn;
  }
  T* op = o + (size_t)(o_map ? __ldg(o_map + i) : i) * ldo + j * d + lane * DPL;
  const float inv = 1.0f / l;
#pragma unroll
  for (int e = 0; e < DPL; ++e) op[e] = from_f<T>(acc[e] * inv);
}

fps_status launch_attention_simt(int dtype, const void* q, const void* kv, void* o, int heads,
                                 int head_dim, const int32_t* cu_q, const int32_t* cu_k,
                                 int n_req, int total_q, cudaStream_t s, int ldo,
                                 const int32_t* o_map) {
  if (total_q <= 0) return FPS_OK;
  if (ldo == 0) ldo = heads * head_dim;
  const long long warps = (long long)total_q * heads;
  const int grid = (int)((warps * 32 + 127) / 128);
#define FPS_ATT_CASE(D)                                                                      \
  if (head_dim == D) {                                                                       \
    if (dtype == FPS_BF16)                                                                   \
      attn_simt_kernel<__nv_bfloat16, D / 32><<<grid, 128, 0, s>>>(                          \
          (const __nv_bfloat16*)q, (const __nv_bfloat16*)kv, (__nv_bfloat16*)o, heads,       \
          total_q, cu_q, cu_k, n_req, ldo, o_map);                                                \
    else                                                                                     \
      attn_simt_kernel<float, D / 32><<<grid, 128, 0, s>>>(                                  \
          (const float*)q, (const float*)kv, (float*)o, heads, total_q, cu_q, cu_k, n_req, ldo, \
          o_map);                                                                            \
    count_launch();                                                                          \
    FPS_LAUNCH_CHECK();                                                                      \
    return FPS_OK;                                                                           \
  }
  FPS_ATT_CASE(32)
  FPS_ATT_CASE(64)
  FPS_ATT_CASE(128)
#undef FPS_ATT_CASE
  return fail(FPS_EUNSUPPORTED, "attention_simt: head_dim %d not in {32,64,128}", head_dim);
}

}  // namespace fps
