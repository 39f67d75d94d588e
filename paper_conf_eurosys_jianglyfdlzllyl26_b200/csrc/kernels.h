// Internal launcher declarations (libflashps). Each returns fps_status and never syncs.
#pragma once
#include "common.cuh"

namespace fps {

// a1
fps_status launch_mask_index(const uint8_t* masks, const int32_t* off, int n_req, int max_len,
                             int32_t* mids, int32_t* uids, int32_t* nm, cudaStream_t s);
// NEXT-4: pixel mask -> token mask (max-pool over f x f blocks, text tokens appended active)
fps_status launch_mask_pool(const uint8_t* pix, int n_req, int Hp, int Wp, int f, int L_txt,
                            uint8_t* tok, cudaStream_t s);
// a2/a9/a3 row movement: dst[dst_ids? dst_ids[i] : i] = src[src_ids ? src_ids[i] : i]
fps_status launch_copy_rows(const void* src, const int32_t* src_ids, const int32_t* dst_ids,
                            int n, int row_bytes, void* dst, cudaStream_t s, int max_ctas = 0,
                            bool profile = true);
// a4: out[out_rows ? out_rows[i] : i] = LN(x[rows ? rows[i] : i]) * (1 + scale[req(i)])
//                                        + shift[req(i)]
fps_status launch_ln_mod(int dtype, const void* x, const int32_t* rows, int n, int H, void* out,
                         const int32_t* cu, int n_req, const void* mod, int shift_off,
                         cudaStream_t s, const int32_t* out_rows = nullptr, int mod_stride = 0);
fps_status launch_ln_ysplit(int dtype, const void* x0, const int32_t* rows0, int n0,
                            const void* x1, const int32_t* rows1, int n1, int H, void* out,
                            void* outb, const int32_t* outb_rows0, const int32_t* outb_rows1,
                            const int32_t* cu0, const int32_t* cu1, int n_req, const void* mod,
                            int shift_off, int mod_stride, const void* gamma, const void* beta,
                            cudaStream_t s);
fps_status launch_ln_mod_2src(int dtype, const void* x0, const int32_t* rows0, int n0,
                              const void* x1, const int32_t* rows1, int n1, int H, void* out,
                              const int32_t* cu0, const int32_t* cu1, int n_req, const void* mod,
                              int shift_off, cudaStream_t s, int mod_stride);
// a4 over two row groups in one launch (double-stream block): rows >= split use cu2 (rows
// counted from split) and vectors soff elements after the first group's
fps_status launch_ln_mod2(int dtype, const void* x, const int32_t* rows, int n, int H, void* out,
                          const int32_t* cu, const int32_t* cu2, int split, int n_req,
                          const void* mod, int shift_off, int soff, cudaStream_t s,
                          int mod_stride);
// a4 (SDXL block, R24): out[out_rows ? out_rows[i] : i] = LN(x[rows ? rows[i] : i]) * gamma + beta
fps_status launch_ln_affine(int dtype, const void* x, const int32_t* rows, int n, int H, void* out,
                            const void* gamma, const void* beta, cudaStream_t s,
                            const int32_t* out_rows = nullptr);
// same over an fp32 residual stream: x [n, H] fp32 -> out [n, H] bf16
fps_status launch_ln_affine_f32in(const float* x, int n, int H, void* out, const void* gamma,
                                  const void* beta, cudaStream_t s);
// GEGLU weight packing: rows of w [2F, K] (value half, then gate half) -> 32-row interleave
// (value rows 32j.., gate rows 32j..) so one 64-column GEMM chunk holds a (value, gate) pair
fps_status launch_geglu_pack(int dtype, const void* w, const void* b, int F, int K, void* w_out,
                             void* b_out, cudaStream_t s);
// x[i] += delta[req(i)] * y[i] over rows of width H (req via cu over rows)
fps_status launch_euler(int dtype, void* x, const void* y, int n, int H, const int32_t* cu,
                        int n_req, const float* delta, cudaStream_t s);
// flow-matching Euler + inpainting blend (R29) over n_req request latents of L rows each:
// masked image rows x += coef[r].x * y; unmasked image rows x = (1 - coef[r].y) z + coef[r].y eps
// (zeps[2r], zeps[2r+1]: the request's [L_img, H] template latent and noise); text rows kept
fps_status launch_flow_blend(int dtype, void* x, const void* y, int n_req, int L, int L_img, int H,
                             const uint8_t* mask, const float2* coef, const void* const* zeps,
                             cudaStream_t s);
// GEMM C = A[M,K] B[N,K]^T with the fused epilogue
fps_status launch_gemm(int dtype, const void* A, const void* B, int M, int N, int K,
                       const Epilogue& ep, cudaStream_t s);
fps_status launch_gemm_simt(int dtype, const void* A, const void* B, int M, int N, int K,
                            const Epilogue& ep, cudaStream_t s);
fps_status launch_gemm_tc(const void* A, const void* B, int M, int N, int K, const Epilogue& ep,
                          cudaStream_t s);
bool gemm_tc_supported(int dtype, int M, int N, int K);
// two GEMMs sharing N and K in one launch: rows [0, M0) of A with B0 / ep0, rows [M0, M0 + M1)
// with B1 / ep1 (ep1 indexes its rows from 0)
// Two GEMMs in one launch: rows [0, M0) of A times B0 [N, K] (ep0), rows [M0, M0 + M1) times
// B1 [N1, K] (ep1); N1 = 0 means N1 = N
fps_status launch_gemm_grouped(int dtype, const void* A, const void* B0, const void* B1, int M0,
                               int M1, int N, int K, const Epilogue& ep0, const Epilogue& ep1,
                               cudaStream_t s, int N1 = 0);
fps_status launch_gemm_tc_grouped(const void* A, const void* B0, const void* B1, int M0, int M1,
                                  int N, int K, const Epilogue& ep0, const Epilogue& ep1,
                                  cudaStream_t s, int N1 = 0);
// Scratch for split-KV attention: partial outputs (S x total_q x H bf16) and per-row
// statistics (S x total_q x heads float2); null = no split
struct AttnScratch {
  void* part;
  size_t part_bytes;
  void* ml;
  size_t ml_bytes;
};
// a6: o[i, head] = softmax(q_i k^T / sqrt(d)) v over the request's merged keys; o rows are
// ldo elements apart (0 = heads * head_dim); o_map: query row i is written to output row
// o_map[i] (null -> i; default tensor-core and SIMT kernels only)
fps_status launch_attention(int dtype, const void* q, const void* kv, void* o, int heads,
                            int head_dim, const int32_t* d_cu_q, const int32_t* d_cu_k,
                            const int32_t* h_cu_q, const int32_t* h_cu_k, int n_req, int total_q,
                            int max_q, int max_k, cudaStream_t s, int ldo = 0,
                            const AttnScratch* sc = nullptr, const int32_t* o_map = nullptr);
fps_status launch_attention_simt(int dtype, const void* q, const void* kv, void* o, int heads,
                                 int head_dim, const int32_t* cu_q, const int32_t* cu_k,
                                 int n_req, int total_q, cudaStream_t s, int ldo = 0,
                                 const int32_t* o_map = nullptr);
fps_status launch_attention_tc(const void* q, const void* kv, void* o, int heads, int head_dim,
                               const int32_t* d_cu_q, const int32_t* d_cu_k, const int32_t* h_cu_q,
                               const int32_t* h_cu_k, int n_req, cudaStream_t s, int ldo = 0,
                               const AttnScratch* sc = nullptr, const int32_t* o_map = nullptr);
bool attention_tc_supported(int dtype, int head_dim);

// true if fps_cache_prefetch also overwrites rows outside U (copy_method 2): fresh rows written
// into the same buffer must then be ordered after the load's ready event
bool cache_writes_all_rows(const fps_cache* c);
// CTAs the cache's TMA row gather (copy_method 3) runs on; 0 for the other methods
int bulk_ctas(const fps_cache* c);

// global switches (tests can force the SIMT kernels): bit0 = no tcgen05 GEMM,
// bit1 = no tensor-core attention
extern int g_disable_tc;
// tests: 0 = choose, 1 = force the 1-SM tcgen05 GEMM, 2 = force the CTA-pair GEMM
extern int g_gemm_force;
extern int g_gemm_epi4;
extern int g_gemm_bn;
// tests: 0 = two query tiles per CTA (default), 1 = force the one-tile attention kernel
extern int g_attn_force;
extern int g_attn_pair;
extern int g_attn_rot;
// tests: force the split-KV factor S (0 = choose)
extern int g_attn_split;
// 1 (default): HBM-arena whole-entry loads copied by a library kernel, 0: driver D2D memcpy
extern int g_d2d_kernel;

}  // namespace fps
