/* flashps.h -- C ABI of the B200-native FlashPS hot path (libflashps.so).
 *
 * FlashPS (EuroSys '26), /root/reference/PAPER.md: the mask-aware transformer-block forward
 * (§3.1, Fig. 5/7), its block-granular cache-load pipeline (§4.2,
 * Alg. 1) and step-level continuous batching (§4.3).  `Lnnn` = PAPER.md line nnn.
 *
 * Conventions for every call
 *  - Pointers prefixed d_ are DEVICE pointers, h_ are HOST pointers. Device buffers are
 *    caller-owned (allocated with any CUDA allocator, e.g. torch); the library never frees them.
 *    Library-owned state lives only inside fps_cache_t / fps_engine_t handles.
 *  - `stream` arguments are cudaStream_t passed as void* (NULL = legacy default stream).
 *    Every device call is asynchronous on its stream: no allocation and no host
 *    synchronisation inside hot calls (fps_run_batch documents its one admission sync).
 *  - Errors: arguments are validated before anything is enqueued, so a failing call has no
 *    side effect and returns FPS_EINVAL / FPS_EUNSUPPORTED; a failed launch returns FPS_ECUDA.
 *    Asynchronous device faults surface at the caller's next synchronisation.
 *    fps_last_error() returns a thread-local message describing the last failure.
 *  - Rows are contiguous and 16-byte aligned (row_bytes % 16 == 0, pointers 16-B aligned).
 *  - Determinism: outputs are bit-reproducible run to run (no split-K atomics).
 *  - There is no CPU fallback: on a machine without a usable sm_100 GPU every device call
 *    returns FPS_ECUDA.
 */
#ifndef FLASHPS_H
#define FLASHPS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define FPS_ABI_VERSION 3

typedef enum {
  FPS_OK = 0,
  FPS_EINVAL = -1,        /* bad argument (null pointer, size, alignment, layout)        */
  FPS_ECUDA = -2,         /* CUDA runtime / launch failure, or no usable sm_100 device     */
  FPS_ENOMEM = -3,        /* host or device allocation failed (handle creation only)       */
  FPS_EUNSUPPORTED = -4,  /* valid request outside what the kernels implement              */
  FPS_ESTATE = -5         /* handle in the wrong state (e.g. prefetch of a never-stored entry) */
} fps_status;

enum { FPS_F32 = 0, FPS_BF16 = 1 };            /* element type of activations and weights */
enum { FPS_MODE_KV = 0, FPS_MODE_Y = 1 };      /* caching variant: Fig. 7 (K/V) or Fig. 5 (Y) */

const char* fps_last_error(void);
int32_t fps_abi_version(void);
/* 1 if a device usable by the kernels (compute capability 10.0) is present, else 0. */
int32_t fps_device_ok(void);
/* Test / bench hooks: number of kernels this thread has launched through the library so far;
 * force the SIMT kernels (bit0: GEMMs, bit1: attention) instead of the tensor-core ones;
 * bits 2-3 = 1 force the 1-SM tcgen05 GEMM, = 2 force the CTA-pair (cta_group::2) GEMM;
 * bits 4-5 = 1 force the one-query-tile attention kernel, = 2 the two-tile kernel with P in
 * shared memory, = 3 the two-tile kernel with P in TMEM and a correction warpgroup (the default);
 * bit 6 = launch without programmatic dependent launch (PDL is on by default);
 * bit 7 = HBM-arena whole-entry prefetch by driver device-to-device memcpy instead of the
 * library copy kernel (experiments only: see cache.cu);
 * bits 8-10 = S > 0 forces the split-KV factor of the tensor-core attention inside block calls
 * (0 = chosen by wave efficiency; S is applied only when the block workspace holds the S
 * partial outputs);
 * bit 11 = the tcgen05 GEMMs (1-SM and CTA-pair) with 4 epilogue warps instead of 8 (A/B);
 * bit 12 = the CTA-pair attention kernel (attn_tc4, head_dim 128);
 * bits 13-14 = 1 / 2 force the 1-SM GEMM's 128- / 256-column tile (A/B experiments);
 * bit 15 = the Y-mode parallel block's two projections (rows M on W1, cached rows U on K|V) as two
 *          launches instead of one grouped launch (A/B; outputs are bit-identical);
 * bit 16 = head_dim 64 attention on attn_tc3 instead of attn_tc5 (three rotating S buffers). */
int64_t fps_launch_count(void);
void fps_set_disable_tc(int32_t flags);
/* Per-kernel-class timing for the bench: when enabled (this also clears old records) every
 * library launch is bracketed by CUDA events on its own stream.  fps_profile_read synchronises
 * on them and fills, per class k in {0 GEMM, 1 attention, 2 row-norm, 3 row copy, 4 cache
 * prefetch, 5 sampler update, 6 mask index}, the summed device ms, algorithmic FLOPs and bytes
 * and the launch count (arrays of 7, each may be NULL).  Returns the number of classes (7) or
 * FPS_ECUDA. */
void fps_profile_enable(int32_t on);
int32_t fps_profile_read(double* ms, double* flops, double* bytes, int64_t* count);
/* The recorded launches in launch order (up to max_n): start / end in ms relative to the first
 * launch's start event, the kernel class, and the stream (as an integer id).  Returns the
 * number written, or FPS_ECUDA. */
int64_t fps_profile_trace(double* start_ms, double* end_ms, int32_t* kind, int64_t* stream,
                          int64_t max_n);

/* ---------------------------------------------------------------------------------------
 * a1 input (NEXT-4)  Pixel mask -> token mask.  L79 (§2.1): the latent (B, C, H, W) is reshaped
 * to (B, H x W, C), one token per latent position; a token covers an f x f block of editing-mask
 * pixels (VAE down-sampling x patchify).  Reading R8: a token is active iff ANY of
 * its pixels is nonzero; reading R9: L_txt text tokens are appended, always active.
 *   d_pix   uint8 [n_req][Hp * Wp] row-major pixel masks (nonzero = edit this pixel).
 *   f       block edge; must divide Hp and Wp (else FPS_EINVAL).
 *   d_tok   uint8 [n_req][(Hp/f) * (Wp/f) + L_txt] written with 0/1 (caller-owned).
 * Bit-exact with oracle/index.py pixel_to_token_mask.  Output feeds fps_build_mask_index. */
fps_status fps_mask_to_tokens(const uint8_t* d_pix, int32_t n_req, int32_t Hp, int32_t Wp,
                              int32_t f, int32_t L_txt, uint8_t* d_tok, void* stream);

/* ---------------------------------------------------------------------------------------
 * a1  Mask -> token index (L130 "categorize the tokens as masked tokens and unmasked tokens").
 *   d_masks       uint8 [total]: request r's token mask occupies [off[r], off[r+1]);
 *                 nonzero = active (masked image token, or text token -- set by the caller).
 *   d_offsets     int32 [n_req+1] on DEVICE, off[0] = 0, non-decreasing.
 *   d_masked_ids  int32 [total]: request r's ascending LOCAL active ids are written to
 *                 d_masked_ids[off[r] .. off[r]+n_r).
 *   d_unmasked_ids int32 [total]: ascending local inactive ids at [off[r] .. off[r]+L_r-n_r).
 *   d_n_masked    int32 [n_req]: n_r.
 *   max_len       upper bound on any L_r (launch sizing only).
 * Bit-exact with the oracle (oracle/index.py). One CTA per request, warp-ballot compaction. */
fps_status fps_build_mask_index(const uint8_t* d_masks, const int32_t* d_offsets, int32_t n_req,
                                int32_t max_len, int32_t* d_masked_ids, int32_t* d_unmasked_ids,
                                int32_t* d_n_masked, void* stream);

/* ---------------------------------------------------------------------------------------
 * a2 / a9  Row movement (L157 "extract the matrix of masked tokens ... replenishing cached
 * activations for the unmasked tokens"). 16-B vectorised, bit-exact.
 *   gather : d_dst[i]          = d_src[d_ids[i]]      i in [0, n)
 *   scatter: d_dst[d_ids[i]]   = d_src[i]
 *   copy   : d_dst[d_dst_ids[i]] = d_src[d_src_ids[i]]   (either id array may be NULL = i)
 * row_bytes % 16 == 0. d_src may be a mapped pinned-host pointer (zero-copy read).          */
fps_status fps_gather_rows(const void* d_src, const int32_t* d_ids, int32_t n, int32_t row_bytes,
                           void* d_dst, void* stream);
fps_status fps_scatter_rows(const void* d_src, const int32_t* d_ids, int32_t n, int32_t row_bytes,
                            void* d_dst, void* stream);
fps_status fps_copy_rows(const void* d_src, const int32_t* d_src_ids, const int32_t* d_dst_ids,
                         int32_t n, int32_t row_bytes, void* d_dst, void* stream);

/* ---------------------------------------------------------------------------------------
 * a3  Activation cache (L203 host-DRAM store; L207 block granularity; reading R7: key =
 * (template, step, layer)).  An entry holds L_img rows of width W elements of the template's
 * full run: KV-mode W = 2H (row = K|V of that token, Fig. 7), Y-mode W = H (block output Y,
 * Fig. 5).  KV-mode also keeps, per step, the final block's Y rows under layer = n_layers
 * (width H) for the last replenish (reading R22).                                           */
typedef struct {
  int32_t mode;          /* FPS_MODE_KV | FPS_MODE_Y                                        */
  int32_t dtype;         /* FPS_BF16 | FPS_F32                                              */
  int32_t H;             /* hidden size                                                     */
  int32_t L_img;         /* rows per entry (image tokens; text rows are never cached, R9)   */
  int32_t n_layers;
  int32_t n_steps;
  int32_t n_templates;   /* templates addressable: template_id in [0, n_templates)          */
  int32_t n_entries;     /* physical entries in the pinned arena; 0 = one per key.  When
                            smaller, key k maps to entry k % n_entries (perf runs only: bytes
                            moved are identical, contents alias)                            */
  int32_t copy_method;   /* how fps_cache_prefetch moves an entry's rows U (all four give the
                            same bytes at rows U; DESIGN.md §6 has the measurements):
                            0 = SM row gather (zero-copy over mapped pinned memory, or from
                                the HBM arena) -- exactly the rows U, but its warps share the
                                SMs with the compute stream;
                            1 = copy-engine DMA of exactly the rows U: one cudaMemcpyAsync
                                per run of consecutive tokens on the load stream (on the HBM
                                arena, location 1, the rows go through the method-0 gather);
                                per-copy overhead: ~47 GB/s on blob masks, ~12 GB/s on
                                random masks (hundreds of runs);
                            2 = copy-engine DMA of the WHOLE entry (all L_img rows, one copy
                                per request): no SM time, full link rate on 1/(1-m) more
                                bytes; rows outside U are overwritten too, so fresh K/V must
                                be written only after `ready_event` (fps_run_batch orders
                                this itself).  The bench default on both tiers;
                            3 = TMA bulk row gather: exactly the rows U, moved host -> smem
                                -> HBM by cp.async.bulk from copy_ctas CTAs (default 4, in
                                TPC pairs) at ~51 GB/s of useful bytes; fps_run_batch with a
                                load stream sizes its compute grids to the other SMs.  Pinned
                                host tiers only need it; rows <= 32 KB.  Give the load stream
                                a high CUDA priority: its gather CTAs then take the reserved
                                SMs ahead of queued compute CTAs (non-persistent grids, PDL
                                early launches).  Inside a step 6-8 CTAs keep the link busy
                                (bench default at configs[3], where whole entries would move
                                1.48x the unmasked bytes)                                    */
  int32_t copy_ctas;     /* CTAs used by method 0 (0 = default: 16 for the host link -- enough
                            for PCIe, few enough not to crowd out the compute stream -- and 64
                            for the HBM tier) and by method 3 (0 = 4; even)                        */
  int32_t location;      /* 0 = pinned host DRAM (L203, streamed over PCIe);
                            1 = device HBM: the template tier one level above host DRAM
                            (the paper's "ideal" no-load case of Fig. 4-Left,
                            L108), prefetch becomes an HBM row gather;
                            2 = pinned host DRAM on 2 MiB pages (THP);
                            3 = pinned host DRAM SHARED by the worker processes of a box
                                (SURVEY §8(e)): the file at shm_path (created / grown to the
                                arena size if needed) is mapped MAP_SHARED and page-locked by
                                each process -- one copy of the templates for all GPUs;
                            4 = a PEER GPU's HBM tier (NEXT-1, the NVLink / NVSwitch level
                                of the hierarchical store, L222-L224): the arena another
                                process exported with fps_cache_export_ipc, opened with CUDA
                                IPC (peer access enabled lazily); loads read it over NVLink
                                exactly like the local HBM tier (methods 0 / 2 / 3 on the
                                device, method 1 takes the gather).  The desc must match the
                                exporter's (same sizes and n_entries); stores write through to
                                the peer                                                     */
  const char* shm_path;  /* location 3: path of the shared arena file (e.g. a memfd opened
                            as /proc/<pid>/fd/<n>, or /dev/shm/<name>); the caller removes
                            it; NULL otherwise                                               */
  const void* peer_ipc_handle;   /* location 4: the 64-byte cudaIpcMemHandle_t written by the
                            owner's fps_cache_export_ipc; NULL otherwise                     */
} fps_cache_desc;

typedef struct fps_cache* fps_cache_t;

fps_status fps_cache_create(const fps_cache_desc* desc, fps_cache_t* out);
fps_status fps_cache_destroy(fps_cache_t c);
/* Host pointer of an entry (tests / tooling); NULL if out of range or the arena is in HBM. */
void* fps_cache_entry_host_ptr(fps_cache_t c, uint32_t template_id, int32_t step, int32_t layer);
/* Address of an entry in whichever memory holds the arena (host or device); NULL if out of range. */
void* fps_cache_entry_ptr(fps_cache_t c, uint32_t template_id, int32_t step, int32_t layer);
size_t fps_cache_entry_bytes(fps_cache_t c, int32_t layer);
/* NEXT-1 peer tier: export an HBM-tier cache's arena (location 1) as a 64-byte CUDA IPC
 * handle for other processes (another GPU's worker opens it as location 4).  The exporting
 * cache must outlive every importer. */
fps_status fps_cache_export_ipc(fps_cache_t c, void* handle_out);
/* D2H: store rows [0, L_img) of d_src (row pitch src_row_bytes >= W*elt) as entry
 * (template_id, step, layer).  Asynchronous on `stream`. */
fps_status fps_cache_store(fps_cache_t c, uint32_t template_id, int32_t step, int32_t layer,
                           const void* d_src, int32_t src_row_bytes, void* stream);

/* H2D layer-ahead prefetch (L207-L209): for each item, rows d_rows[0..n_rows) (LOCAL token
 * ids < L_img, ascending) of entry (template_id, step, layer) are copied to the SAME row
 * positions of d_dst (row pitch dst_row_bytes).  All items are issued on `load_stream`; if
 * `ready_event` (cudaEvent_t) is non-NULL it is recorded after the last copy. */
typedef struct {
  uint32_t template_id;
  int32_t step;
  int32_t layer;
  int32_t n_rows;
  const int32_t* d_rows;   /* device, [n_rows] local row ids (unmasked tokens U); read by
                              the row gathers: methods 0 and 3, and method 1 on the HBM
                              arena (FPS_EINVAL if NULL there)                             */
  const int32_t* h_rows;   /* host mirror of d_rows: read by method 1 on a host arena (one
                              DMA per run); may be NULL otherwise                          */
  void* d_dst;             /* device row 0 of this request's [L, W] region                */
  int32_t dst_row_bytes;
} fps_prefetch_item;

fps_status fps_cache_prefetch(fps_cache_t c, const fps_prefetch_item* items, int32_t n_items,
                              void* load_stream, void* ready_event);

/* ---------------------------------------------------------------------------------------
 * a4-a8  Block forward (L146 block definition; L157 mask-aware; L161 KV variant).
 * Block (oracle/block.py):  h1 = LN(x)(1+sc1)+sh1; Q,K,V = h1 W^T + b; A = softmax(QK^T/sqrt(d))V
 * per head; x1 = x + g1 (A Wo^T + bo); y = x1 + g2 (GELU_tanh(LN(x1)(1+sc2)+sh2 W1^T + b1) W2^T + b2).
 * Weights use the nn.Linear layout W[out, in], row-major, dtype = `dtype`; biases may be NULL.
 *
 * kind = FPS_BLOCK_PAR (NEXT-2, reading R23): the parallel (Flux single-stream) block
 *   h = LN(x)(1+sc1)+sh1; [Q|K|V|Z] = h W1^T + b1; y = x + g1 ([A | GELU_tanh(Z)] W2^T + b2)
 * with W1 = w_qkv [3H+F, H] (rows Wq, Wk, Wv, then the F MLP-input rows), b1 = b_qkv [3H+F],
 * W2 = w_down [H, H+F], b2 = b_down [H]; w_o, b_o, w_up, b_up must be NULL; only
 * (shift1, scale1, gate1) of the modulation vector are read.  Same masked modes and cache.
 *
 * kind = FPS_BLOCK_SDXL (NEXT-2, reading R24): the SDXL UNet transformer block (the paper
 *   evaluates SDXL, L65 / L305) -- self-attention, cross-attention to the request's prompt
 *   encoding, GEGLU feed-forward, each behind an affine LayerNorm, ungated residuals:
 *   h1 = LN(x) g1 + b1;  x1 = x + (A(h1 Wq^T, h1 Wk^T, h1 Wv^T) Wo^T + bo)
 *   h2 = LN(x1) g2 + b2; x2 = x1 + (A(h2 Wq2^T, Kc, Vc) Wo2^T + bo2),  [Kc | Vc] = ctx Wkv2^T
 *   h3 = LN(x2) g3 + b3; [P | G] = h3 Wup^T + bup;  y = x2 + ((P * GELU_tanh(G)) Wdown^T + bdown)
 *   w_up / b_up must be in the PACKED layout fps_geglu_pack writes ([2F, H], F % 32 == 0);
 *   the per-request context keys / values Kc | Vc come precomputed in the batch (d_ctx_kv,
 *   written by fps_context_kv); d_mod is ignored.  bf16 only (tcgen05 path; H, F % 64 == 0).
 *
 * kind = FPS_BLOCK_DOUBLE (NEXT-2, reading R25): Flux's double-stream (MM-DiT) block.  Image
 *   rows and text rows keep their own sequential-block weights (image: the fields above; text:
 *   the t_* fields) and adaLN vectors (the request's modulation vector is [12H]: image 6H, then
 *   text 6H) and meet in ONE joint attention over all rows.  The batch must describe the
 *   stream-major order of its active rows (fps_varlen_batch.d_sm_perm etc.); text rows are
 *   always active (R9), so cached rows U are image rows.
 */
enum { FPS_BLOCK_SEQ = 0, FPS_BLOCK_PAR = 1, FPS_BLOCK_SDXL = 2, FPS_BLOCK_DOUBLE = 3 };
typedef struct {
  int32_t H, heads, head_dim, F;   /* H = heads*head_dim; F = MLP width                    */
  int32_t dtype;                   /* FPS_BF16 (tcgen05 path) | FPS_F32 (SIMT fp32 path)   */
  const void *w_qkv, *b_qkv;       /* [3H, H], [3H]  rows: Wq, Wk, Wv  (PAR: W1, b1)        */
  const void *w_o, *b_o;           /* [H, H], [H]                      (PAR: NULL)          */
  const void *w_up, *b_up;         /* [F, H], [F]  (PAR: NULL; SDXL: packed GEGLU [2F, H])  */
  const void *w_down, *b_down;     /* [H, F], [H]                      (PAR: W2 [H, H+F], b2) */
  int32_t kind;                    /* FPS_BLOCK_SEQ | FPS_BLOCK_PAR | FPS_BLOCK_SDXL        */
  /* SDXL block only (NULL / 0 otherwise); biases may be NULL, LN vectors may not.          */
  int32_t D_ctx;                   /* prompt-encoding width (2048 in SDXL)                  */
  const void *ln1_w, *ln1_b, *ln2_w, *ln2_b, *ln3_w, *ln3_b;   /* [H] gamma, beta          */
  const void *w_q2, *b_q2;         /* [H, H], [H]   cross-attention query projection       */
  const void *w_kv2, *b_kv2;       /* [2H, D_ctx], [2H]  rows Wk2 then Wv2 (fps_context_kv) */
  const void *w_o2, *b_o2;         /* [H, H], [H]   cross-attention output projection      */
  /* DOUBLE block only: the text stream's weights, same shapes as w_qkv .. b_down.           */
  const void *t_qkv, *tb_qkv, *t_o, *tb_o, *t_up, *tb_up, *t_down, *tb_down;
} fps_block_weights;

/* One varlen launch over a continuous batch (L237): request r owns active rows
 * [cu_q[r], cu_q[r+1]) of the compact activation arrays and merged key rows
 * [cu_k[r], cu_k[r+1]) of d_kv. */
typedef struct {
  int32_t n_req;
  int32_t total_q, total_k;        /* sum n_r, sum L_r                                      */
  int32_t max_q, max_k;            /* max n_r, max L_r                                      */
  const int32_t* d_cu_q;           /* [n_req+1]                                             */
  const int32_t* d_cu_k;           /* [n_req+1]                                             */
  const int32_t* h_cu_q;           /* host mirrors (launch sizing, no device sync)           */
  const int32_t* h_cu_k;
  const int32_t* d_q_row;          /* [total_q] merged-buffer row of each active row;
                                      NULL = identity (dense block: total_q == total_k)      */
  const void* d_mod;               /* [n_req, 6H] adaLN (shift1,scale1,gate1,shift2,scale2,
                                      gate2) in dtype, or NULL = identity modulation         */
  int32_t mode;                    /* FPS_MODE_KV | FPS_MODE_Y                               */
  /* Y-mode only (Fig. 5-Bottom): cached input rows U feed the K/V projection.             */
  int32_t total_u;                 /* sum u_r                                               */
  const int32_t* d_cu_u;           /* [n_req+1]                                             */
  const int32_t* d_u_src;          /* [total_u] row index into d_xu of each cached row      */
  const int32_t* d_u_row;          /* [total_u] merged-buffer row of each cached row        */
  /* SDXL blocks only: request r's cross-attention keys / values are rows
   * [cu_ctx[r], cu_ctx[r+1]) of d_ctx_kv ([total_ctx, 2H], row = Kc|Vc, fps_context_kv).    */
  const void* d_ctx_kv;
  const int32_t* d_cu_ctx;         /* [n_req+1] device                                      */
  const int32_t* h_cu_ctx;         /* [n_req+1] host mirror                                  */
  /* Elements between consecutive requests' modulation vectors in d_mod (0 = 6H, or 12H for
   * a DOUBLE block).                                                                       */
  int32_t mod_stride;
  /* DOUBLE blocks only: the stream-major order of the active rows -- every request's image
   * rows (request-major, ascending), then every request's text rows.                        */
  int32_t total_q_img;             /* active image rows of the batch                        */
  const int32_t* d_sm_perm;        /* [total_q] compact (request-major) row of stream row i  */
  const int32_t* d_sm_kvrow;       /* [total_q] merged-buffer row of stream row i            */
  const int32_t* d_cu_img;         /* [n_req+1] prefix sums of active image rows            */
  const int32_t* d_cu_txt;         /* [n_req+1] prefix sums of text rows                    */
  const int32_t* d_sm_inv;         /* [total_q] stream row of compact row r (the inverse of
                                      d_sm_perm), or NULL: the block then reorders its rows
                                      with two extra row copies                              */
  /* a2 fused into the block (NEXT-4): 1 = d_x_act is the FULL merged buffer [total_k, H] and
   * active row i is its row d_q_row[i] (d_sm_kvrow for DOUBLE blocks) -- the first norm and
   * the residual read the rows there, so no gathered copy of the active rows is needed;
   * 0 = d_x_act is compact [total_q, H] (request-major).  Requires d_q_row.                */
  int32_t x_full_rows;
} fps_varlen_batch;

/* SDXL block helpers (R24), run once per weight load / per request prompt, not per step.
 * fps_geglu_pack: d_w [2F, K] (rows: GEGLU value half, then gate half -- diffusers' GEGLU
 *   proj layout) and optional d_b [2F] -> d_w_out / d_b_out in the packed layout the block's
 *   fused GEGLU epilogue reads (32-row groups: value rows 32j..32j+31, then gate rows
 *   F+32j..F+32j+31).  F % 32 == 0, K*elt % 16 == 0; outputs must not alias inputs.
 * fps_context_kv: d_ctx_kv[n_rows, 2H] = d_ctx[n_rows, D_ctx] Wkv2^T (+ b_kv2) with the
 *   block's cross-attention weights -- the K|V rows fps_varlen_batch.d_ctx_kv expects. */
fps_status fps_geglu_pack(int32_t dtype, const void* d_w, const void* d_b, int32_t F, int32_t K,
                          void* d_w_out, void* d_b_out, void* stream);
fps_status fps_context_kv(const fps_block_weights* w, const void* d_ctx, int32_t n_rows,
                          void* d_ctx_kv, void* stream);

/* Workspace bytes fps_masked_block_forward needs for up to max_q active / max_u cached rows. */
size_t fps_block_workspace_bytes(int32_t H, int32_t F, int32_t dtype, int32_t max_q, int32_t max_u);

/* Mask-aware block over a varlen batch.
 *   d_x_act [total_q, H]  input rows (active tokens, request-major, ascending ids).
 *   d_y_act [total_q, H]  output rows. May alias nothing else.
 *   d_kv    [total_k, 2H] merged key buffer, row = K|V.  KV-mode: rows NOT named by d_q_row
 *           must already hold (or be in flight to) the cached K|V (fps_cache_prefetch);
 *           this call writes the fresh rows d_q_row.  Y-mode: fully written by this call.
 *   d_xu    Y-mode: base of the cached input rows (indexed by b->d_u_src); NULL in KV-mode.
 *   kv_ready (cudaEvent_t or NULL): waited on `stream` right before the first kernel that
 *           reads cached rows (attention in KV-mode, the K/V projection in Y-mode), so the
 *           fresh Q/K/V projection overlaps the in-flight load.
 *   d_ws / ws_bytes: scratch of at least fps_block_workspace_bytes(...). */
fps_status fps_masked_block_forward(const fps_block_weights* w, const fps_varlen_batch* b,
                                    const void* d_x_act, void* d_y_act, void* d_kv,
                                    const void* d_xu, void* kv_ready, void* d_ws, size_t ws_bytes,
                                    void* stream);

/* The projection building block of a5/a7/a8 on its own (tests and per-kernel measurement):
 * d_out[M, N] = act(d_a[M, K] . d_w[N, K]^T + d_bias) with act 0 = identity, 1 = GELU_tanh.
 * bf16 with K % 64 == 0 and N % 8 == 0 runs the tcgen05 GEMM, anything else the SIMT kernel. */
fps_status fps_linear(int32_t dtype, const void* d_a, const void* d_w, const void* d_bias,
                      int32_t M, int32_t N, int32_t K, int32_t act, void* d_out, void* stream);

/* a6 on its own (tests and per-kernel measurement): for request r and head j,
 * d_o[i, j] = softmax(q_i K_j^T / sqrt(head_dim)) V_j over the request's merged key rows
 * [cu_k[r], cu_k[r+1]) of d_kv ([total_k, 2H], row = K|V), for its active rows
 * [cu_q[r], cu_q[r+1]) of d_q / d_o ([total_q, H]).  Device and host copies of both prefix-sum
 * arrays are required (launch sizing without a device sync). */
fps_status fps_masked_attention(int32_t dtype, const void* d_q, const void* d_kv, void* d_o,
                                int32_t heads, int32_t head_dim, const int32_t* d_cu_q,
                                const int32_t* d_cu_k, const int32_t* h_cu_q,
                                const int32_t* h_cu_k, int32_t n_req, void* stream);

/* Dense block (Fig. 5-Top; the uncached blocks of Fig. 9-Bottom): all L_r rows of every
 * request; b->d_q_row must be NULL and total_q == total_k.  d_kv is scratch [total_k, 2H]. */
fps_status fps_dense_block_forward(const fps_block_weights* w, const fps_varlen_batch* b,
                                   const void* d_x, void* d_y, void* d_kv, void* d_ws,
                                   size_t ws_bytes, void* stream);

/* ---------------------------------------------------------------------------------------
 * a10  Alg. 1 (L211-L219): choose use_cache[l] minimising the step's pipeline latency, under
 * the pipeline model of reading R11: one load stream (cached blocks' loads in
 * order, back to back), one compute stream; KV-mode: block l waits for its own load, plans are
 * monotone, and a final load of `final_load` (the last block's Y rows) ends the step;
 * Y-mode: block l+1 waits for block l's load.  Unbounded staging slots.  Host only.
 *   c_cached[N] = C_w^m, c_dense[N] = C_w/o, load[N] = L^m (any time unit).
 *   use_cache[N] (out), latency (out).  Exact: KV-mode O(N) scan over the N+1 feasible plans;
 *   Y-mode exact Pareto-front DP over (compute end, load end). */
fps_status fps_plan_pipeline(const double* c_cached, const double* c_dense, const double* load,
                             int32_t N, int32_t mode, double final_load, uint8_t* use_cache,
                             double* latency);
/* Cross-step prefetch (NEXT-2, reading R26): loads of step s+1 may start as soon as the load
 * stream is free and step s has consumed their staging slot (one slot per cached block), so
 * the link does not idle at step boundaries.  The per-step latency of a plan is then the
 * long-run step time of that multi-step pipeline (mean over steps 9..16 of a 16-step
 * simulation); the planner scans the N+1 suffix plans.  Host only. */
fps_status fps_plan_pipeline_cross(const double* c_cached, const double* c_dense,
                                   const double* load, int32_t N, int32_t mode,
                                   double final_load, uint8_t* use_cache, double* latency);
double fps_pipeline_latency_cross(const uint8_t* use_cache, const double* c_cached,
                                  const double* c_dense, const double* load, int32_t N,
                                  int32_t mode, double final_load);
/* KV-mode with the transition block (reading R28): the N+1 suffix plans, each priced with its
 * uncached prefix's last block at c_transition[l] (a masked block whose K|V projection covers
 * every row, Y-mode work) instead of c_dense[l] -- when both the prefix and the cached suffix
 * are non-empty.  cross_step 0: the R11 model (fps_pipeline_latency); 1: the R26 steady-state
 * model (fps_pipeline_latency_cross).  Ties -> fewer cached blocks.  c_transition[N] as the
 * other cost arrays.  Host only; FPS_EINVAL on NULL arrays or N < 0. */
fps_status fps_plan_pipeline_kv_transition(const double* c_cached, const double* c_dense,
                                           const double* c_transition, const double* load,
                                           int32_t N, double final_load, int32_t cross_step,
                                           uint8_t* use_cache, double* latency);
/* The model itself (for tests and the balancer): latency of a given plan; +inf if infeasible. */
double fps_pipeline_latency(const uint8_t* use_cache, const double* c_cached,
                            const double* c_dense, const double* load, int32_t N, int32_t mode,
                            double final_load);

/* ---------------------------------------------------------------------------------------
 * Step-level continuous batching over a stack of N blocks (L237, §4.3; Fig. 9 pipeline).
 */
typedef struct {
  int32_t H, heads, F, n_layers, dtype, mode;
  int32_t L_img, L_txt;            /* per-request tokens (text appended after image, R9)   */
  int32_t max_batch;               /* max requests per fps_run_batch call (L326: 8)         */
  int32_t n_steps;                 /* denoising steps of the schedule                       */
  const fps_block_weights* layers; /* [n_layers], device weight pointers (caller-owned)     */
  const void* d_mod_table;         /* [n_layers, n_steps, 6H] adaLN vectors, or NULL        */
  const float* h_deltas;           /* [n_steps] Euler coefficients (copied at create)       */
  fps_cache_t cache;               /* template activation cache (required)                  */
  int32_t slots;                   /* staging slots for layer-ahead prefetch (0 = n_layers) */
  int32_t plan_policy;             /* 0 = Alg. 1 planner; 1 = all cached; 2 = none (dense);
                                      3 = explicit h_plan                                   */
  const uint8_t* h_plan;           /* [n_layers] when plan_policy == 3 (copied at create)   */
  double cost_model[4];            /* planner latency model: comp = a*FLOPs + b,
                                      load = c*bytes + e  -> {a, b, c, e}  (§4.4)     */
  int32_t L_ctx, D_ctx;            /* SDXL blocks: prompt tokens / width of each request's
                                      fps_request.d_ctx (0 if no layer is FPS_BLOCK_SDXL)   */
  int32_t mod_width;               /* elements per d_mod_table row: 0 = 6H; 12H when any
                                      layer is FPS_BLOCK_DOUBLE (image 6H, text 6H; other
                                      blocks read the first 6H)                              */
  int32_t cross_step;              /* 1: cross-step prefetch (R26) -- the next step's loads
                                      start as soon as their slots are consumed, and
                                      plan_policy 0 uses fps_plan_pipeline_cross; needs one
                                      slot per block (slots = 0 or >= n_layers)              */
  int32_t sampler;                 /* the update after the stack (a9):
                                      FPS_SAMPLER_EULER (0): synthetic x += h_deltas[s] * y
                                        over the whole latent (reading R21);
                                      FPS_SAMPLER_FLOW_BLEND (1): flow-matching Euler with
                                        inpainting blend (reading R29): masked image rows
                                        x += (sigma_{s+1} - sigma_s) y, unmasked image rows
                                        x = (1 - sigma_{s+1}) z + sigma_{s+1} eps (the
                                        request's template latent z re-noised with its noise
                                        eps), text rows unchanged                            */
  const float* h_sigmas;           /* [n_steps + 1] noise levels sigma_0 > ... > sigma_S
                                      (FPS_SAMPLER_FLOW_BLEND; copied at create), else NULL  */
  const double* h_layer_comp;      /* [n_layers][2] per-block compute models (a_l, b_l) in
                                      cost_model units -- e.g. fitted per block kind (§4.4
                                      regression per block type); NULL = cost_model[0..1] for
                                      every block.  Copied at create.                        */
} fps_engine_desc;

#define FPS_SAMPLER_EULER 0
#define FPS_SAMPLER_FLOW_BLEND 1

typedef struct fps_engine* fps_engine_t;

typedef struct {
  uint32_t template_id;
  int32_t step;            /* in/out: next denoising step of this request                 */
  int32_t n_steps;         /* request leaves the batch when step == n_steps                */
  const uint8_t* d_mask;   /* [L_img + L_txt] device token mask (text rows nonzero)         */
  void* d_x;               /* [L, H] device latent tokens, updated in place                 */
  int32_t status;          /* out: 0 = running, 1 = finished                                */
  const void* d_ctx;       /* [L_ctx, D_ctx] device prompt encoding (SDXL blocks), or NULL  */
  const void* d_z;         /* [L_img, H] device template latent (FPS_SAMPLER_FLOW_BLEND)    */
  const void* d_noise;     /* [L_img, H] device noise of the request (FPS_SAMPLER_FLOW_BLEND) */
} fps_request;

fps_status fps_engine_create(const fps_engine_desc* desc, fps_engine_t* out);
fps_status fps_engine_destroy(fps_engine_t e);
/* Run up to n_steps denoising steps over reqs[0..n_req) (n_req <= max_batch).  Each step
 * every unfinished request advances by one; a request whose step reaches its n_steps leaves
 * at that step boundary (status = 1) and the batch shrinks.  Admission reads the active-row
 * counts back to the host once per call (the only host sync).  Each step: mask-aware stack
 * with the Alg. 1 plan, layer-ahead prefetch on `load_stream`, final replenish + Euler update
 * x <- x + delta_s * y (reading R21).  The engine's last plan is available below.
 * SDXL blocks: at admission the engine projects every request's d_ctx to the cross-attention
 * K|V of each SDXL block once (fps_context_kv); the prompt is fixed over the steps.
 * Admission reuse: when a call's unfinished requests are exactly the previous call's (same
 * order, same d_mask / d_x / d_ctx pointers and template_id) and none finished since, the call
 * reuses that admission (mask index, batch metadata, prompt K|V, plan) and skips its host
 * synchronisation -- so a serving loop that advances its batch one step per call pays it once
 * per batch change.  Contract: a request's mask and prompt buffers must not be modified while
 * the request is in flight (between its first and its last fps_run_batch call). */
fps_status fps_run_batch(fps_engine_t e, fps_request* reqs, int32_t n_req, int32_t n_steps,
                         void* compute_stream, void* load_stream);
/* Plan and predicted latency (ms) of the last step; use_cache may be NULL. */
fps_status fps_engine_last_plan(fps_engine_t e, uint8_t* use_cache, double* latency_ms);
/* Kernels the engine launched in its last fps_run_batch call (own kernels only). */
int64_t fps_engine_last_launches(fps_engine_t e);
/* Admission reuse on (default, on != 0) or off (every call re-admits; experiments). */
void fps_engine_set_admission_reuse(fps_engine_t e, int32_t on);
/* KV-mode transition block on (default, on != 0) or off (experiments).  In a KV-mode plan the
 * last uncached block before the cached suffix has only its active rows' outputs read later
 * (the next block takes its unmasked K|V from the cache), so the engine runs it as a masked
 * block whose K|V projection covers every row of the fresh full input: the same values for
 * every row read afterwards at the cost of the active rows' attention and MLP (R28).
 * Off: that block runs densely over all rows. */
void fps_engine_set_kv_transition(fps_engine_t e, int32_t on);
/* Measurement switch (default off): when on, the engine issues no cache loads -- each load's
 * ready event is still recorded on the load stream, so the compute stream's ordering is
 * unchanged, and the staging slots keep whatever an earlier step loaded into them.  The step
 * then runs the same plan and the same kernels without any host-link traffic: the "no-load"
 * arm against which exposed load time is measured.  Results are NOT the
 * method's (the cached rows are stale); never use it for output. */
void fps_engine_set_skip_loads(fps_engine_t e, int32_t on);
/* Template run (L130 "prior full inference", L203 the activation store): when on, every block
 * the step runs densely also stores its cache entry (template_id, step, layer) of each request
 * -- KV-mode its K|V rows, Y-mode its output rows, rows [0, L_img) -- with fps_cache_store on
 * the compute stream, and a KV-mode step that ends dense stores the final Y entry (layer =
 * n_layers).  Run the template's requests with plan_policy 2 (all dense) to fill the cache.
 * Default off. */
void fps_engine_set_record(fps_engine_t e, int32_t on);

#ifdef __cplusplus
}
#endif
#endif /* FLASHPS_H */
