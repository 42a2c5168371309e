/*
 * mg.h — C ABI of the B200-native Multigrain compound sparse attention forward.
 *
 * Paper: H. Li, J. Choi, J. H. Ahn, "A Slice and Dice Approach to Accelerate Compound
 * Sparse Attention on GPU" (IISWC 2022). "P:n" = line n of that paper's text
 * (/root/reference/PAPER.md at build time; not needed at run time).
 *
 * What the library computes (§2.2): for every batch b and head h, with
 * Q_h, K_h, V_h of shape L x D_h,
 *     S = Q_h K_h^T * (1/sqrt(D_h))          (SDDMM + scaling; reading A1)
 *     S[not M] = -inf                         (masking)
 *     P = row-softmax(S) over the non-zeros   (SpSoftmax)
 *     C_h = P V_h                              (SpMM)
 * where M is the compound mask: sliding window |r-c| <= window/2, symmetric global
 * tokens, and an arbitrary extra residual E.
 *
 * How (§3.1): a host plan splits M into three disjoint parts — coarse BSR tiles
 * (tensor cores), a fine CSR residual (warp-per-row kernels), dense global rows — and
 * the forward merges their softmax statistics so the result is exactly the masked
 * softmax attention above (up to floating-point rounding).
 *
 * Conventions for every function:
 *   - No exceptions cross the ABI. Every call returns an mg_status; on error a
 *     thread-local message is available from mg_last_error().
 *   - Validation happens before any device work; on error nothing is launched and
 *     outputs are untouched.
 *   - Index arrays are int32, tensors are 16-bit (bf16 or fp16) with element strides.
 */
#ifndef MG_H_
#define MG_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MG_ABI_VERSION 1

#if defined(__GNUC__)
#define MG_API __attribute__((visibility("default")))
#else
#define MG_API
#endif

typedef struct mg_plan_s* mg_plan_t;

typedef enum {
  MG_OK = 0,
  MG_ERR_INVALID_ARG = 1,   /* bad sizes, indices out of range, null pointers, layout mismatch */
  MG_ERR_UNSUPPORTED = 2,   /* valid but not implemented (head_dim other than 64/128, block other than 64/128 on fwd, ...) */
  MG_ERR_OUT_OF_MEMORY = 3, /* host or device allocation failed */
  MG_ERR_CUDA = 4,          /* a CUDA runtime/driver error; message in mg_last_error() */
  MG_ERR_INTERNAL = 5
} mg_status;

typedef enum { MG_BF16 = 0, MG_FP16 = 1 } mg_dtype;

/* A [batch, heads, seq_len, head_dim] view of 16-bit data with element strides; the
 * head_dim stride is 1. Both [B,H,L,d] (stride_l = d) and [B,L,H,d] (stride_h = d,
 * stride_l = H*d) are accepted (per-head L x D_h slices of L x D_m hidden states).
 * `data` is a device pointer for mg_sparse_attention_fwd and a host pointer for
 * mg_sparse_attention_fwd_host. data must be 16-byte aligned and every stride a multiple
 * of 8 elements (TMA requirement). */
typedef struct {
  void* data;
  int32_t dtype;      /* mg_dtype */
  int32_t reserved;
  int64_t batch;
  int64_t heads;
  int64_t seq_len;
  int64_t head_dim;
  int64_t stride_b, stride_h, stride_l;
} mg_tensor;

/* ------------------------------------------------------------------------------------
 * Plan (§3.1 steps 1-2: classification and metadata "before inferring the model").
 *
 * mg_plan_create(L, heads, d, window, global_idx, n_global, extra_idx, n_extra, &plan)
 *   L          sequence length, > 0.
 *   heads      number of heads, > 0 (the pattern is shared by all heads).
 *   d          head dimension; v1 supports d == 64 only (else MG_ERR_UNSUPPORTED).
 *   window     local window size, >= 0 and even: |r-c| <= window/2 is valid (reading A2).
 *   global_idx host int32[n_global], positions of global tokens in [0, L); attend to and are
 *              attended by every token (reading A3). Duplicates collapse.
 *   extra_idx  host int32[n_extra][2], (row, col) pairs of extra valid elements in [0, L)^2
 *              (random / selected / dilated residual). Duplicates collapse; pairs
 *              already inside the band or a global row/column are absorbed.
 *   plan       out: a new plan. The index arrays are copied; the caller may free them.
 * The partition is the canonical one (DESIGN.md §3 O-3): tiles of b x b (b = 128) touched by
 * the band of a non-global row are coarse; the coarse tile owns every union element it
 * covers (overlap invalidation); the remaining non-global elements form the CSR
 * residual; global rows are dense and owned by the dense-row part.
 * If a CUDA device is present the metadata is uploaded synchronously to the current device;
 * otherwise the upload is deferred to the first forward call.
 * Errors: INVALID_ARG (L <= 0, heads <= 0, d <= 0, window < 0 or odd, index out of range, tau
 * outside [0, 1],
 * null array with a non-zero count, null plan), UNSUPPORTED (d != 64, CSR nnz >= 2^31),
 * OUT_OF_MEMORY, CUDA.
 * ---------------------------------------------------------------------------------- */
MG_API mg_status mg_plan_create(int64_t L, int32_t heads, int32_t d, int32_t window,
                         const int32_t* global_idx, int64_t n_global,
                         const int32_t* extra_idx, int64_t n_extra,
                         mg_plan_t* plan_out);

/* Test/ablation options. Zero-initialised means "default". */
typedef struct {
  int32_t block;          /* tile size b; 0 -> 128. Any b <= 64 or multiple of 64 builds a plan
                             (for export tests); the forward takes b = 128 or b = 64 (the paper's
                             block: its 64 x 64 BSR tiles run as the quadrants of
                             128 x 128 tcgen05 tiles, non-member quadrants masked, so the forward
                             executes exactly the b = 64 coarse/fine partition). */
  int32_t force_all_fine; /* 1: no coarse tiles; every non-global element goes to the CSR part */
  int32_t strip_max_cols; /* max gathered columns per row block for the tensor-core strip path of
                             the CSR residual; 0 -> default (128); -1 disables the strip path */
  int32_t num_sms;        /* persistent grid size override; 0 -> device SM count */
  int32_t fine_kernel;    /* CSR rows outside strip tiles: 0 -> warp-level tensor-core kernel
                             (mma.sync, default), 1 -> CUDA-core shuffle-reduction kernel (A/B) */
  int32_t concurrency;    /* coarse vs CUDA-core CSR kernels: 0 -> library default, 1 -> serial (fine
                             kernel, then coarse kernel merging its partials), 2 -> concurrent on two
                             streams, rows merged by whichever side finishes second,
                             3 -> SM split: the coarse kernel first on a persistent grid of one CTA
                             per SM on a share of the SMs proportional to its estimated work (env
                             MG_SPLIT_CTAS overrides), the fine kernel beside it on a second stream
                             over the whole device with dynamically claimed rows, merge as in 2
                             (north_star item 5, "run concurrently in different SMs") */
  float tau;              /* tile rule: 0 -> every tile touched by the band of a non-global row is
                             coarse (default, A7); (0, 1] -> a tile is coarse iff its
                             non-global union elements number >= tau * block^2 (A17) */
  int32_t dense_chunk;    /* column tiles per dense-row (global-row) work item: 0 -> default (8),
                             -1 -> one item per 128-row group; chunks are merged by log-sum-exp */
} mg_plan_opts;

MG_API mg_status mg_plan_create_ex(int64_t L, int32_t heads, int32_t d, int32_t window,
                            const int32_t* global_idx, int64_t n_global,
                            const int32_t* extra_idx, int64_t n_extra,
                            const mg_plan_opts* opts, mg_plan_t* plan_out);

/* Batched plan with per-sample special-token positions ("their locations are highly dependent on
 * the input sequence"; the metadata is generated per input): sample b has global tokens
 * global_idx[global_ptr[b] .. global_ptr[b+1]) and extra pairs extra_idx[extra_ptr[b] ..
 * extra_ptr[b+1]) (COO (row, col), int32 [*][2]); the pattern of sample b is the single-plan pattern
 * with those lists (A2-A7). All samples are merged into one work list, so one forward launch
 * covers the whole batch. The forward's Q/K/V/O batch must equal `batch`. Not supported with a
 * batched plan: mg_plan_export and the staged entry points (UNSUPPORTED); mg_plan_info_get returns
 * counts summed over the samples. opts as for mg_plan_create_ex (block 64 or 128; dense-row items
 * are not split). Errors: as mg_plan_create, plus INVALID_ARG for batch <= 0, null or decreasing
 * offset arrays, global_ptr[0] or extra_ptr[0] != 0. */
MG_API mg_status mg_plan_create_batched(int64_t L, int32_t heads, int32_t d, int32_t window, int64_t batch,
                                        const int64_t* global_ptr, const int32_t* global_idx,
                                        const int64_t* extra_ptr, const int32_t* extra_idx,
                                        const mg_plan_opts* opts, mg_plan_t* plan_out);

/* Frees host and device memory of the plan. Must not race with in-flight forwards that use
 * it (synchronize their streams first). Null is accepted (no-op). */
MG_API mg_status mg_plan_destroy(mg_plan_t plan);

/* Thread-local message of the last failing call on this thread ("" if none). */
MG_API const char* mg_last_error(void);

typedef struct {
  int64_t L;
  int32_t heads, d, window, block;
  int64_t n_row_blocks;     /* nb = ceil(L / b) */
  int64_t n_tiles;          /* |T|, coarse BSR tiles */
  int64_t n_full_tiles;     /* tiles whose b*b bits are all set */
  int64_t nnz_coarse;       /* popcount of all tile masks */
  int64_t nnz_fine;         /* CSR residual nnz */
  int64_t n_global;         /* |G| */
  int64_t nnz_total;        /* |M| = nnz_coarse + nnz_fine + n_global * L */
  int64_t n_fine_rows;      /* rows run by the CUDA-core fine kernel */
  int64_t nnz_fine_strip;   /* CSR nnz executed by the tensor-core strip path */
  int64_t nnz_fine_cuda;    /* CSR nnz executed by the warp-per-row CUDA-core kernel */
  int64_t n_items;          /* coarse-kernel work items per (batch, head) */
  int64_t n_strip_tiles;    /* gathered strip tiles per (batch, head) */
  int64_t computed_scores;  /* tensor-core scores per (batch, head) incl. masked waste */
  int32_t kernels_per_fwd;  /* kernel launches per mg_sparse_attention_fwd call */
  int32_t reserved;
} mg_plan_info;

MG_API mg_status mg_plan_info_get(mg_plan_t plan, mg_plan_info* info);

/* Copies the canonical partition into host buffers sized from mg_plan_info:
 *   bsr_row_ptr int32[n_row_blocks+1], bsr_col int32[n_tiles],
 *   tile_masks uint64[n_tiles * block * ceil(block/64)] (row-major, LSB = lowest column),
 *   csr_row_ptr int32[L+1], csr_col int32[nnz_fine], global_rows int32[n_global].
 * Any pointer may be null to skip that array. */
MG_API mg_status mg_plan_export(mg_plan_t plan, int32_t* bsr_row_ptr, int32_t* bsr_col, uint64_t* tile_masks,
                         int32_t* csr_row_ptr, int32_t* csr_col, int32_t* global_rows);

/* ------------------------------------------------------------------------------------
 * Forward (P:96 step 3).
 * mg_sparse_attention_fwd(plan, Q, K, V, O, stream)
 *   Q, K, V  device tensors [batch, heads, L, d] (mg_tensor strides), read only.
 *   O        device tensor, same shape; written for every (b, h, row).
 *   stream   a cudaStream_t (passed as void*); 0 = legacy default stream.
 * Asynchronous: returns after enqueueing; no host synchronisation on the steady-state path.
 * O must not alias Q, K or V (Q/K/V tiles of later work items are read while O rows are written).
 * Q/K/V/O must stay alive until the stream work completes. The plan's fwd workspace (fp32
 * partial statistics of the CSR part) is plan-owned and grown stream-ordered on `stream`,
 * so one plan must not be used by two concurrent forwards on different streams.
 * Errors: INVALID_ARG (null, shape/dtype mismatch with the plan or between tensors,
 * head_dim stride != 1, misaligned data or strides), UNSUPPORTED (block not 64 or 128,
 * dtypes that differ, (L - 1) * stride_l of K or V >= 2^32 elements), CUDA.
 * ---------------------------------------------------------------------------------- */
MG_API mg_status mg_sparse_attention_fwd(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K,
                                  const mg_tensor* V, mg_tensor* O, void* stream);

/* Padded batch ("zero-padding ... masked with -inf"; reading A18): valid_len is a
 * DEVICE int32 array [batch] (values clamped to [0, L]); for batch element b with n = valid_len[b]
 * the mask is M(r,c) AND r < n AND c < n, and the rows r >= n of O are written as 0. Same
 * arguments, asynchrony and errors as mg_sparse_attention_fwd (INVALID_ARG also for a null
 * valid_len). The staged entry points do not take a padding mask. */
MG_API mg_status mg_sparse_attention_fwd_padded(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K,
                                         const mg_tensor* V, mg_tensor* O, const int32_t* valid_len,
                                         void* stream);

/* Same computation with HOST tensors (dense [B,H,L,d] or [B,L,H,d]): copies Q/K/V host->device
 * into plan-owned staging buffers, runs the forward, copies O device->host. The batch is processed
 * in up to 8 chunks on plan-owned copy streams forked from and joined back to `stream`, so the
 * H2D copies of chunk c+1 and the D2H copy of chunk c-1 overlap the forward of chunk c (batched
 * plans: one chunk). Asynchronous with respect to the host (host buffers should be pinned; the
 * caller synchronises `stream` before reading O). Same errors as mg_sparse_attention_fwd. */
MG_API mg_status mg_sparse_attention_fwd_host(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K,
                                       const mg_tensor* V, mg_tensor* O, void* stream);

/* ------------------------------------------------------------------------------------
 * Staged forward ("paper dataflow"): the steps of the method as separate calls with
 * the scores S and probabilities P materialised in the plan's formats, so that each step can be
 * checked on its own and the fused forward can be compared with the paper's dataflow. Same
 * result as mg_sparse_attention_fwd (within the tolerance; P is rounded to 16 bits here).
 *
 * Formats, per (batch, head) unit u = b * heads + h, all row-major device arrays:
 *   S_tiles  float  [B*H][n_tiles][128][128]  coarse scores Q_I K_J^T / sqrt(d) of each BSR tile
 *            (BSR order of mg_plan_export), -inf where the canonical tile bit is 0      (a-2)
 *   S_csr    float  [B*H][nnz_fine]           CSR residual scores, canonical CSR order   (a-3)
 *   S_global float  [B*H][n_global][Lpad]     dense-row scores, -inf at columns >= L     (a-4)
 *   P_tiles / P_csr / P_global: the same shapes in the tensor dtype (bf16 / fp16, RNE):
 *            the compound SpSoftmax of each row over its tiles and CSR elements (global rows:
 *            over their dense row), three sweeps max / sum / normalise as in P:128-131  (a-5)
 *   O_csr    float  [B*H][L][64]              sum_c P(r,c) V[c] over each row's CSR part (a-6);
 *            rows without CSR elements are not written
 *   O        the caller's output tensor: sum_J P_IJ V_J + O_csr (global rows: P_g V)  (a-7, a-8)
 * with Lpad = 128 * ceil(L / 128). mg_staged_get_sizes returns the per-unit element counts
 * (a zero-size part may be passed as NULL). Requires block == 128. All calls are asynchronous
 * on `stream`; buffers belong to the caller. Errors: INVALID_ARG (null plan / tensors / a
 * required buffer, shape mismatch), UNSUPPORTED (block != 128), CUDA.
 * mg_sparse_attention_fwd_staged runs the three calls with plan-owned buffers (grown
 * stream-ordered like the fused forward's workspace).
 * ---------------------------------------------------------------------------------- */
typedef struct {
  int64_t tile_elems;    /* n_tiles * 128 * 128 */
  int64_t csr_elems;     /* nnz_fine */
  int64_t global_elems;  /* n_global * Lpad */
  int64_t ocsr_elems;    /* L * 64 */
  int64_t lpad;
} mg_staged_sizes;

MG_API mg_status mg_staged_get_sizes(mg_plan_t plan, mg_staged_sizes* out);
MG_API mg_status mg_staged_sddmm(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K, float* S_tiles,
                                 float* S_csr, float* S_global, void* stream);
MG_API mg_status mg_staged_softmax(mg_plan_t plan, int64_t batch, mg_dtype dtype, const float* S_tiles,
                                   const float* S_csr, const float* S_global, void* P_tiles, void* P_csr,
                                   void* P_global, void* stream);
MG_API mg_status mg_staged_spmm(mg_plan_t plan, const void* P_tiles, const void* P_csr, const void* P_global,
                                const mg_tensor* V, mg_tensor* O, float* O_csr, void* stream);
MG_API mg_status mg_sparse_attention_fwd_staged(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K,
                                                const mg_tensor* V, mg_tensor* O, void* stream);
/* mg_sparse_attention_fwd_staged_ex: as mg_sparse_attention_fwd_staged; flags bit 0
 * (MG_STAGED_MULTI_STREAM) runs the coarse and fine kernels of each step concurrently on a
 * plan-owned second stream forked from and joined back into `stream` (the paper's multi-stream
 * execution, P:96 step 3): SDDMM of the BSR tiles and dense rows || SDDMM of the CSR
 * residual; the compound SpSoftmax (which needs both parts' statistics) after the join; SpMM of
 * the dense-row chunks || SpMM of the CSR residual, then the BSR row blocks (which add O_csr).
 * Same results bit for bit as the single-stream call. INVALID_ARG for unknown flag bits. */
#define MG_STAGED_MULTI_STREAM 1
MG_API mg_status mg_sparse_attention_fwd_staged_ex(mg_plan_t plan, const mg_tensor* Q, const mg_tensor* K,
                                                   const mg_tensor* V, mg_tensor* O, int32_t flags, void* stream);

/* ------------------------------------------------------------------------------------
 * Profiling (tracing subsystem). When enabled, every forward records CUDA events on its
 * stream around each kernel it launches; mg_plan_get_profile() synchronises on the recorded
 * events, returns the summed device durations since the last enable/reset, and resets.
 * Durations are per kernel class: fine = CUDA-core CSR kernel, coarse = tensor-core kernel
 * (band + strip + dense-row items), total = from the first to the last launch of each call.
 * ---------------------------------------------------------------------------------- */
typedef struct {
  int64_t calls;
  double fine_ms, coarse_ms, total_ms;
} mg_profile;

MG_API mg_status mg_plan_set_profiling(mg_plan_t plan, int32_t enable);
MG_API mg_status mg_plan_get_profile(mg_plan_t plan, mg_profile* out);
/* mg_plan_get_profile_calls: as mg_plan_get_profile, and also writes the first-to-last-launch
 * duration of each recorded call, in call order, to per_call_ms[0 .. min(calls, cap)) (host
 * buffer owned by the caller; may be null when cap == 0), so that a caller can report the median
 * and minimum of a timed run. INVALID_ARG: null plan/out, cap < 0, or cap > 0 with a null buffer. */
MG_API mg_status mg_plan_get_profile_calls(mg_plan_t plan, mg_profile* out, double* per_call_ms, int64_t cap);

/* ------------------------------------------------------------------------------------
 * Per-pattern choice of the coarse/fine split by measured cost ("the more low-sparsity
 * sparse blocks there are, the more benefits the fine-grained kernel has"; blocked
 * patterns). mg_plan_autotune builds one plan per candidate (block b in {128, 64} x density
 * threshold tau in {0, 0.1, 0.25, 0.5}, A17), times each candidate's forward on the caller's
 * device tensors (2 warm-up + 5 timed calls, CUDA events on `stream`, median) and returns the
 * fastest plan; *chosen (may be null) receives its options and *best_ms its median time. The
 * patterns are as for mg_plan_create; O is overwritten (scratch). Synchronous (it waits for the
 * timing events). Errors: as mg_plan_create and mg_sparse_attention_fwd; the candidates' plans are
 * destroyed on every path.
 * ---------------------------------------------------------------------------------- */
MG_API mg_status mg_plan_autotune(int64_t L, int32_t heads, int32_t d, int32_t window, const int32_t* global_idx,
                                  int64_t n_global, const int32_t* extra_idx, int64_t n_extra, const mg_tensor* Q,
                                  const mg_tensor* K, const mg_tensor* V, mg_tensor* O, void* stream,
                                  mg_plan_t* plan_out, mg_plan_opts* chosen, double* best_ms);

/* ------------------------------------------------------------------------------------
 * Diagnostics (used by the GPU tests; not part of the attention path).
 * mg_selftest_umma(mode, A, B, D, stream): one 128 x N x K tcgen05 MMA on device buffers.
 *   mode 0: D[128x128] fp32 = A[128x64] bf16 (K-major, SMEM) * B[128x64]^T bf16 (K-major)
 *   mode 1: D[128x64]  fp32 = A[128x128] bf16 (staged SMEM->TMEM, TS form) * B[128x64] bf16
 *           (B row-major over K: MN-major operand)
 * All buffers are row-major device arrays. Returns CUDA on launch failure.
 * ---------------------------------------------------------------------------------- */
MG_API mg_status mg_selftest_umma(int32_t mode, const void* A, const void* B, float* D, void* stream);

/* mg_plan_set_trace(plan, buf, cap): diagnostics. While set, a library built with MG_TRACE adds
 * per-role, per-phase cycle counters of the tensor-core kernel (uint64, summed over CTAs) to the
 * zeroed device buffer `buf` of `cap` >= 128 uint64 elements: element role*16 + k is phase k of
 * role (0 producer, 1 MMA issuer, 2/3 softmax column halves), element role*16 + 15 the number of
 * CTAs that reported. Normal builds ignore the buffer. (null, 0) turns it off. Errors:
 * INVALID_ARG for a null plan or a buffer with cap < 128. */
MG_API mg_status mg_plan_set_trace(mg_plan_t plan, void* device_buffer, int64_t capacity_events);

MG_API int32_t mg_abi_version(void);

#ifdef __cplusplus
}
#endif

#endif /* MG_H_ */
