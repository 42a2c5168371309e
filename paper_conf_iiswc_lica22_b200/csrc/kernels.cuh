// Device-side parameter blocks and launchers of the Multigrain forward kernels (sm_100a).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "plan.hpp"

namespace mg {

// Strided [B, H, L, 64] 16-bit tensor view (element strides).
struct TensorView {
  uint16_t* data;
  int64_t sb, sh, sl;
};

// Coarse / dense-row / strip kernel: tcgen05 SDDMM -> online SpSoftmax -> tcgen05 SpMM,
// persistent over (item, batch*head) units. See coarse_pp_sm100.cu.
struct CoarseParams {
  const Item* items;
  const TileRef* trefs;
  const uint64_t* masks;
  const int32_t* strip_cols;
  const int32_t* global_rows;
  const int32_t* fine_slot;   // [L]; >= 0: merge fine partial of that slot
  const float* part_acc;      // [BH * n_fine_rows * 64]
  const float2* part_ml;      // [BH * n_fine_rows]  (max in raw score units, sum)
  int32_t* counter;           // [0] work counter, [1] CTAs finished (pp kernel: reset by the last CTA)
  TensorView q, k, v, o;
  int64_t L;
  int32_t H, BH;
  int32_t d;                  // head dimension (64 or 128)
  int32_t n_items, n_dense_items;   // (BH = units per item: B*H, or H for a batched plan)
  int32_t n_global, n_fine_rows;
  int32_t batched;            // batched plan: Item::useB = sample, unit -> (item, head), fine_slot [B][L]
  int32_t total_units;
  float scale_log2;           // (1/sqrt(d)) * log2(e)
  unsigned long long* trace;  // diagnostics: event trace of CTA 0 (null = off)
  int32_t trace_cap;
  // 2-D [rows, 64] views for TMA row gathers (paired-pipeline kernel): row of (b, h, l) =
  // b * r.x + h * r.y + l * r.z; gather_tma = 0 when the strides do not allow such a view
  int32_t gather_tma;
  longlong3 rq, rk, rv;
  // concurrent coarse || fine (plan option): the rows with both a coarse and a CUDA-core CSR part are
  // merged by whichever side finishes the row second (per-row counters, parity = "other side done")
  int32_t concurrent;
  float* part_c_acc;          // [BH * n_fine_rows * 64] coarse partial (written when concurrent)
  float2* part_c_ml;
  int32_t* part_flags;        // [BH * n_fine_rows], +1 per side per forward (even between forwards)
  // padding (A18): valid length per batch element (device [B]) or null; columns >= n_b are masked
  // for every row, rows >= n_b are written as 0
  const int32_t* valid_len;
  // split dense-row items (Item::nrowsB > 1): per (b*h, row group) chunk partials and counters
  float* dense_part;          // [BH][n_dense_groups][dense_nsplit][128][68]: acc[64], m, l, pad (16-B rows)
  int32_t* dense_ctr;         // [BH][n_dense_groups], finished chunks of the current forward (wraps to 0)
  int32_t n_dense_groups, dense_nsplit;
  // band items whose rows are all theirs to write (Item::useA) store O by TMA from shared memory
  // (the item's Q buffer) instead of per-thread row stores
  int32_t tma_store;
  int32_t unit_group;         // band units: 0 = (b,h)-major; G > 0 = groups of G (b,h) units, item-major
                              // within a group (items by decreasing tile count)
  int32_t debug_flags;        // diagnostics (env MG_DEBUG_FLAGS): 1 = no softmax arithmetic, 2 = no MMA, 4 = no loads,
                              // 16 = no S loads from TMEM, 64 = MMA ignores P-ready/O-free (timing only)
};

// Fine CSR kernel: warp per (row, batch*head); SDDMM -> online softmax -> SpMM on CUDA cores.
struct FineParams {
  const int32_t* fine_rows;    // row | (final << 31)
  const int32_t* row_ptr;      // [n_fine_rows + 1]
  const int32_t* cols;
  float* part_acc;
  float2* part_ml;
  TensorView q, k, v, o;
  int32_t H, BH, n_fine_rows;   // (BH = row units per fine row: B*H, or H for a batched plan)
  int32_t d;                    // head dimension (64 or 128; the CUDA-core kernel takes 64 only)
  longlong3 rq, rk, rv;         // TMA gather variant: row of (b, h, l) in the 2-D [rows, 64] views
  const int32_t* fine_sample;   // batched plan: sample of each fine row (else null)
  float scale_log2;
  int32_t concurrent;         // see CoarseParams::concurrent
  const int32_t* valid_len;   // see CoarseParams::valid_len
  const float* part_c_acc;
  const float2* part_c_ml;
  int32_t* part_flags;
  // SM-split mode (plan concurrency 3): rows are claimed dynamically in chunks of 4 from
  // row_ctr[0] (row_ctr[1] counts finished blocks; the last one resets both), so blocks that start
  // late, once the coarse kernel's CTAs leave their SMs, take the remaining rows. null: the static
  // grid-stride row order.
  int32_t* row_ctr;
};

// Staged (paper dataflow) kernels: S and P materialised in the plan's formats; see staged.cu.
struct StagedParams {
  const int32_t* bsr_row_ptr;   // canonical plan (block 128)
  const int32_t* bsr_col;
  const int32_t* tile_row;      // [n_tiles] row block of each tile
  const uint64_t* tile_masks;   // [n_tiles][128][2]
  const int32_t* csr_row_ptr;   // [L + 1]
  const int32_t* csr_col;
  const int32_t* global_rows;
  const uint8_t* row_is_global; // [L]
  TensorView q, k, v, o;
  float* S_t;
  float* S_f;
  float* S_g;
  uint16_t* P_t;
  uint16_t* P_f;
  uint16_t* P_g;
  float* O_f;
  int64_t L, nnz_csr, Lpad;
  int32_t blk0;                 // staged_spmm_tiles: first block index of this launch (split launches)
  int32_t H, BH, nb, n_tiles, n_global;
  float sf;                     // 1 / sqrt(d)
};

// `side`: stream of the CSR kernels (== stream: single-stream order). With a separate side stream
// the caller forks it from `stream` before and joins it after; launch_staged_spmm makes `stream`
// wait for the CSR SpMM (event `ev`) before the BSR row blocks that add O_csr.
cudaError_t launch_staged_sddmm(const StagedParams& p, bool bf16, cudaStream_t stream, cudaStream_t side);
cudaError_t launch_staged_softmax(const StagedParams& p, bool bf16, cudaStream_t stream);
cudaError_t launch_staged_spmm(const StagedParams& p, bool bf16, cudaStream_t stream, cudaStream_t side,
                               cudaEvent_t ev);

// Paired-pipeline variant: two CTAs per SM (grid = 2 x SMs), see coarse_pp_sm100.cu.
cudaError_t launch_coarse_pp(const CoarseParams& p, const CUtensorMap& tmq, const CUtensorMap& tmk,
                             const CUtensorMap& tmv, const CUtensorMap& tmq2, const CUtensorMap& tmk2,
                             const CUtensorMap& tmv2, const CUtensorMap& tmo, bool bf16, bool split_dense, int grid,
                             cudaStream_t stream);
int coarse_pp_ctas_per_sm(int d);
cudaError_t launch_fine(const FineParams& p, bool bf16, cudaStream_t stream);
// Warp-level tensor-core variant (mma.sync m16n8k16), the default; see fine_mma.cu.
cudaError_t launch_fine_mma(const FineParams& p, bool bf16, int sms, cudaStream_t stream);
// Two heads per warp with TMA tile::gather4 row gathers (d = 64, even head count, gather views).
cudaError_t launch_fine_tma2(const FineParams& p, const CUtensorMap& tmq2, const CUtensorMap& tmk2,
                             const CUtensorMap& tmv2, bool bf16, int sms, cudaStream_t stream);
cudaError_t launch_selftest_umma(int mode, const void* A, const void* B, float* D, cudaStream_t stream);

}  // namespace mg
