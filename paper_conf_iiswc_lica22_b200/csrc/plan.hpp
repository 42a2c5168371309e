// Host-side Multigrain plan: canonical coarse/fine/dense-row partition + kernel work lists.
// Paper: P:94-96 (§3.1 steps 1-2, metadata generated before inference), P:101 (local ->
// coarse BSR, selected -> fine CSR), P:103/P:133 (global rows dense and independent),
// P:126 (overlap invalidated). Rules: DESIGN.md §3 (O-3).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

namespace mg {

bool item_major_order();   // band units item-major with items by decreasing tile count (plan.cpp)

struct PlanOptions {
  int block = 128;
  bool force_all_fine = false;
  int strip_max_cols = 128;  // <= 0 disables the tensor-core strip path for the CSR residual
  double tau = 0.0;          // 0: band rule; > 0: a tile is coarse iff its density >= tau (A17)
  int dense_chunk = 8;       // column tiles per split dense-row work item
  int dense_split = 0;       // 0: split dense items when the forward has few of them, 1: never, 2: always
};

// Device work-list encodings. The tensor-core kernel processes one 128-row
// Q tile per work item against the item's list of K/V tiles.
//   Item {kind, rowA, -, ntiles, tref_begin, nrowsA, ...}:
//     kind 0: band row block starting at row rowA (a block with coarse tiles);
//     kind 1: gathered global rows global_rows[rowA ..) against column tiles (dense part); the
//       row group's nb column tiles are split into nrowsB chunks of <= dense_chunk tiles, one item
//       each: rowB = row group, turns = chunk index; with nrowsB > 1 every chunk writes an fp32
//       partial and the last chunk to finish merges them;
//     nrowsA = valid rows of the Q tile. useA (kind 0): bit 0 = no global row in the block, bit 1 =
//     no CUDA-core CSR row (then every row is written by this item alone, so O may be stored as a
//     tile; bit 1 matters only in the concurrent mode).
//     useB is reserved (0).
//   TileRef {arg, kind, ncols, maskA, -}: one K/V tile of the item:
//     kind 0 = contiguous column tile at column `arg`; kind 1 = gathered strip whose column list
//     starts at strip_cols[arg] (ncols a multiple of 32); maskA = index of a 128 x 2-word bitmask,
//     -1 = all valid. maskB is reserved (-2).
struct Item {
  int32_t kind, rowA, rowB, ntiles, tref_begin, nrowsA, nrowsB;
  int32_t turns;
  uint64_t useA, useB;
};
struct TileRef { int32_t arg, kind, ncols, maskA, maskB, pad0, pad1, pad2; };
constexpr int32_t kMaskFull = -1, kMaskSkip = -2;

struct HostPlan {
  // inputs
  int64_t L = 0;
  int32_t heads = 0, d = 0, window = 0, block = 128;
  PlanOptions opts;
  // canonical partition (exported, bit-exact vs oracle)
  std::vector<int32_t> global_rows, bsr_row_ptr, bsr_col, csr_row_ptr, csr_col;
  std::vector<uint64_t> tile_masks;  // n_tiles * block * wpr
  int64_t nnz_coarse = 0, n_full_tiles = 0;
  // kernel-side structures (built only when block == 128)
  bool kernel_ready = false;
  std::vector<uint64_t> dev_masks;   // 128 x 2 words per entry: tiles, then strip/ragged masks
  std::vector<Item> items;           // dense items first, then band items in row-block order
  int32_t n_dense_items = 0;
  int32_t n_dense_groups = 0, dense_nsplit = 1;
  // batched plan (per-sample global / extra positions): batch > 0 samples merged into one
  // work list; Item::useB = sample; fine_slot is [batch][L]; fine_sample[i] = sample of fine row i
  int64_t batch = 0;
  std::vector<int32_t> fine_sample;
  int64_t nnz_total_sum = 0;
  // alternative work list with the dense items split into chunks (same band items after them)
  std::vector<Item> items_split;
  int32_t n_dense_items_split = 0;
  std::vector<TileRef> trefs;
  std::vector<int32_t> strip_cols;   // gathered column lists (padded with -1)
  std::vector<int32_t> fine_rows;    // rows executed by the CUDA-core fine kernel; bit 31 = write final O
  std::vector<int32_t> fine_slot;    // per row: index into fine_rows for partial merge, or -1
  std::vector<int32_t> fine_row_ptr; // compacted CSR (cuda part only) [n_fine_rows + 1]
  std::vector<int32_t> fine_col;
  int64_t nnz_fine_strip = 0, n_strip_tiles = 0, computed_scores = 0, softmax_tiles = 0;

  int64_t nb() const { return (L + block - 1) / block; }
  int wpr() const { return (block + 63) / 64; }
};

// Per-sample plans merged into one batched work list (see HostPlan::batch). Returns "" or an error.
std::string build_batched_plan(HostPlan& out, int64_t L, int32_t heads, int32_t d, int32_t window, int64_t batch,
                               const int64_t* global_ptr, const int32_t* global_idx, const int64_t* extra_ptr,
                               const int32_t* extra_idx, const PlanOptions& opts, bool* unsupported);

// Returns "" on success, else an error message; *unsupported is set for UNSUPPORTED errors.
std::string build_plan(HostPlan& p, int64_t L, int32_t heads, int32_t d, int32_t window,
                       const int32_t* global_idx, int64_t n_global, const int32_t* extra_idx,
                       int64_t n_extra, const PlanOptions& opts, bool* unsupported);

}  // namespace mg
