// Host-side Multigrain plan: canonical coarse/fine/dense-row partition + kernel work lists.
// Paper: P:94-96 (§3.1 steps 1-2, metadata generated before inference), P:101 (local ->
// coarse BSR, selected -> fine CSR), P:103/P:133 (global rows dense and independent),
// P:126 (overlap invalidated). Rules: DESIGN.md §3 (O-3).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

namespace mg {

struct PlanOptions {
  int block = 128;
  bool force_all_fine = false;
  int strip_max_cols = 128;  // <= 0 disables the tensor-core strip path for the CSR residual
};

// Device work-list encodings. The tensor-core kernel runs two softmax
// streams (A and B) on two 128-row Q tiles that share the K/V tiles of one work item.
//   Item {kind, rowA, rowB, ntiles, tref_begin, nrowsA, nrowsB}:
//     kind 0: band row blocks starting at rows rowA and rowB (adjacent blocks with coarse tiles);
//     kind 1: gathered global rows global_rows[rowA ..) against every column tile (dense part);
//     kind 2: like kind 1, but both streams work on the same rows (rowA == rowB) and take
//             alternate column tiles (A even, B odd); their partial rows are merged at the end;
//     nrowsX = valid rows of stream X (0 = stream unused); useX = bit j set if stream X uses tile j
//     (items with more than 64 tiles are dense items: kind 1 uses every tile, kind 2 alternates).
//   TileRef {arg, kind, ncols, maskA, maskB}: one K/V tile of the item, loaded once:
//     kind 0 = contiguous column tile at column `arg`; kind 1 = gathered strip whose column list
//     starts at strip_cols[arg]; maskX = index of a 128 x 2-word bitmask for stream X,
//     -1 = all valid, -2 = stream X does not use this tile.
struct Item {
  int32_t kind, rowA, rowB, ntiles, tref_begin, nrowsA, nrowsB;
  int32_t turns;  // exp half-tiles per softmax stream (max over A, B) when both are active, else 0
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

// Returns "" on success, else an error message; *unsupported is set for UNSUPPORTED errors.
std::string build_plan(HostPlan& p, int64_t L, int32_t heads, int32_t d, int32_t window,
                       const int32_t* global_idx, int64_t n_global, const int32_t* extra_idx,
                       int64_t n_extra, const PlanOptions& opts, bool* unsupported);

}  // namespace mg
