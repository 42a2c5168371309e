// Host plan builder. See plan.hpp and DESIGN.md §3-§5.
//
// Canonical partition (must be bit-identical to oracle/plan.py; readings A2-A7):
//   M(r,c) = |r-c| <= w/2 or G[r] or G[c] or (r,c) in E
//   T = {(I,J): some non-global r in row block I has band columns in column block J}
//       ("local pattern -> coarse BSR"; tau = 0), or with tau > 0 (A17)
//   T = {(I,J): #non-global union elements in the tile >= tau * b^2}
//   tile bits = M restricted to the tile, global rows cleared
//   CSR = non-global union elements outside T ("selected -> fine CSR")
#include "plan.hpp"

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <iterator>

namespace mg {

namespace {

inline int popcount64(uint64_t x) { return __builtin_popcountll(x); }

}  // namespace

// Band items in decreasing tile count (stable), for the coarse kernel's item-major unit order
// (CoarseParams::unit_order): the short band-edge items are claimed last, so the persistent CTAs'
// finishing times differ by less than one short item. MG_UNIT_ORDER=0 keeps the build order (A/B).
bool item_major_order() {
  static const bool on = [] {
    const char* e = std::getenv("MG_UNIT_ORDER");
    return !(e && e[0] == '0');
  }();
  return on;
}
void sort_band_items(std::vector<Item>& items, int32_t n_dense) {
  if (!item_major_order() || (int32_t)items.size() <= n_dense) return;
  std::stable_sort(items.begin() + n_dense, items.end(),
                   [](const Item& a, const Item& b) { return a.ntiles > b.ntiles; });
}


std::string build_plan(HostPlan& p, int64_t L, int32_t heads, int32_t d, int32_t window,
                       const int32_t* global_idx, int64_t n_global, const int32_t* extra_idx,
                       int64_t n_extra, const PlanOptions& opts, bool* unsupported) {
  *unsupported = false;
  if (L <= 0) return "L must be > 0";
  if (heads <= 0) return "heads must be > 0";
  if (d <= 0) return "d must be > 0";
  if (window < 0 || (window & 1)) return "window must be >= 0 and even";
  if (n_global < 0 || n_extra < 0) return "negative index count";
  if (n_global > 0 && !global_idx) return "global_idx is null";
  if (n_extra > 0 && !extra_idx) return "extra_idx is null";
  const int b = opts.block;
  if (b < 1 || (b > 64 && b % 64) || b > 1024) return "block must be <= 64 or a multiple of 64 (<= 1024)";
  if (!(opts.tau >= 0.0 && opts.tau <= 1.0)) return "tau must be in [0, 1]";
  if (d != 64 && d != 128) { *unsupported = true; return "head_dim must be 64 or 128"; }
  for (int64_t i = 0; i < n_global; ++i)
    if (global_idx[i] < 0 || global_idx[i] >= L) return "global index out of range";
  for (int64_t i = 0; i < 2 * n_extra; ++i)
    if (extra_idx[i] < 0 || extra_idx[i] >= L) return "extra index out of range";

  p = HostPlan();
  p.L = L; p.heads = heads; p.d = d; p.window = window; p.block = b; p.opts = opts;
  const int64_t w1 = window / 2;
  const int64_t nb = p.nb();
  const int wpr = p.wpr();

  // ---- global rows: sorted unique
  std::vector<uint8_t> isG(L, 0);
  for (int64_t i = 0; i < n_global; ++i) isG[global_idx[i]] = 1;
  for (int64_t r = 0; r < L; ++r) if (isG[r]) p.global_rows.push_back((int32_t)r);
  const std::vector<int32_t>& gcols = p.global_rows;

  // ---- extras: set semantics, grouped by row
  std::vector<int64_t> keys(n_extra);
  for (int64_t i = 0; i < n_extra; ++i) keys[i] = (int64_t)extra_idx[2 * i] * L + extra_idx[2 * i + 1];
  std::sort(keys.begin(), keys.end());
  keys.erase(std::unique(keys.begin(), keys.end()), keys.end());
  std::vector<int64_t> ext_ptr(L + 1, 0);
  for (int64_t k : keys) ext_ptr[k / L + 1]++;
  for (int64_t r = 0; r < L; ++r) ext_ptr[r + 1] += ext_ptr[r];

  // ---- per row block: tiles, bits, CSR
  std::vector<int32_t> tile_of_J(nb, -1);
  std::vector<int64_t> csr_ptr(L + 1, 0);
  p.bsr_row_ptr.push_back(0);
  std::vector<std::vector<int32_t>> outs(b);   // off-band union columns of each row of the block
  std::vector<int64_t> cnt(nb, 0);
  for (int64_t I = 0; I < nb; ++I) {
    const int64_t r0 = I * b, r1 = std::min<int64_t>(L, r0 + b);
    // off-band columns from globals and extras, merged ascending, unique
    for (int64_t r = r0; r < r1; ++r) {
      std::vector<int32_t>& outside = outs[r - r0];
      outside.clear();
      if (isG[r]) continue;
      const int64_t lo = std::max<int64_t>(0, r - w1), hi = std::min<int64_t>(L - 1, r + w1);
      size_t gi = 0;
      int64_t ei = ext_ptr[r], ee = ext_ptr[r + 1];
      while (gi < gcols.size() || ei < ee) {
        int64_t c;
        if (ei >= ee || (gi < gcols.size() && gcols[gi] <= keys[ei] % L)) {
          c = gcols[gi++];
          if (ei < ee && keys[ei] % L == c) ++ei;
        } else {
          c = keys[ei++] % L;
        }
        if (c < lo || c > hi) outside.push_back((int32_t)c);
      }
    }
    std::vector<uint8_t> inT(nb, 0);
    if (!opts.force_all_fine && opts.tau <= 0.0) {
      for (int64_t r = r0; r < r1; ++r) {
        if (isG[r]) continue;
        const int64_t jlo = std::max<int64_t>(0, r - w1) / b;
        const int64_t jhi = std::min<int64_t>(L - 1, r + w1) / b;
        for (int64_t J = jlo; J <= jhi; ++J) inT[J] = 1;
      }
    } else if (!opts.force_all_fine) {
      // density rule: count the union elements of the block's non-global rows per column block
      std::fill(cnt.begin(), cnt.end(), 0);
      for (int64_t r = r0; r < r1; ++r) {
        if (isG[r]) continue;
        const int64_t lo = std::max<int64_t>(0, r - w1), hi = std::min<int64_t>(L - 1, r + w1);
        for (int64_t J = lo / b; J <= hi / b; ++J)
          cnt[J] += std::min<int64_t>(hi, J * b + b - 1) - std::max<int64_t>(lo, J * b) + 1;
        for (int32_t c : outs[r - r0]) cnt[c / b]++;
      }
      const double thr = opts.tau * (double)b * (double)b;
      for (int64_t J = 0; J < nb; ++J) inT[J] = (double)cnt[J] >= thr;
    }
    for (int64_t J = 0; J < nb; ++J) {
      tile_of_J[J] = -1;
      if (inT[J]) { tile_of_J[J] = (int32_t)p.bsr_col.size(); p.bsr_col.push_back((int32_t)J); }
    }
    p.bsr_row_ptr.push_back((int32_t)p.bsr_col.size());
    p.tile_masks.resize(p.bsr_col.size() * (size_t)b * wpr, 0ull);

    for (int64_t r = r0; r < r1; ++r) {
      if (isG[r]) continue;  // global rows: owned by the dense-row part
      const int64_t a = r - r0;
      auto take = [&](int64_t c) {  // c is a union column of row r
        const int64_t J = c / b;
        const int32_t t = tile_of_J[J];
        if (t >= 0) {
          const int64_t beta = c - J * b;
          p.tile_masks[((size_t)t * b + a) * wpr + beta / 64] |= 1ull << (beta % 64);
        } else {
          p.csr_col.push_back((int32_t)c);
          csr_ptr[r + 1]++;
        }
      };
      const int64_t lo = std::max<int64_t>(0, r - w1), hi = std::min<int64_t>(L - 1, r + w1);
      const std::vector<int32_t>& outside = outs[a];
      // emit in ascending column order: outside-left, band, outside-right
      size_t oi = 0;
      while (oi < outside.size() && outside[oi] < lo) take(outside[oi++]);
      for (int64_t c = lo; c <= hi; ++c) take(c);
      while (oi < outside.size()) take(outside[oi++]);
    }
  }
  for (int64_t r = 0; r < L; ++r) csr_ptr[r + 1] += csr_ptr[r];
  if (csr_ptr[L] >= (int64_t(1) << 31)) { *unsupported = true; return "CSR nnz >= 2^31"; }
  p.csr_row_ptr.assign(csr_ptr.begin(), csr_ptr.end());

  const int64_t nt = (int64_t)p.bsr_col.size();
  for (int64_t t = 0; t < nt; ++t) {
    int64_t pc = 0;
    for (int64_t w = 0; w < (int64_t)b * wpr; ++w) pc += popcount64(p.tile_masks[t * b * wpr + w]);
    p.nnz_coarse += pc;
    if (pc == (int64_t)b * b) p.n_full_tiles++;
  }

  // ---- kernel-side structures: the tcgen05 kernel computes 128 x 128 tiles (M = 128). With b = 128
  // the kernel tiles are the BSR tiles. With b = 64 (the paper's block size) each
  // kernel tile groups the 2 x 2 block of 64-tiles it covers: its bitmask is the union of the member
  // 64-tiles' masks, non-member quadrants are all zero (their union elements are in the b = 64 CSR
  // residual), so the forward executes exactly the b = 64 partition.
  if (b != 128 && b != 64) return "";
  p.kernel_ready = true;
  const int64_t B = 128;
  const int64_t nbk = (L + B - 1) / B;
  std::vector<int32_t> k_row_ptr, k_col;
  if (b == 128) {
    k_row_ptr = p.bsr_row_ptr;
    k_col = p.bsr_col;
    p.dev_masks.assign(p.tile_masks.begin(), p.tile_masks.end());  // 256 words per tile
  } else {
    k_row_ptr.push_back(0);
    std::vector<int32_t> slot(nbk, -1);
    for (int64_t I = 0; I < nbk; ++I) {
      const int64_t first = (int64_t)k_col.size();
      for (int64_t a = 0; a < 2 && 2 * I + a < nb; ++a)
        for (int32_t t = p.bsr_row_ptr[2 * I + a]; t < p.bsr_row_ptr[2 * I + a + 1]; ++t) {
          const int32_t Jk = p.bsr_col[t] / 2;
          if (slot[Jk] < 0) {
            slot[Jk] = 0;
            k_col.push_back(Jk);
          }
        }
      std::sort(k_col.begin() + first, k_col.end());
      for (int64_t i = first; i < (int64_t)k_col.size(); ++i) slot[k_col[i]] = (int32_t)i;
      p.dev_masks.resize(k_col.size() * 256, 0ull);
      for (int64_t a = 0; a < 2 && 2 * I + a < nb; ++a)
        for (int32_t t = p.bsr_row_ptr[2 * I + a]; t < p.bsr_row_ptr[2 * I + a + 1]; ++t) {
          const int32_t kt = slot[p.bsr_col[t] / 2], q = p.bsr_col[t] & 1;
          for (int r = 0; r < 64; ++r) p.dev_masks[(size_t)kt * 256 + (a * 64 + r) * 2 + q] = p.tile_masks[(size_t)t * 64 + r];
        }
      for (int64_t i = first; i < (int64_t)k_col.size(); ++i) slot[k_col[i]] = -1;
      k_row_ptr.push_back((int32_t)k_col.size());
    }
  }
  const int64_t nkt = (int64_t)k_col.size();
  std::vector<uint8_t> tile_full(nkt, 0);
  for (int64_t t = 0; t < nkt; ++t) {
    bool full = true;
    for (int w = 0; w < 256 && full; ++w) full = p.dev_masks[t * 256 + w] == ~0ull;
    tile_full[t] = full;
  }
  auto new_mask = [&]() -> int32_t {
    const int32_t id = (int32_t)(p.dev_masks.size() / 256);
    p.dev_masks.resize(p.dev_masks.size() + 256, 0ull);
    return id;
  };
  auto count = [&](int32_t mask, int ncols, int nrows) {
    if (mask == kMaskSkip || nrows == 0) return;
    p.computed_scores += B * ncols;
    p.softmax_tiles += 1;
  };

  // dense items (global rows): two streams of up to 128 gathered rows, every column tile
  int32_t ragged_mask = kMaskFull;
  if (L % B) {
    ragged_mask = new_mask();
    const int64_t valid = L - (nbk - 1) * B;
    for (int a = 0; a < 128; ++a)
      for (int64_t c = 0; c < valid; ++c) p.dev_masks[(size_t)ragged_mask * 256 + a * 2 + c / 64] |= 1ull << (c % 64);
  }
  // dense items (global rows): up to 128 gathered rows against every column tile
  const int64_t G = (int64_t)p.global_rows.size();
  for (int64_t k = 0; k < G; k += 128) {
    const int32_t nr = (int32_t)std::min<int64_t>(128, G - k);
    Item it{1, (int32_t)k, (int32_t)(k / 128), (int32_t)nbk, (int32_t)p.trefs.size(), nr, 1, 0, 0ull, 0ull};
    for (int64_t J = 0; J < nbk; ++J) {
      const int32_t m = (J == nbk - 1) ? ragged_mask : kMaskFull;
      p.trefs.push_back(TileRef{(int32_t)(J * B), 0, 128, m, kMaskSkip, 0, 0, 0});
      count(m, 128, nr);
    }
    p.items.push_back(it);
    p.n_dense_groups++;
  }
  // the same rows split into chunks of <= dense_chunk column tiles (a separate work list, chosen
  // per forward when the dense items would be too few to spread over the SMs); the chunks' fp32
  // partials are merged by the last chunk to finish. The chunks reuse the unsplit items' tile refs.
  const int64_t chunk = std::max<int64_t>(1, std::min<int64_t>(opts.dense_chunk, nbk));
  const int32_t nsplit = (int32_t)((nbk + chunk - 1) / chunk);
  p.dense_nsplit = nsplit;
  for (const Item& d : p.items) {
    for (int32_t sc = 0; sc < nsplit; ++sc) {
      const int64_t J0 = sc * chunk, J1 = std::min<int64_t>(nbk, J0 + chunk);
      p.items_split.push_back(Item{1, d.rowA, d.rowB, (int32_t)(J1 - J0), d.tref_begin + (int32_t)J0, d.nrowsA,
                                   nsplit, sc, 0ull, 0ull});
    }
  }
  p.n_dense_items_split = (int32_t)p.items_split.size();
  p.n_dense_items = (int32_t)p.items.size();

  // distinct CSR columns of each row block
  std::vector<std::vector<int32_t>> blk_cols(nbk);
  for (int64_t I = 0; I < nbk; ++I) {
    const int64_t r0 = I * B, r1 = std::min<int64_t>(L, r0 + B);
    auto& cols = blk_cols[I];
    for (int64_t r = r0; r < r1; ++r)
      cols.insert(cols.end(), p.csr_col.begin() + p.csr_row_ptr[r], p.csr_col.begin() + p.csr_row_ptr[r + 1]);
    std::sort(cols.begin(), cols.end());
    cols.erase(std::unique(cols.begin(), cols.end()), cols.end());
  }
  const int strip_max = opts.strip_max_cols;
  std::vector<uint8_t> blk_strip(nbk, 0);  // CSR residual of the block carried by a strip tile
  // strip tile over `cols` with the bitmask of row block I (kMaskSkip if I < 0)
  auto strip_mask = [&](int64_t I, const std::vector<int32_t>& cols, int ncols) -> int32_t {
    if (I < 0) return kMaskSkip;
    const int64_t r0 = I * B, r1 = std::min<int64_t>(L, r0 + B);
    const int32_t m = new_mask();
    bool full = r1 - r0 == B;
    for (int64_t r = r0; r < r0 + B; ++r) {
      const int64_t a = r - r0;
      if (r >= r1) continue;
      const int32_t* cb = p.csr_col.data() + p.csr_row_ptr[r];
      const int32_t* ce = p.csr_col.data() + p.csr_row_ptr[r + 1];
      if (ce - cb != ncols) full = false;
      for (const int32_t* c = cb; c != ce; ++c) {
        const int64_t beta = std::lower_bound(cols.begin(), cols.end(), *c) - cols.begin();
        p.dev_masks[(size_t)m * 256 + a * 2 + beta / 64] |= 1ull << (beta % 64);
      }
      p.nnz_fine_strip += ce - cb;
    }
    if (full) {  // drop the unused mask again (it is the last one allocated)
      p.dev_masks.resize(p.dev_masks.size() - 256);
      return kMaskFull;
    }
    return m;
  };
  auto push_strip = [&](int64_t I, const std::vector<int32_t>& cols) {
    const int ncols = (int)((cols.size() + 31) / 32 * 32);
    const int32_t off = (int32_t)p.strip_cols.size();
    for (int i = 0; i < ncols; ++i) p.strip_cols.push_back(i < (int)cols.size() ? cols[i] : -1);
    const int32_t m = strip_mask(I, cols, ncols);
    p.trefs.push_back(TileRef{off, 1, ncols, m, kMaskSkip, 0, 0, 0});
    count(m, ncols, 1);
    p.n_strip_tiles++;
  };

  // band items: one per row block with coarse tiles (its BSR tiles, then its strip if any)
  for (int64_t I = 0; I < nbk; ++I) {
    if (k_row_ptr[I + 1] == k_row_ptr[I]) continue;
    const int32_t nr = (int32_t)std::min<int64_t>(B, L - I * B);
    Item it{0, (int32_t)(I * B), 0, 0, (int32_t)p.trefs.size(), nr, 0, 0, 0ull, 0ull};
    for (int32_t t = k_row_ptr[I]; t < k_row_ptr[I + 1]; ++t) {
      const int32_t m = tile_full[t] ? kMaskFull : t;
      p.trefs.push_back(TileRef{k_col[t] * (int32_t)B, 0, 128, m, kMaskSkip, 0, 0, 0});
      count(m, 128, nr);
    }
    // CSR residual as a tensor-core strip where the block's distinct columns are few
    const std::vector<int32_t>& cols = blk_cols[I];
    if (strip_max > 0 && !cols.empty() && (int)cols.size() <= strip_max) {
      push_strip(I, cols);
      blk_strip[I] = 1;
    }
    it.ntiles = (int32_t)p.trefs.size() - it.tref_begin;
    p.items.push_back(it);
    p.items_split.push_back(it);
  }

  // CSR rows left to the CUDA-core fine kernel
  p.fine_slot.assign(L, -1);
  for (int64_t I = 0; I < nbk; ++I) {
    if (blk_strip[I]) continue;
    const bool has_tiles = k_row_ptr[I + 1] > k_row_ptr[I];
    const int64_t r0 = I * B, r1 = std::min<int64_t>(L, r0 + B);
    for (int64_t r = r0; r < r1; ++r) {
      if (p.csr_row_ptr[r + 1] == p.csr_row_ptr[r]) continue;
      if (has_tiles) p.fine_slot[r] = (int32_t)p.fine_rows.size();
      p.fine_rows.push_back((int32_t)r | (has_tiles ? 0 : (int32_t)0x80000000));
    }
  }
  // band items whose rows are all written by this item (bit 0: no global row; bit 1: no CUDA-core
  // CSR row, which the concurrent mode may let the fine kernel write)
  for (auto* list : {&p.items, &p.items_split}) {
    for (Item& it : *list) {
      if (it.kind != 0) continue;
      bool no_global = true, no_fine = true;
      for (int64_t r = it.rowA; r < it.rowA + it.nrowsA; ++r) {
        no_global = no_global && !isG[r];
        no_fine = no_fine && p.fine_slot[r] < 0;
      }
      it.useA = (no_global ? 1ull : 0ull) | (no_fine ? 2ull : 0ull);
    }
  }
  p.fine_row_ptr.assign(1, 0);
  for (int32_t enc : p.fine_rows) {
    const int32_t r = enc & 0x7fffffff;
    p.fine_col.insert(p.fine_col.end(), p.csr_col.begin() + p.csr_row_ptr[r], p.csr_col.begin() + p.csr_row_ptr[r + 1]);
    p.fine_row_ptr.push_back((int32_t)p.fine_col.size());
  }
  sort_band_items(p.items, p.n_dense_items);
  sort_band_items(p.items_split, p.n_dense_items_split);
  return "";
}

std::string build_batched_plan(HostPlan& out, int64_t L, int32_t heads, int32_t d, int32_t window, int64_t batch,
                               const int64_t* global_ptr, const int32_t* global_idx, const int64_t* extra_ptr,
                               const int32_t* extra_idx, const PlanOptions& opts, bool* unsupported) {
  *unsupported = false;
  if (batch <= 0) return "batch must be > 0";
  if (!global_ptr || !extra_ptr) return "global_ptr / extra_ptr is null";
  if (global_ptr[0] != 0 || extra_ptr[0] != 0) return "global_ptr[0] and extra_ptr[0] must be 0";
  for (int64_t b = 0; b < batch; ++b)
    if (global_ptr[b + 1] < global_ptr[b] || extra_ptr[b + 1] < extra_ptr[b]) return "offsets must be non-decreasing";
  if (opts.block != 128 && opts.block != 64) { *unsupported = true; return "batched plans require block 64 or 128"; }
  PlanOptions po = opts;
  po.dense_split = 1;   // the split dense-row list is not built for batched plans
  std::vector<HostPlan> ps(batch);
  for (int64_t b = 0; b < batch; ++b) {
    const int64_t ng = global_ptr[b + 1] - global_ptr[b], ne = extra_ptr[b + 1] - extra_ptr[b];
    std::string e = build_plan(ps[b], L, heads, d, window, global_idx ? global_idx + global_ptr[b] : nullptr, ng,
                               extra_idx ? extra_idx + 2 * extra_ptr[b] : nullptr, ne, po, unsupported);
    if (!e.empty()) return "sample " + std::to_string(b) + ": " + e;
  }
  out = HostPlan();
  out.L = L; out.heads = heads; out.d = d; out.window = window; out.block = 128; out.opts = po;
  out.kernel_ready = true;
  out.batch = batch;
  out.fine_slot.assign((size_t)batch * L, -1);
  out.fine_row_ptr.assign(1, 0);
  // dense items of every sample first (longest first, as in a single plan), then the band items
  std::vector<int32_t> tref_off(batch), mask_off(batch), strip_off(batch), grow_off(batch), fine_off(batch);
  for (int64_t b = 0; b < batch; ++b) {
    const HostPlan& h = ps[b];
    tref_off[b] = (int32_t)out.trefs.size();
    mask_off[b] = (int32_t)(out.dev_masks.size() / 256);
    strip_off[b] = (int32_t)out.strip_cols.size();
    grow_off[b] = (int32_t)out.global_rows.size();
    fine_off[b] = (int32_t)out.fine_rows.size();
    for (TileRef tr : h.trefs) {
      if (tr.maskA >= 0) tr.maskA += mask_off[b];
      if (tr.kind == 1) tr.arg += strip_off[b];
      out.trefs.push_back(tr);
    }
    out.dev_masks.insert(out.dev_masks.end(), h.dev_masks.begin(), h.dev_masks.end());
    out.strip_cols.insert(out.strip_cols.end(), h.strip_cols.begin(), h.strip_cols.end());
    out.global_rows.insert(out.global_rows.end(), h.global_rows.begin(), h.global_rows.end());
    for (size_t i = 0; i < h.fine_rows.size(); ++i) {
      out.fine_rows.push_back(h.fine_rows[i]);
      out.fine_sample.push_back((int32_t)b);
      const int32_t* cb = h.fine_col.data() + h.fine_row_ptr[i];
      const int32_t* ce = h.fine_col.data() + h.fine_row_ptr[i + 1];
      out.fine_col.insert(out.fine_col.end(), cb, ce);
      out.fine_row_ptr.push_back((int32_t)out.fine_col.size());
    }
    for (int64_t r = 0; r < L; ++r)
      if (h.fine_slot[r] >= 0) out.fine_slot[(size_t)b * L + r] = h.fine_slot[r] + fine_off[b];
    out.nnz_coarse += h.nnz_coarse;
    out.n_full_tiles += h.n_full_tiles;
    out.nnz_fine_strip += h.nnz_fine_strip;
    out.n_strip_tiles += h.n_strip_tiles;
    out.computed_scores += h.computed_scores;
    out.softmax_tiles += h.softmax_tiles;
    out.nnz_total_sum += h.nnz_coarse + (int64_t)h.csr_col.size() + (int64_t)h.global_rows.size() * L;
    out.csr_col.resize(out.csr_col.size() + h.csr_col.size());   // (counts only; not exported)
    out.bsr_col.resize(out.bsr_col.size() + h.bsr_col.size());
  }
  for (int pass = 0; pass < 2; ++pass) {
    for (int64_t b = 0; b < batch; ++b) {
      const HostPlan& h = ps[b];
      for (int32_t i = 0; i < (int32_t)h.items.size(); ++i) {
        const bool dense = i < h.n_dense_items;
        if (dense != (pass == 0)) continue;
        Item it = h.items[i];
        it.tref_begin += tref_off[b];
        if (it.kind == 1) it.rowA += grow_off[b];
        it.useB = (uint64_t)b;
        out.items.push_back(it);
      }
    }
    if (pass == 0) out.n_dense_items = (int32_t)out.items.size();
  }
  sort_band_items(out.items, out.n_dense_items);
  out.items_split = out.items;
  out.n_dense_items_split = out.n_dense_items;
  out.dense_nsplit = 1;
  if (out.csr_col.size() >= (size_t(1) << 31)) { *unsupported = true; return "CSR nnz >= 2^31"; }
  return "";
}

}  // namespace mg
