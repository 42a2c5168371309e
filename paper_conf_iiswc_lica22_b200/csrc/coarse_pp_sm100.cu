// Coarse-grained fused kernel for sm_100a, "paired pipelines" design: two co-resident CTAs per SM,
// each an independent pipeline over the work items of the plan. One work item = one 128-row Q
// tile (a band row block, or up to 128 gathered global rows) of one (batch, head) and its list of
// K/V tiles:
//   SDDMM   S = Q K_j^T            tcgen05.mma (SS), S in TMEM            (§3.2)
//   scale + mask + online SpSoftmax  thread t owns row t of the Q tile   (§3.3)
//   SpMM    O += P_j V_j           tcgen05.mma (TS: P from TMEM)         (§3.2)
// The per-row running (max, sum) is carried across the row's tiles instead of re-reading S
// (A14: the paper's 3-sweep SpSoftmax becomes an online softmax; same result).
//   kind 0 items: a band row block with its BSR tiles (+ a gathered "strip" tile carrying the
//     block's CSR residual on the tensor cores); the epilogue merges the fp32 partial statistics
//     written by the CUDA-core fine kernel for any remaining CSR rows (compound SpSoftmax);
//   kind 1 items: gathered global rows against every column tile (dense-row part).
//
// TMEM (256 columns per CTA, two CTAs fill the SM's 512): S [0,128) fp32, P [128,192) packed
// 16-bit pairs, O [192,256) fp32. S and P are separate so that S(n+1) is issued as soon as the
// softmax warps have *read* S(n) (s_free), i.e. while they compute the exponentials of tile n;
// P(n) is stored at the end of the tile, after P.V(n-1) has consumed P(n-1) (pv_done).
// While one CTA's softmax waits on its MMA chain, the other CTA's softmax owns the SM's MUFU and
// FMA pipes: the two pipelines interleave without any shared barrier.
//
// Warp roles (256 threads = two warpgroups):
//   warps 0-3  softmax + epilogue: thread t = row t of the Q tile = TMEM lane t (warp w owns the
//              TMEM lane quarter w, as tcgen05.ld/st require)
//   warp 4     producer: TMA of Q/K/V tiles (SWIZZLE_128B) and bitmasks; TMA row gathers
//              (tile::gather4) for global-row Q tiles and strip K/V tiles
//   warp 5     TMEM allocator; lane 0 issues the MMAs: S(n), then P.V(n-1)
//   warp 6     scheduler: claims work items (atomic counter) into a 4-deep ring, L2 prefetch of
//              each band item's Q tile
//   warp 7     idle (completes the control warpgroup for setmaxnreg)
// Shared memory: Q[2], K[2], V[2] 16 KB tiles (separate K and V rings: K(n+2) may load as soon
// as S(n) has completed, V(n+2) after P.V(n)).
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "kernels.cuh"
#include "sm100_ptx.cuh"

namespace mg {

using namespace ptx;

namespace {

// Column-split softmax: 8 softmax warps per CTA, two per TMEM lane quarter, each taking 64 of a
// tile's 128 columns (the pair exchanges its half-tile row maxima through shared memory and a
// 64-thread named barrier); 384 threads per CTA, control warps 8-11. At d = 128 (one CTA per SM)
// this gives each SM sub-partition two softmax warps instead of one (MG_CSPLIT128, default on);
// at d = 64 (two CTAs per SM, MG_CSPLIT) it measured slower (C2 0.1555 vs 0.1427 ms).
#ifndef MG_CSPLIT
#define MG_CSPLIT 0
#endif
#ifndef MG_CSPLIT128
#define MG_CSPLIT128 1
#endif
template <int kD>
struct WCfg {
  static constexpr bool kCS = kD == 64 ? (bool)MG_CSPLIT : (bool)MG_CSPLIT128;
  static constexpr int kSoftWarps = kCS ? 8 : 4;
  static constexpr int kThreads = 32 * (kSoftWarps + 4);
  static constexpr int kWProd = kSoftWarps, kWMma = kSoftWarps + 1, kWSched = kSoftWarps + 2, kWIdle = kSoftWarps + 3;
  // setmaxnreg per warpgroup: (65536 / CTAs per SM / threads, rounded down to 8) per thread in the pool
  static constexpr int kRegsCtl = kCS ? (kD == 64 ? 48 : 88) : 64;
  static constexpr int kRegsSoftmax = kCS ? (kD == 64 ? 96 : 208) : 192;
};
static_assert(256 * 96 + 128 * 48 <= (65536 / 2 / 384 & ~7) * 384, "register pool (column split, d = 64)");
static_assert(256 * 208 + 128 * 88 <= (65536 / 1 / 384 & ~7) * 384, "register pool (column split, d = 128)");
constexpr int kThreads = 256;
constexpr int kSt = 2;                       // K ring and V ring depth
// work-item ring depth: a CTA's scheduler claims at most kItems - 1 items ahead of its softmax warps;
// 2 measured best (C2 0.1393 vs 0.1410, C3 0.0734 vs 0.0754, C5 1.048 vs 1.068 ms at 4; 6 worse
// still): items claimed ahead by a busy CTA are the end-of-kernel imbalance
#ifndef MG_ITEMS
#define MG_ITEMS 2
#endif
constexpr int kItems = MG_ITEMS;
constexpr uint32_t kSub = 128 * 128;         // one SWIZZLE_128B sub-tile: 128 rows x 64 x 16-bit
constexpr uint32_t kMaskBytes = 128 * 16;    // 128 rows x 128 validity bits
constexpr uint32_t kTS = 0, kTP = 128;       // TMEM columns of S (fp32) and P (packed 16-bit pairs)

// Head dimension kD = 64 or 128 (D_h). A Q/K/V/O tile is kD / 64 sub-tiles of 64 columns
// (one TMA box / one 128-byte swizzle row each). d = 64: two CTAs per SM (TMEM 256 columns: S, P,
// O [192, 256)); d = 128: one CTA per SM (TMEM 512: S, P, O [256, 384); shared memory 6 x 32 KB).
template <int kD>
struct DCfg {
  static constexpr uint32_t kTileBytes = 128 * kD * 2;
  static constexpr int kNSub = kD / 64;
  static constexpr uint32_t kTmemCols = kD == 64 ? 256 : 512;
  static constexpr uint32_t kTO = kD == 64 ? 192 : 256;
  static constexpr int kMinBlocks = kD == 64 ? 2 : 1;
};

struct __align__(16) Slot {
  Item item;
  int32_t u, bh, pad0, pad1;
};

struct __align__(16) Ctl {
  Slot slot[kItems];
  int32_t kcols[kSt];                         // ncols of the tile in K stage s (producer -> MMA)
  int2 vdesc[kSt];                            // {ncols, maskA} of the tile in V stage s (-> softmax)
  uint32_t cmask[kSt][4];                     // padding: valid columns of the tile in V stage s
  uint64_t item_full[kItems], item_empty[kItems];
  uint64_t q_full[2], q_empty[2];
  uint64_t k_full[kSt], k_empty[kSt], v_full[kSt], v_empty[kSt];
  uint64_t s_full, s_free, p_full, pv_done;
  uint64_t mk_full[kSt], mk_empty[kSt];       // late-P.V mode: tile descriptor / bitmask ring
  uint32_t tmem_base;
  int32_t dense_last;                         // split dense item: this chunk finished its row group last
  float xmax[2][2][128];                      // column split: [tile parity][half][row] half-tile maxima
  float xsum[128];                            // column split: half 1's row sum for the epilogue
};

template <int kD>
constexpr size_t smem_bytes() {
  return 1024 + 6 * DCfg<kD>::kTileBytes + kSt * kMaskBytes + sizeof(Ctl);
}
static_assert(smem_bytes<64>() <= 113 * 1024, "two CTAs per SM at d = 64");
static_assert(smem_bytes<128>() <= 227 * 1024, "one CTA per SM at d = 128");
// setmaxnreg applies per warpgroup: warps 0-3 (softmax) grow, warps 4-7 (control) shrink. The
// pool of one CTA is (65536 / CTAs per SM / kThreads) x kThreads registers.
constexpr int kRegsCtl = 64, kRegsSoftmax = 192;
static_assert(128 * kRegsCtl + 128 * kRegsSoftmax <= (65536 / 2 / kThreads & ~7) * kThreads, "register pool");

struct UnitInfo {
  int item, bh;
};

// dense units first (long items start early), then band units: in groups of unit_group (b,h) units
// (a group's K/V stays in L2), item-major within a group with the items sorted by decreasing tile
// count on the host, so the short band-edge items come last; or (b,h)-major, row-block order
__device__ __forceinline__ UnitInfo decode_unit(const CoarseParams& p, int u) {
  const int dense_units = p.n_dense_items * p.BH;
  if (u < dense_units) return {u % p.n_dense_items, u / p.n_dense_items};
  const int v = u - dense_units;
  const int nband = p.n_items - p.n_dense_items;
  if (p.unit_group > 0) {   // groups of unit_group (b,h) units, item-major within a group
    const int per_group = nband * p.unit_group;
    const int hg = v / per_group, w = v - hg * per_group;
    const int gsize = min(p.unit_group, p.BH - hg * p.unit_group);
    return {p.n_dense_items + w / gsize, hg * p.unit_group + w % gsize};
  }
  return {p.n_dense_items + v % nband, v / nband};
}

// Copy rows idx[0..nvalid) (idx < 0 -> zeros) of a [*, kD] 16-bit matrix into a K-major
// SWIZZLE_128B tile of kD / 64 sub-tiles (64-column sub-tile s at dst + s * kSub; row r at r*128 B,
// 16-byte chunk c at (c ^ (r & 7)) * 16); rows [nvalid, nfill) are zero-filled. One warp; each lane
// keeps kBatch 16-byte loads in flight.
template <int kD>
__device__ __forceinline__ void gather_rows(uint32_t dst, const uint16_t* base, int64_t sl, const int32_t* idx,
                                            int nvalid, int nfill, int lane) {
  constexpr int kBatch = 4, kCh = kD / 8;   // 16-byte chunks per row
  const int total = nfill * kCh;
  for (int e0 = 0; e0 < total; e0 += 32 * kBatch) {
    int4 val[kBatch];
#pragma unroll
    for (int k = 0; k < kBatch; ++k) {
      const int e = e0 + k * 32 + lane, r = e / kCh;
      val[k] = make_int4(0, 0, 0, 0);
      if (e < total && r < nvalid) {
        const int src = __ldg(idx + r);
        if (src >= 0) val[k] = ld_nc_v4(base + (int64_t)src * sl + (e % kCh) * 8);
      }
    }
#pragma unroll
    for (int k = 0; k < kBatch; ++k) {
      const int e = e0 + k * 32 + lane, r = e / kCh, ch = e % kCh;
      if (e < total) {
        const uint32_t a = dst + (ch >> 3) * kSub + r * 128 + (((ch & 7) ^ (r & 7)) << 4);
        asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(val[k].x), "r"(val[k].y),
                     "r"(val[k].z), "r"(val[k].w)
                     : "memory");
      }
    }
  }
}


// 4 consecutive gather indices idx[i0 .. i0+4) (entries at or beyond n -> -1), 16-byte aligned
__device__ __forceinline__ int4 load_idx4(const int32_t* idx, int i0, int n) {
  int4 v = make_int4(-1, -1, -1, -1);
  if (i0 + 3 < n) {
    v = __ldg(reinterpret_cast<const int4*>(idx + i0));
  } else if (i0 < n) {
    v.x = __ldg(idx + i0);
    if (i0 + 1 < n) v.y = __ldg(idx + i0 + 1);
    if (i0 + 2 < n) v.z = __ldg(idx + i0 + 2);
  }
  return v;
}


template <bool kBF16>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  return kBF16 ? pack_bf16(lo, hi) : pack_f16(lo, hi);
}

__device__ __forceinline__ int4 ld_shared_v4(uint32_t a) {
  int4 v;
  asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}

// S values of one 32-column chunk with validity bits `bits` (bit i = column i): masked -> -inf.
__device__ __forceinline__ void apply_mask(uint32_t (&r)[32], uint32_t bits) {
#pragma unroll
  for (int i = 0; i < 32; ++i)
    if (!((bits >> i) & 1u)) r[i] = __float_as_uint(-INFINITY);
}

__device__ __forceinline__ float chunk_max(const uint32_t (&r)[32], float mx) {
  float a = mx, b = -INFINITY, c = -INFINITY, d = -INFINITY;
#pragma unroll
  for (int i = 0; i < 32; i += 8) {
    a = fmax3(a, __uint_as_float(r[i]), __uint_as_float(r[i + 1]));
    b = fmax3(b, __uint_as_float(r[i + 2]), __uint_as_float(r[i + 3]));
    c = fmax3(c, __uint_as_float(r[i + 4]), __uint_as_float(r[i + 5]));
    d = fmax3(d, __uint_as_float(r[i + 6]), __uint_as_float(r[i + 7]));
  }
  return fmaxf(fmaxf(a, b), fmaxf(c, d));
}

// 2^x for a pair on the FMA pipe (x <= 8): Cody-Waite split x = j + f with j = rint(x) (1.5 * 2^23
// magic add), f in [-1/2, 1/2]; 2^f by a cubic (relative error 2.2e-4, far below the 2^-9 of the
// 16-bit P it feeds); 2^j added to the exponent field. x is clamped to -126 so that masked (-inf)
// scores give a denormal-range value ~1e-38 instead of 0, which no output can distinguish.
__device__ __forceinline__ float2 exp2_fma2(float2 x) {
  x.x = fmaxf(x.x, -126.f);
  x.y = fmaxf(x.y, -126.f);
  const float2 t = __fadd2_rn(x, make_float2(12582912.f, 12582912.f));
  const float2 r = __fadd2_rn(t, make_float2(-12582912.f, -12582912.f));
  const float2 f = __fadd2_rn(x, make_float2(-r.x, -r.y));
  float2 p = __ffma2_rn(make_float2(0.05286743491888046f, 0.05286743491888046f), f,
                        make_float2(0.2421518862247467f, 0.2421518862247467f));
  p = __ffma2_rn(p, f, make_float2(0.6935867667198181f, 0.6935867667198181f));
  p = __ffma2_rn(p, f, make_float2(0.9999627470970154f, 0.9999627470970154f));
  return make_float2(__int_as_float(__float_as_int(t.x) * 0x800000 + __float_as_int(p.x)),
                     __int_as_float(__float_as_int(t.y) * 0x800000 + __float_as_int(p.y)));
}

// Pairs (of 16 per 32-column chunk) whose exponentials run on the FMA pipe instead of MUFU.
// Measured on C2/C3/C4 (tools/ab_variants.sh): with the exponentials ahead of the P.V(n-1) wait the
// steady state is MUFU-bound, and 2 of 16 pairs per 32-column chunk on the FMA pipe is best
// (C2 0.1466 -> 0.1423 ms; 1 or 3 pairs: 0.1433 / 0.1462; 4: 0.154; C3 within 1%).
#ifndef MG_EXP_EMU
#define MG_EXP_EMU 2
#endif
constexpr int kExpEmu = MG_EXP_EMU;

// Diagnostics builds (MG_DBG=bits, results are garbage): 1 = no exponentials, 2 = no MMAs,
// 4 = no K/V loads. Compile-time so that the measured build carries no runtime checks.
#ifndef MG_DBG
#define MG_DBG 0
#endif
constexpr bool kDbgNoExp = MG_DBG & 1, kDbgNoMma = MG_DBG & 2, kDbgNoLoads = MG_DBG & 4;
#ifndef MG_SKIP_MAX
#define MG_SKIP_MAX 1
#endif

// p = 2^(s*c - m*c) for 32 columns, packed to 16-bit pairs; row sum accumulated in rs[0..1]
template <bool kBF16>
__device__ __forceinline__ void chunk_exp(const uint32_t (&r)[32], float2 c2, float2 nb2, float2 (&rs)[2],
                                          uint32_t (&pk)[16]) {
#pragma unroll
  for (int i = 0; i < 32; i += 2) {
    const float2 x = __ffma2_rn(make_float2(__uint_as_float(r[i]), __uint_as_float(r[i + 1])), c2, nb2);
    float2 pp;
    if (kDbgNoExp) {
      pp = x;
    } else if ((i >> 1) < kExpEmu) {
      pp = exp2_fma2(x);
    } else {
      pp.x = ex2(x.x);
      pp.y = ex2(x.y);
    }
    rs[(i >> 1) & 1] = __fadd2_rn(rs[(i >> 1) & 1], pp);
    pk[i >> 1] = pack2<kBF16>(pp.x, pp.y);
  }
}

// p = 2^(s*c - m*c) for 32 columns in place (fp32); row sum accumulated in rs[0..1]
__device__ __forceinline__ void chunk_exp_f32(uint32_t (&r)[32], float2 c2, float2 nb2, float2 (&rs)[2]) {
#pragma unroll
  for (int i = 0; i < 32; i += 2) {
    const float2 x = __ffma2_rn(make_float2(__uint_as_float(r[i]), __uint_as_float(r[i + 1])), c2, nb2);
    float2 pp;
    if ((i >> 1) < kExpEmu) {
      pp = exp2_fma2(x);
    } else {
      pp.x = ex2(x.x);
      pp.y = ex2(x.y);
    }
    rs[(i >> 1) & 1] = __fadd2_rn(rs[(i >> 1) & 1], pp);
    r[i] = __float_as_uint(pp.x);
    r[i + 1] = __float_as_uint(pp.y);
  }
}

// Diagnostics (MG_TIMELINE builds only): per-tile event clocks (low 32 bits of clock64) of every
// CTA for its first kTlTiles tiles, kTlF fields per tile (16 S in registers, 17 exponentials done,
// 18 = 1 if S(n+1) was complete when P(n) was stored), after 256 uint64 header words of p.trace:
// 0 softmax S(n)+V(n) ready, 1 softmax P.V(n-1) done, 2 softmax warp 0 P(n) stored, 3 MMA S(n)
// issued, 4 MMA P.V(n) issued, 5 producer K(n) issued, 6 producer V(n) issued, 7 MMA sees p_full(n),
// 8-10 softmax warps 1-3 P(n) stored, 11/12/13 epilogue start / O read / end (last tile of an
// item), 14 MMA sees k_full(n), 15 SM id (tile 0 only). tools/timeline_pp.py reads it.
constexpr int kTlTiles = 128, kTlF = 24;   // tiles recorded per CTA, fields per tile
__device__ __forceinline__ void tl_rec(const CoarseParams& p, uint32_t n, int field) {
#ifdef MG_TIMELINE
  if (p.trace == nullptr || n >= (uint32_t)kTlTiles ||
      (int64_t)p.trace_cap < 256 + (int64_t)(kTlF / 2) * kTlTiles * (int64_t)gridDim.x)
    return;
  uint32_t v = (uint32_t)clock64();
  if (field == 15) asm("mov.u32 %0, %%smid;" : "=r"(v));
  reinterpret_cast<uint32_t*>(p.trace + 256)[((size_t)blockIdx.x * kTlTiles + n) * kTlF + field] = v;
#endif
}

// a value instead of a clock (field 18: S(n+1) already complete when P(n) is stored)
__device__ __forceinline__ void tl_val(const CoarseParams& p, uint32_t n, int field, uint32_t v) {
#ifdef MG_TIMELINE
  if (p.trace == nullptr || n >= (uint32_t)kTlTiles ||
      (int64_t)p.trace_cap < 256 + (int64_t)(kTlF / 2) * kTlTiles * (int64_t)gridDim.x)
    return;
  reinterpret_cast<uint32_t*>(p.trace + 256)[((size_t)blockIdx.x * kTlTiles + n) * kTlF + field] = v;
#endif
}

// Item-level events (MG_TIMELINE): [CTA][item < 32][8] uint32 after the tile records: 0 scheduler
// slot free, 1 scheduler item published, 2 producer item seen, 3 producer Q issued, 4 producer tile
// refs loaded, 5 softmax item seen, 6 MMA item seen, 7 MMA Q ready.
__device__ __forceinline__ void tl_item(const CoarseParams& p, uint32_t it, int field) {
#ifdef MG_TIMELINE
  if (p.trace == nullptr || it >= 32u ||
      (int64_t)p.trace_cap < 256 + (int64_t)((kTlF / 2) * kTlTiles + 128) * (int64_t)gridDim.x)
    return;
  reinterpret_cast<uint32_t*>(p.trace + 256)[(size_t)gridDim.x * kTlTiles * kTlF + ((size_t)blockIdx.x * 32 + it) * 8 +
                                             field] = (uint32_t)clock64();
#endif
}

// lane quarters without valid rows skip the softmax: measured slower (C2 0.1525 vs 0.1428 ms, C3
// 0.0819 vs 0.0779, same box, r02), so off by default (MG_IDLE_QUARTERS=1 builds it)
#ifndef MG_IDLE_QUARTERS
#define MG_IDLE_QUARTERS 0
#endif
constexpr bool kIdleQuarters = MG_IDLE_QUARTERS;

// Mask ring (MG_MASK_RING, default): the tile descriptors and bitmasks travel in their own
// two-stage ring, released by the softmax warps once read, instead of with the V stage (released
// only when P.V(n) has completed), so a tile's softmax never waits for its V load (measured C2
// 0.1426 vs 0.1433 ms, C3 0.0774 vs 0.0782, same box).
// Late P.V (MG_PV_LATE, off): the MMA warp issues P.V(n-1) after S(n+1) instead of after S(n), so
// the next S does not queue behind a P.V in the in-order tensor pipe (an item's last P.V, which the
// epilogue waits on, still goes right after the next S): measured slower (C2 0.168 vs 0.141 ms),
// the softmax then waits on the later P.V before its P store.
#ifndef MG_PV_LATE
#define MG_PV_LATE 0
#endif
#ifndef MG_MASK_RING
#define MG_MASK_RING 1
#endif
constexpr bool kLatePV = MG_PV_LATE;
constexpr bool kLate = MG_MASK_RING || MG_PV_LATE;   // (the mask ring; the late P.V needs it)

#ifndef MG_PRE_CHUNKS
#define MG_PRE_CHUNKS 4
#endif
constexpr int kPre = MG_PRE_CHUNKS;   // chunks whose exponentials precede the P.V(n-1) wait

struct TileCtx {
  uint32_t tl;          // TMEM address of this warp's lane quarter (column 0)
  uint32_t mask_row;    // shared address of this row's 16 mask bytes
  bool masked;          // the tile has a bitmask (else all columns valid)
  const uint32_t* cmask;  // padding: 4 words of valid columns (shared memory), or null
  uint32_t n;           // tile sequence number (CTA lifetime)
  int j;                // tile index within the item
  uint32_t s_free, pv_done, p_full;
  float c, thresh;
  const CoarseParams* prm;   // diagnostics only (tl_rec, debug_flags)
  uint32_t s_full;           // diagnostics only (timeline field 18)
};

// One tile of the online SpSoftmax for this thread's row (NQ x 32 columns): read S(n) from TMEM
// and release it, mask, row max, lazy rescale decision, then (after P.V(n-1)) rescale O if the
// max moved and store P(n) = 2^(s*c - m*c) as packed 16-bit pairs, chunk by chunk.
template <int NQ, bool kBF16, int kD>
__device__ __forceinline__ void softmax_tile(const TileCtx& x, float& m, float& l) {
  constexpr uint32_t kTO = DCfg<kD>::kTO;
  const uint32_t lane = threadIdx.x & 31;
  uint32_t r[NQ][32];
#pragma unroll
  for (int q = 0; q < NQ; ++q) tmem_ld32(x.tl + kTS + q * 32, r[q]);
  tmem_wait_ld();
  if (threadIdx.x == 0) tl_rec(*x.prm, x.n, 16);
  tc_fence_before();
  __syncwarp();
  if (lane == 0) mbar_arrive(x.s_free);                 // S may be overwritten by S(n+1)
  if (x.masked || x.cmask) {
    uint32_t w4[4] = {~0u, ~0u, ~0u, ~0u};
    if (x.masked) {
      const int4 mw = ld_shared_v4(x.mask_row);
      w4[0] = (uint32_t)mw.x;
      w4[1] = (uint32_t)mw.y;
      w4[2] = (uint32_t)mw.z;
      w4[3] = (uint32_t)mw.w;
    }
    if (x.cmask) {
#pragma unroll
      for (int q = 0; q < NQ; ++q) w4[q] &= x.cmask[q];
    }
#pragma unroll
    for (int q = 0; q < NQ; ++q) apply_mask(r[q], w4[q]);
  }
  float tmax = -INFINITY;
#pragma unroll
  for (int q = 0; q < NQ; ++q) tmax = chunk_max(r[q], tmax);
  const bool need = tmax > m + x.thresh || (m == -INFINITY && tmax != -INFINITY);
  float alpha = 1.f;
  if (need) {
    alpha = ex2((m - tmax) * x.c);                      // 0 when m = -inf
    m = tmax;
  }
  l *= alpha;
  const float mu = (m == -INFINITY) ? 0.f : m;
  const float2 c2 = make_float2(x.c, x.c);
  const float2 nb2 = make_float2(-mu * x.c, -mu * x.c);
  float2 rs[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
  // the first kPre chunks' exponentials are computed before waiting for P.V(n-1) (they overlap its
  // issue and execution; their packed P waits in registers)
  constexpr int kPreN = kPre < NQ ? kPre : NQ;
  uint32_t pre[kPreN > 0 ? kPreN : 1][16];
#pragma unroll
  for (int q = 0; q < kPreN; ++q) chunk_exp<kBF16>(r[q], c2, nb2, rs, pre[q]);
  if (threadIdx.x == 0) tl_rec(*x.prm, x.n, 17);
  // P.V(n-1) has consumed P(n-1) and updated O: rescale O if the max moved, then store P(n)
  // chunk by chunk as it is produced (the other CTA on this SM keeps the pipes busy meanwhile)
  if (x.n > 0) mbar_wait(x.pv_done, (x.n - 1) & 1);
  if (threadIdx.x == 0) tl_rec(*x.prm, x.n, 1);
  tc_fence_after();
  if (x.j > 0 && __any_sync(0xffffffffu, need && alpha != 1.f)) {
#pragma unroll 1
    for (int h = 0; h < kD / 16; ++h) {
      uint32_t o[16];
      tmem_ld16(x.tl + kTO + h * 16, o);
      tmem_wait_ld();
#pragma unroll
      for (int i = 0; i < 16; ++i) o[i] = __float_as_uint(__uint_as_float(o[i]) * alpha);
      tmem_st16(x.tl + kTO + h * 16, o);
    }
  }
#pragma unroll
  for (int q = 0; q < kPreN; ++q) tmem_st16(x.tl + kTP + q * 16, pre[q]);
#pragma unroll
  for (int q = kPreN; q < NQ; ++q) {
    uint32_t pk[16];
    chunk_exp<kBF16>(r[q], c2, nb2, rs, pk);
    tmem_st16(x.tl + kTP + q * 16, pk);
  }
  l += (rs[0].x + rs[0].y) + (rs[1].x + rs[1].y);
  tmem_wait_st();
  tc_fence_before();
  __syncwarp();
  if (lane == 0) {
    mbar_arrive(x.p_full);
    tl_rec(*x.prm, x.n, threadIdx.x == 0 ? 2 : 7 + (threadIdx.x >> 5));
#ifdef MG_TIMELINE
    if (threadIdx.x == 0) tl_val(*x.prm, x.n, 18, mbar_test_wait(x.s_full, (x.n + 1) & 1) ? 1u : 0u);
#endif
  }
}

// Column-split variant of softmax_tile (d = 64): this warp holds NH (0..2) of the tile's 32-column
// chunks, chunks [2h, 2h + NH); the half-tile maxima of the two warps sharing the rows are combined
// before the lazy-rescale decision, so both warps take the same (deterministic) decision and use
// the same reference max for P. Each warp keeps its own partial row sum; it rescales O columns
// [32h, 32h + 32) and stores P columns [32h, 32h + 32) (packed pairs).
template <int NH, bool kBF16, int kD>
__device__ __forceinline__ void softmax_tile_cs(const TileCtx& x, float& m, float& l, int h, int row,
                                                uint32_t xbar, float* xmax) {
  constexpr uint32_t kTO = DCfg<kD>::kTO;
  const uint32_t lane = threadIdx.x & 31;
  uint32_t r[NH > 0 ? NH : 1][32];
#pragma unroll
  for (int q = 0; q < NH; ++q) tmem_ld32(x.tl + kTS + (2 * h + q) * 32, r[q]);
  if (NH > 0) tmem_wait_ld();
  tc_fence_before();
  __syncwarp();
  if (lane == 0) mbar_arrive(x.s_free);                 // S may be overwritten by S(n+1)
  if (NH > 0 && (x.masked || x.cmask)) {
    uint32_t w2[2] = {~0u, ~0u};
    if (x.masked) {
      const int4 mw = ld_shared_v4(x.mask_row);
      w2[0] = (uint32_t)(h ? mw.z : mw.x);
      w2[1] = (uint32_t)(h ? mw.w : mw.y);
    }
    if (x.cmask) {
#pragma unroll
      for (int q = 0; q < NH; ++q) w2[q] &= x.cmask[2 * h + q];
    }
#pragma unroll
    for (int q = 0; q < NH; ++q) apply_mask(r[q], w2[q]);
  }
  float tmax = -INFINITY;
#pragma unroll
  for (int q = 0; q < NH; ++q) tmax = chunk_max(r[q], tmax);
  // half-tile maxima of the pair -> tile max (double-buffered by tile parity: a slot is rewritten two
  // tiles later, after the partner has passed the next tile's pair barrier)
  float* xm = xmax + (x.n & 1) * 256;
  xm[h * 128 + row] = tmax;
  named_bar_sync(xbar, 64);
  tmax = fmaxf(tmax, xm[(1 - h) * 128 + row]);
  const bool need = tmax > m + x.thresh || (m == -INFINITY && tmax != -INFINITY);
  float alpha = 1.f;
  if (need) {
    alpha = ex2((m - tmax) * x.c);                      // 0 when m = -inf
    m = tmax;
  }
  l *= alpha;
  const float mu = (m == -INFINITY) ? 0.f : m;
  const float2 c2 = make_float2(x.c, x.c);
  const float2 nb2 = make_float2(-mu * x.c, -mu * x.c);
  float2 rs[2] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
  uint32_t pre[NH > 0 ? NH : 1][16];
#pragma unroll
  for (int q = 0; q < NH; ++q) chunk_exp<kBF16>(r[q], c2, nb2, rs, pre[q]);
  if (x.n > 0) mbar_wait(x.pv_done, (x.n - 1) & 1);
  if (threadIdx.x == 0) tl_rec(*x.prm, x.n, 1);
  tc_fence_after();
  if (x.j > 0 && __any_sync(0xffffffffu, need && alpha != 1.f)) {
#pragma unroll 1
    for (int k = 0; k < kD / 32; ++k) {   // this half's kD / 2 columns of O
      uint32_t o[16];
      tmem_ld16(x.tl + kTO + h * (kD / 2) + k * 16, o);
      tmem_wait_ld();
#pragma unroll
      for (int i = 0; i < 16; ++i) o[i] = __float_as_uint(__uint_as_float(o[i]) * alpha);
      tmem_st16(x.tl + kTO + h * (kD / 2) + k * 16, o);
    }
  }
#pragma unroll
  for (int q = 0; q < NH; ++q) tmem_st16(x.tl + kTP + (2 * h + q) * 16, pre[q]);
  l += (rs[0].x + rs[0].y) + (rs[1].x + rs[1].y);
  tmem_wait_st();
  tc_fence_before();
  __syncwarp();
  if (lane == 0) {
    mbar_arrive(x.p_full);
    tl_rec(*x.prm, x.n, threadIdx.x == 0 ? 2 : 7 + ((threadIdx.x >> 5) & 3));
  }
}

}  // namespace

template <bool kBF16, int kMode, bool kPad, int kD>
__global__ void __launch_bounds__(WCfg<kD>::kThreads, DCfg<kD>::kMinBlocks)
    coarse_pp_kernel(const __grid_constant__ CUtensorMap tmq, const __grid_constant__ CUtensorMap tmk,
                     const __grid_constant__ CUtensorMap tmv, const __grid_constant__ CUtensorMap tmq2,
                     const __grid_constant__ CUtensorMap tmk2, const __grid_constant__ CUtensorMap tmv2,
                     const __grid_constant__ CUtensorMap tmo, const CoarseParams p) {
  // kMode: 0 = single plan, 1 = single plan with split dense-row items, 2 = batched plan, 3 = single
  // plan without CUDA-core CSR rows (no partial to merge). The mode paths are compiled only into
  // the instantiations that need them: their code costs the common path registers and time
  // (measured: 5% on C2 for the batched branches).
  constexpr bool kSplit = kMode == 1, kBatched = kMode == 2, kNoFine = kMode == 3;
  constexpr uint32_t kTileBytes = DCfg<kD>::kTileBytes, kTmemCols = DCfg<kD>::kTmemCols, kTO = DCfg<kD>::kTO;
  constexpr int kNSub = DCfg<kD>::kNSub;
  using W = WCfg<kD>;
  constexpr bool kCS = W::kCS;
  constexpr int kSoftWarps = W::kSoftWarps;
  constexpr int kRegsCtl = W::kRegsCtl, kRegsSoftmax = W::kRegsSoftmax;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t sbase = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const uint32_t sQ = sbase;
  const uint32_t sK = sQ + 2 * kTileBytes;
  const uint32_t sV = sK + kSt * kTileBytes;
  const uint32_t sMsk = sV + kSt * kTileBytes;            // [V stage] tile bitmasks
  Ctl* ctl = reinterpret_cast<Ctl*>(smem_raw + (sMsk + kSt * kMaskBytes - smem_u32(smem_raw)));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  auto bar = [&](const uint64_t& b) { return smem_u32(&b); };

  if (threadIdx.x == 0) {
    for (int b = 0; b < kItems; ++b) {
      mbar_init(bar(ctl->item_full[b]), 1);
      mbar_init(bar(ctl->item_empty[b]), 2 + kSoftWarps);   // producer + MMA thread + softmax warps
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(bar(ctl->q_full[b]), 1);
      mbar_init(bar(ctl->q_empty[b]), 1);
    }
    for (int s = 0; s < kSt; ++s) {
      mbar_init(bar(ctl->k_full[s]), 1);
      mbar_init(bar(ctl->k_empty[s]), 1);
      mbar_init(bar(ctl->v_full[s]), 1);
      mbar_init(bar(ctl->v_empty[s]), 1);
      mbar_init(bar(ctl->mk_full[s]), 1);
      mbar_init(bar(ctl->mk_empty[s]), kSoftWarps);
    }
    mbar_init(bar(ctl->s_full), 1);
    mbar_init(bar(ctl->s_free), kSoftWarps);
    mbar_init(bar(ctl->p_full), kSoftWarps);
    mbar_init(bar(ctl->pv_done), 1);
    fence_barrier_init();
  }
  if (warp == W::kWProd && lane == 0) {
    prefetch_tmap(&tmq);
    prefetch_tmap(&tmk);
    prefetch_tmap(&tmv);
    if (p.gather_tma) {
      prefetch_tmap(&tmq2);
      prefetch_tmap(&tmk2);
      prefetch_tmap(&tmv2);
    }
  }
  if (warp == W::kWMma) {
    tmem_alloc(smem_u32(&ctl->tmem_base), kTmemCols);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = ctl->tmem_base;

  if (warp == W::kWProd) {
    // ============================================================ producer
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
    const uint64_t pol_kv = policy_evict_last();   // K/V tiles are re-read by neighbouring items
    const uint64_t pol_q = policy_evict_first();   // Q tiles are read once
    uint32_t g = 0;
    for (uint32_t it = 0;; ++it) {
      const uint32_t slot = it % kItems;
      mbar_wait(bar(ctl->item_full[slot]), (it / kItems) & 1);
      const int u = ctl->slot[slot].u;
      const Item item = ctl->slot[slot].item;
      const int bh = ctl->slot[slot].bh;
      __syncwarp();
      if (lane == 0) {
        mbar_arrive(bar(ctl->item_empty[slot]));
        tl_item(p, it, 2);
      }
      if (u >= p.total_units) break;
      const int bb = bh / p.H, hh = bh % p.H;
      const uint32_t qs = it & 1;
      const uint32_t dQ = sQ + qs * kTileBytes;
      const uint32_t qf = bar(ctl->q_full[qs]);
      mbar_wait(bar(ctl->q_empty[qs]), ((it >> 1) & 1) ^ 1);
      if (item.kind == 0) {
        if (lane == 0) {
          mbar_arrive_expect_tx(qf, kTileBytes);
#pragma unroll
          for (int sb = 0; sb < kNSub; ++sb) tma_load_4d(dQ + sb * kSub, &tmq, qf, 64 * sb, item.rowA, hh, bb, pol_q);
        }
      } else if (p.gather_tma) {
        if (lane == 0) mbar_arrive_expect_tx(qf, kTileBytes);
        __syncwarp();
        const int4 ix = load_idx4(p.global_rows + item.rowA, 4 * lane, item.nrowsA);
#pragma unroll
        for (int sb = 0; sb < kNSub; ++sb)
          gather4(dQ + sb * kSub + lane * 512, &tmq2, qf, row_coords(ix, bb * p.rq.x + hh * p.rq.y + sb, p.rq.z),
                  pol_q);
      } else {
        gather_rows<kD>(dQ, p.q.data + bb * p.q.sb + hh * p.q.sh, p.q.sl, p.global_rows + item.rowA, item.nrowsA,
                        128, lane);
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(qf);
      }
      if (lane == 0) tl_item(p, it, 3);
      const int64_t krow0 = bb * p.rk.x + hh * p.rk.y, vrow0 = bb * p.rv.x + hh * p.rv.y;
      for (int j0 = 0; j0 < item.ntiles; j0 += 32) {
        // the item's tile references, 32 at a time (one per lane), broadcast per tile
        int4 mine = make_int4(0, 0, 0, -1);
        if (j0 + lane < item.ntiles) mine = __ldg(reinterpret_cast<const int4*>(p.trefs + item.tref_begin + j0 + lane));
        const int nj = min(32, item.ntiles - j0);
        if (j0 == 0 && __shfl_sync(0xffffffffu, mine.z, 0) >= 0 && lane == 0) tl_item(p, it, 4);
        for (int jj = 0; jj < nj; ++jj, ++g) {
          const int arg = __shfl_sync(0xffffffffu, mine.x, jj), kind = __shfl_sync(0xffffffffu, mine.y, jj);
          const int ncols = __shfl_sync(0xffffffffu, mine.z, jj), maskA = __shfl_sync(0xffffffffu, mine.w, jj);
          const uint32_t st = g % kSt, sph = ((g / kSt) & 1) ^ 1;
          const uint32_t dK = sK + st * kTileBytes, dV = sV + st * kTileBytes;
          // strip tiles: the column indices of this lane's 4 gathered rows
          int4 six = make_int4(-1, -1, -1, -1);
          if (kind != 0 && p.gather_tma) six = load_idx4(p.strip_cols + arg, 4 * lane, ncols);
          const uint32_t kf = bar(ctl->k_full[st]), vf = bar(ctl->v_full[st]);
          mbar_wait(bar(ctl->k_empty[st]), sph);
          if (lane == 0) {
            ctl->kcols[st] = ncols;   // published by the k_full arrive
            tl_rec(p, g, 5);
          }
          if (kind == 0) {
            if (lane == 0) {
              mbar_arrive_expect_tx(kf, kDbgNoLoads ? 0 : kTileBytes);
              if (!kDbgNoLoads) {
#pragma unroll
                for (int sb = 0; sb < kNSub; ++sb) tma_load_4d(dK + sb * kSub, &tmk, kf, 64 * sb, arg, hh, bb, pol_kv);
              }
            }
          } else if (p.gather_tma) {
            if (lane == 0) mbar_arrive_expect_tx(kf, ncols * 2 * kD);
            __syncwarp();
            if (4 * lane < ncols) {
#pragma unroll
              for (int sb = 0; sb < kNSub; ++sb)
                gather4(dK + sb * kSub + lane * 512, &tmk2, kf, row_coords(six, krow0 + sb, p.rk.z), pol_kv);
            }
          } else {
            gather_rows<kD>(dK, p.k.data + bb * p.k.sb + hh * p.k.sh, p.k.sl, p.strip_cols + arg, ncols, ncols, lane);
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(kf);
          }
          const uint32_t mbytes = maskA >= 0 ? kMaskBytes : 0;
          // the tile's descriptor / bitmask stage: with the V stage, or (late P.V) its own ring
          if (kLate) mbar_wait(bar(ctl->mk_empty[st]), sph);
          else mbar_wait(bar(ctl->v_empty[st]), sph);
          if (kPad) {
            // padding: the tile's columns below n_b (published with vdesc by the v_full arrive)
            const int nvalid = min(max(__ldg(p.valid_len + bb), 0), (int)p.L);
            uint32_t w[4];
            if (kind == 0) {
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                const int lim = nvalid - (arg + 32 * q);
                w[q] = lim >= 32 ? ~0u : (lim <= 0 ? 0u : (1u << lim) - 1u);
              }
            } else {
              const int4 cx = load_idx4(p.strip_cols + arg, 4 * lane, ncols);
              const uint32_t b0 = __ballot_sync(0xffffffffu, cx.x >= 0 && cx.x < nvalid);
              const uint32_t b1 = __ballot_sync(0xffffffffu, cx.y >= 0 && cx.y < nvalid);
              const uint32_t b2 = __ballot_sync(0xffffffffu, cx.z >= 0 && cx.z < nvalid);
              const uint32_t b3 = __ballot_sync(0xffffffffu, cx.w >= 0 && cx.w < nvalid);
              // column 32q + i is entry i % 4 of lane 8q + i / 4
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                uint32_t v = 0;
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                  const uint32_t bk = (i & 3) == 0 ? b0 : (i & 3) == 1 ? b1 : (i & 3) == 2 ? b2 : b3;
                  v |= ((bk >> (8 * q + (i >> 2))) & 1u) << i;
                }
                w[q] = v;
              }
            }
            if (lane == 0) {
#pragma unroll
              for (int q = 0; q < 4; ++q) ctl->cmask[st][q] = w[q];
            }
          }
          if (lane == 0) {
            ctl->vdesc[st] = make_int2(ncols, maskA);   // published by the v_full (mk_full) arrive
            tl_rec(p, g, 6);
          }
          const uint32_t vmb = kLate ? 0u : mbytes;     // mask bytes completing on the V barrier
          if (kLate) {
            const uint32_t mf = bar(ctl->mk_full[st]);
            if (lane == 0) {
              if (mbytes) {
                mbar_arrive_expect_tx(mf, mbytes);
                bulk_load(sMsk + st * kMaskBytes, p.masks + (size_t)maskA * 256, kMaskBytes, mf);
              } else {
                mbar_arrive(mf);
              }
            }
            mbar_wait(bar(ctl->v_empty[st]), sph);
          }
          if (kind == 0) {
            if (lane == 0) {
              mbar_arrive_expect_tx(vf, (kDbgNoLoads ? 0 : kTileBytes) + vmb);
              if (!kDbgNoLoads) {
#pragma unroll
                for (int sb = 0; sb < kNSub; ++sb) tma_load_4d(dV + sb * kSub, &tmv, vf, 64 * sb, arg, hh, bb, pol_kv);
              }
            }
          } else if (p.gather_tma) {
            if (lane == 0) mbar_arrive_expect_tx(vf, ncols * 2 * kD + vmb);
            __syncwarp();
            if (4 * lane < ncols) {
#pragma unroll
              for (int sb = 0; sb < kNSub; ++sb)
                gather4(dV + sb * kSub + lane * 512, &tmv2, vf, row_coords(six, vrow0 + sb, p.rv.z), pol_kv);
            }
          } else {
            gather_rows<kD>(dV, p.v.data + bb * p.v.sb + hh * p.v.sh, p.v.sl, p.strip_cols + arg, ncols, ncols, lane);
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive_expect_tx(vf, vmb);
          }
          if (!kLate && lane == 0 && mbytes) bulk_load(sMsk + st * kMaskBytes, p.masks + (size_t)maskA * 256, kMaskBytes, vf);
        }
      }
    }
  } else if (warp == W::kWSched) {
    // ============================================================ scheduler
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
    // Claims work items (dynamic counter) into a kItems-deep ring, i.e. up to kItems items ahead of
    // the slowest consumer, and warms L2 with each band item's Q tile.
    for (uint32_t it = 0;; ++it) {
      const uint32_t slot = it % kItems;
      int u = 0;
      if (lane == 0) {
        mbar_wait(bar(ctl->item_empty[slot]), ((it / kItems) & 1) ^ 1);
        tl_item(p, it, 0);
        u = atomicAdd(p.counter, 1);
        Slot sl;
        sl.u = u;
        if (u < p.total_units) {
          const UnitInfo ui = decode_unit(p, u);
          sl.item = p.items[ui.item];
          // batched plans: the unit's second index is the head, the sample comes with the item
          sl.bh = kBatched ? (int)sl.item.useB * p.H + ui.bh : ui.bh;
          if (sl.item.kind == 0) tma_prefetch_4d(&tmq, 0, sl.item.rowA, sl.bh % p.H, sl.bh / p.H);
        }
        ctl->slot[slot] = sl;
        mbar_arrive(bar(ctl->item_full[slot]));
        tl_item(p, it, 1);
      }
      u = __shfl_sync(0xffffffffu, u, 0);
      if (u >= p.total_units) break;
      __syncwarp();
    }
  } else if (warp == W::kWMma) {
    // ============================================================ MMA issuer (lane 0)
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
    if (lane == 0) {
      // Tile sequence n = 0, 1, ... over the CTA's lifetime. Iteration n issues S(n) (after the
      // softmax has read S(n-1)), then P.V(n-1) once its P is stored. P.V(n) of an item's first
      // tile overwrites O (accumulate = 0): its P is stored only after the softmax warps have
      // read the previous item's O in their epilogue, so no separate O barrier is needed.
      const uint32_t idesc_pv = idesc_f16(kBF16, 128, 64, false, true);
      uint32_t n = 0;
      struct Pend {
        uint32_t n, st;
        int ncols;
        bool first, valid, last;
      } pend{0, 0, 0, false, false, false};
      // late P.V: up to two pending P.V (tiles n-2, n-1 while S(n) is issued), in tile order
      Pend fifo[2];
      int nfifo = 0;
      auto issue_pv = [&](const Pend& e) {
        mbar_wait(bar(ctl->v_full[e.st]), (e.n / kSt) & 1);
        mbar_wait(bar(ctl->p_full), e.n & 1);
        tl_rec(p, e.n, 7);
        tc_fence_after();
        const uint32_t vA = sV + e.st * kTileBytes;
        // chunk c (16 keys): P at columns [kTP + 8c, kTP + 8c + 8) (packed pairs), V rows [16c, 16c + 16);
        // one N = 64 MMA per 64-column V sub-tile (O columns [kTO + 64 sb, kTO + 64 sb + 64))
#pragma unroll
        for (int sb = 0; sb < kNSub; ++sb)
          for (int c = 0; c < (kDbgNoMma ? 0 : e.ncols >> 4); ++c)
            mma_ts(tmem + kTO + 64 * sb, tmem + kTP + c * 8, smem_desc_sw128(vA + sb * kSub + c * 2048, 8192, 1024),
                   idesc_pv, (e.first && c == 0) ? 0u : 1u);
        tl_rec(p, e.n, 4);
        mma_commit(bar(ctl->pv_done));
        mma_commit(bar(ctl->v_empty[e.st]));
      };
      auto flush_fifo = [&]() {
        for (int i = 0; i < nfifo; ++i) issue_pv(fifo[i]);
        nfifo = 0;
      };
      for (uint32_t it = 0;; ++it) {
        const uint32_t slot = it % kItems;
        mbar_wait(bar(ctl->item_full[slot]), (it / kItems) & 1);
        const int u = ctl->slot[slot].u;
        const int ntiles = ctl->slot[slot].item.ntiles;
        mbar_arrive(bar(ctl->item_empty[slot]));
        tl_item(p, it, 6);
        if (u >= p.total_units) break;
        const uint32_t qs = it & 1;
        // finish the previous item first unless this item's Q tile is already resident
        if (kLatePV) {
          if (nfifo && !mbar_test_wait(bar(ctl->q_full[qs]), (it >> 1) & 1)) flush_fifo();
        } else if (pend.valid && !mbar_test_wait(bar(ctl->q_full[qs]), (it >> 1) & 1)) {
          issue_pv(pend);
          pend.valid = false;
        }
        mbar_wait(bar(ctl->q_full[qs]), (it >> 1) & 1);
        tl_item(p, it, 7);
        const uint32_t qa = sQ + qs * kTileBytes;
        for (int j = 0; j < ntiles; ++j, ++n) {
          const uint32_t st = n % kSt;
          mbar_wait(bar(ctl->k_full[st]), (n / kSt) & 1);
          tl_rec(p, n, 14);
          if (n == 0) tl_rec(p, 0, 15);
          const int ncols = ctl->kcols[st];
          if (n > 0) mbar_wait(bar(ctl->s_free), (n - 1) & 1);
          tc_fence_after();
          const uint32_t idesc_s = idesc_f16(kBF16, 128, ncols, false, false);
          const uint32_t kA = sK + st * kTileBytes;
#pragma unroll
          for (int kk = 0; kk < (kDbgNoMma ? 0 : kD / 16); ++kk) {
            const uint32_t ko = (kk >> 2) * kSub + (kk & 3) * 32;   // K step kk: sub-tile kk / 4, 32 B each
            mma_ss(tmem + kTS, smem_desc_sw128(qa + ko, 16, 1024), smem_desc_sw128(kA + ko, 16, 1024), idesc_s,
                   kk > 0);
          }
          mma_commit(bar(ctl->s_full));
          mma_commit(bar(ctl->k_empty[st]));
          // (q_empty is arrived by the softmax epilogue: the Q buffer also stages the item's O tile)
          tl_rec(p, n, 3);
          if (kLatePV) {
            // due now: P.V(k) for k <= n - 2, and P.V(n - 1) if it is its item's last tile
            int done = 0;
            while (done < nfifo && (fifo[done].n + 2 <= n || fifo[done].last)) issue_pv(fifo[done++]);
            for (int i = done; i < nfifo; ++i) fifo[i - done] = fifo[i];
            nfifo -= done;
            fifo[nfifo++] = Pend{n, st, ncols, j == 0, true, j == ntiles - 1};
          } else {
            if (pend.valid) issue_pv(pend);
            pend = Pend{n, st, ncols, j == 0, true, false};
          }
        }
      }
      if (kLatePV) flush_fifo();
      if (pend.valid) issue_pv(pend);
    }
    __syncwarp();
  } else if (warp == W::kWIdle) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
  } else {
    // ============================================================ softmax + epilogue
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(kRegsSoftmax) : "memory");
    // row of the Q tile = TMEM lane (warp w owns lane quarter w % 4); column split: half h = w / 4
    const int hh_cs = kCS ? warp >> 2 : 0;
    const int t = kCS ? (warp & 3) * 32 + lane + 128 * hh_cs : warp * 32 + lane;   // (> 127: half-1 warp)
    const int row = (warp & 3) * 32 + lane;
    const uint32_t tl = tmem + ((uint32_t)((warp & 3) * 32) << 16);
    const float c = p.scale_log2;
    // lazy rescaling (O accumulates in TMEM): the exponent keeps a stale row max m until a tile's
    // max exceeds it by more than 2^8 in probability, so p <= 256 and O rarely needs a rescale
    const float thresh = 8.f / c;
    uint32_t n = 0;
    for (uint32_t it = 0;; ++it) {
      const uint32_t slot = it % kItems;
      mbar_wait(bar(ctl->item_full[slot]), (it / kItems) & 1);
      const int u = ctl->slot[slot].u;
      const Item item = ctl->slot[slot].item;
      const int ubh = ctl->slot[slot].bh;
      __syncwarp();
      if (lane == 0) mbar_arrive(bar(ctl->item_empty[slot]));
      if (threadIdx.x == 0) tl_item(p, it, 5);
      if (u >= p.total_units) break;
      // epilogue metadata, loaded now so its latency hides behind the item's tiles
      int r_out = -1, slot_f = -1;
      if (t < item.nrowsA) {
        r_out = item.kind == 0 ? item.rowA + t : __ldg(p.global_rows + item.rowA + t);
        if (!kNoFine && item.kind == 0)
          slot_f = __ldg(p.fine_slot + (kBatched ? (int64_t)item.useB * p.L : 0) + item.rowA + t);
      }
      float m = -INFINITY, l = 0.f;
      // a lane quarter without a valid row (a gathered global-row item with <= 96 rows, e.g. C2's 32
      // global rows) does no softmax work: its S is not read and its P rows are left as they are
      // (P.V computes garbage O rows that are never stored, and the next item's first P.V
      // overwrites O). It still takes part in the per-tile barriers, in order (s_free(n), then
      // p_full(n) only after P.V(n-1): a p_full arrival may not run ahead into the next phase).
      const bool idle = kIdleQuarters && warp * 32 >= item.nrowsA;
      for (int j = 0; j < item.ntiles; ++j, ++n) {
        if (idle) {
          mbar_wait(bar(ctl->s_full), n & 1);
          __syncwarp();
          if (lane == 0) mbar_arrive(bar(ctl->s_free));
          if (n > 0) mbar_wait(bar(ctl->pv_done), (n - 1) & 1);
          __syncwarp();
          if (lane == 0) {
            mbar_arrive(bar(ctl->p_full));
            if (kLate) mbar_arrive(bar(ctl->mk_empty[n % kSt]));
          }
          continue;
        }
        const uint32_t st = n % kSt;
        mbar_wait(bar(ctl->s_full), n & 1);
        // the tile's descriptor and bitmask travel with its V stage (freed only after P.V(n)), or in
        // their own ring (late P.V)
        mbar_wait(bar(kLate ? ctl->mk_full[st] : ctl->v_full[st]), (n / kSt) & 1);
        tc_fence_after();
        const int2 desc = ctl->vdesc[st];                 // {ncols, maskA}
        const TileCtx tc{tl, sMsk + st * kMaskBytes + row * 16, desc.y >= 0, kPad ? ctl->cmask[st] : nullptr,
                         n, j, bar(ctl->s_free),
                         bar(ctl->pv_done), bar(ctl->p_full), c, thresh, &p, bar(ctl->s_full)};
        if (threadIdx.x == 0) tl_rec(p, n, 0);
        if constexpr (kCS) {
          // this warp's 32-column chunks of the tile: [2h, 2h + nh)
          const int nh = min(max((desc.x >> 5) - 2 * hh_cs, 0), 2);
          const uint32_t xbar = 2 + (warp & 3);
          float* xm = &ctl->xmax[0][0][0];
          switch (nh) {
            case 2: softmax_tile_cs<2, kBF16, kD>(tc, m, l, hh_cs, row, xbar, xm); break;
            case 1: softmax_tile_cs<1, kBF16, kD>(tc, m, l, hh_cs, row, xbar, xm); break;
            default: softmax_tile_cs<0, kBF16, kD>(tc, m, l, hh_cs, row, xbar, xm); break;
          }
        } else {
          switch (desc.x >> 5) {                          // 32-column chunks of the tile
            case 4: softmax_tile<4, kBF16, kD>(tc, m, l); break;
            case 3: softmax_tile<3, kBF16, kD>(tc, m, l); break;
            case 2: softmax_tile<2, kBF16, kD>(tc, m, l); break;
            default: softmax_tile<1, kBF16, kD>(tc, m, l); break;
          }
        }
        if (kLate) {   // this tile's descriptor / mask stage may be refilled
          __syncwarp();
          if (lane == 0) mbar_arrive(bar(ctl->mk_empty[st]));
        }
      }
      // ---------------------------------------------------------------- epilogue (a-8)
      if constexpr (kCS) {
        // column split: the row sum is the two halves' sums; the half-0 warps (0-3) run the epilogue
        if (hh_cs == 1) ctl->xsum[row] = l;
        named_bar_sync(2 + (warp & 3), 64);
        if (hh_cs == 1) continue;
        l += ctl->xsum[row];
      }
      // (d = 64 keeps its single-pass epilogue: the per-half form below measured 3% slower on C2)
      bool tma_out;
      if constexpr (kNSub == 1) {
        float mf = -INFINITY, lf = 0.f;
        const float4* accf = nullptr;
        const size_t fidx = (size_t)(kBatched ? ubh % p.H : ubh) * p.n_fine_rows + slot_f;
        if (slot_f >= 0 && !p.concurrent) {
          const float2 ml = p.part_ml[fidx];
          mf = ml.x;
          lf = ml.y;
          accf = reinterpret_cast<const float4*>(p.part_acc + fidx * 64);
        }
        if (threadIdx.x == 0) tl_rec(p, n - 1, 11);
        mbar_wait(bar(ctl->pv_done), (n - 1) & 1);          // the item's last P.V
        tc_fence_after();
        uint32_t o[2][32];
        tmem_ld32(tl + kTO, o[0]);
        tmem_ld32(tl + kTO + 32, o[1]);
        tmem_wait_ld();
        tc_fence_before();
        if (threadIdx.x == 0) tl_rec(p, n - 1, 12);
        bool skip = false;
        if (kSplit && item.kind == 1 && item.nrowsB > 1) {
          // split dense-row item: publish this chunk's (m, l, acc) per row; the chunk that finishes
          // its row group last merges all chunks by log-sum-exp and writes O (a-4 over column chunks)
          const size_t gidx = (size_t)ubh * p.n_dense_groups + item.rowB;
          float* part = p.dense_part + ((gidx * p.dense_nsplit + item.turns) * 128 + t) * 68;
          if (t < item.nrowsA) {
            float4* dst = reinterpret_cast<float4*>(part);
  #pragma unroll
            for (int i = 0; i < 16; ++i)
              __stcg(dst + i, make_float4(__uint_as_float(o[i >> 3][(i & 7) * 4]), __uint_as_float(o[i >> 3][(i & 7) * 4 + 1]),
                                          __uint_as_float(o[i >> 3][(i & 7) * 4 + 2]),
                                          __uint_as_float(o[i >> 3][(i & 7) * 4 + 3])));
            __stcg(reinterpret_cast<float2*>(part + 64), make_float2(m, l));
          }
          __threadfence();
          named_bar_sync(1, 128);
          // per-group chunk counter in [0, nrowsB): atomicInc wraps it back to 0 on the last chunk, so it
          // is ready for the next forward and never overflows
          if (threadIdx.x == 0)
            ctl->dense_last = atomicInc(reinterpret_cast<unsigned*>(p.dense_ctr) + gidx, (unsigned)item.nrowsB - 1u) ==
                              (unsigned)item.nrowsB - 1u;
          named_bar_sync(1, 128);
          skip = !ctl->dense_last;
          if (!skip && t < item.nrowsA) {
            __threadfence();
            const float* base = p.dense_part + (gidx * p.dense_nsplit * 128 + t) * 68;
            float mm = -INFINITY;
            for (int k = 0; k < item.nrowsB; ++k) mm = fmaxf(mm, __ldcg(base + (size_t)k * 128 * 68 + 64));
            const float mu0 = mm == -INFINITY ? 0.f : mm;
            // merged row accumulated in place of this chunk's O registers
  #pragma unroll
            for (int i = 0; i < 64; ++i) o[i >> 5][i & 31] = 0u;
            float den0 = 0.f;
            for (int k = 0; k < item.nrowsB; ++k) {
              const float* pk = base + (size_t)k * 128 * 68;
              const float2 ml = __ldcg(reinterpret_cast<const float2*>(pk + 64));
              const float a = ex2((ml.x - mu0) * c);
              den0 += ml.y * a;
              const float4* src = reinterpret_cast<const float4*>(pk);
  #pragma unroll
              for (int i = 0; i < 16; ++i) {
                const float4 v = __ldcg(src + i);
                uint32_t* q4 = &o[i >> 3][(i & 7) * 4];
                q4[0] = __float_as_uint(fmaf(v.x, a, __uint_as_float(q4[0])));
                q4[1] = __float_as_uint(fmaf(v.y, a, __uint_as_float(q4[1])));
                q4[2] = __float_as_uint(fmaf(v.z, a, __uint_as_float(q4[2])));
                q4[3] = __float_as_uint(fmaf(v.w, a, __uint_as_float(q4[3])));
              }
            }
            // hand the merged row to the common store below: O = o (scale 1), l = den0, m = mm
            m = mm;
            l = den0;
          }
        }
        if (slot_f >= 0 && p.concurrent) {
          // publish this row's coarse partial; the side that finishes the row second merges both
          float4* dst = reinterpret_cast<float4*>(p.part_c_acc + fidx * 64);
  #pragma unroll
          for (int i = 0; i < 16; ++i)
            __stcg(dst + i, make_float4(__uint_as_float(o[i >> 3][(i & 7) * 4]), __uint_as_float(o[i >> 3][(i & 7) * 4 + 1]),
                                        __uint_as_float(o[i >> 3][(i & 7) * 4 + 2]), __uint_as_float(o[i >> 3][(i & 7) * 4 + 3])));
          __stcg(p.part_c_ml + fidx, make_float2(m, l));
          __threadfence();
          const int old = atomicAdd(p.part_flags + fidx, 1);
          if (old & 1) {
            __threadfence();
            const float2 ml = __ldcg(p.part_ml + fidx);
            mf = ml.x;
            lf = ml.y;
            accf = reinterpret_cast<const float4*>(p.part_acc + fidx * 64);
          } else {
            skip = true;
          }
        }
        const float mt = fmaxf(m, mf);
        const float mu = mt == -INFINITY ? 0.f : mt;
        const float ac = ex2((m - mu) * c), af = ex2((mf - mu) * c);
        const float den = l * ac + lf * af;
        // normalised row -> 16-bit, 8 x 16-byte stores of this thread's row. A row with no valid
        // element in this item (a global row inside a band row block: it is owned by the dense-row
        // part, A5) is not written. (Staging the tile through shared memory for 4-rows-per-
        // instruction stores measured 10% slower: tools/experiments/.)
        // padding (A18): rows at or beyond the batch element's valid length are written as 0 by
        // every item that holds them (whatever the merge protocol decided)
        const bool pad_row = kPad && r_out >= 0 &&
                             r_out >= min(max(__ldg(p.valid_len + ubh / p.H), 0), (int)p.L);
        // (only blocks without global rows and without CUDA-core CSR rows: no other writer, no partial
        // to merge; measured: merging partials in this path costs C2 3% and gains nothing on C4)
        tma_out = !kPad && p.tma_store && item.kind == 0 && (item.useA & 3) == 3;   // uniform per item
        if (tma_out) {
          // normalised rows into the item's Q buffer (SWIZZLE_128B layout of the O tensor map), then one
          // TMA store of the 128 x 64 tile (rows beyond L are clipped by the map)
          const uint32_t sO = sQ + (it & 1) * kTileBytes;
          const float inv = (r_out >= 0 && mt != -INFINITY) ? __frcp_rn(den) : 0.f;
  #pragma unroll
          for (int h = 0; h < 2; ++h) {
  #pragma unroll
            for (int q8 = 0; q8 < 4; ++q8) {
              float a[8];
  #pragma unroll
              for (int i = 0; i < 8; ++i) a[i] = __uint_as_float(o[h][q8 * 8 + i]) * (ac * inv);
              const int ch = h * 4 + q8;
              asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(sO + t * 128 + ((ch ^ (t & 7)) << 4)),
                           "r"(pack2<kBF16>(a[0], a[1])), "r"(pack2<kBF16>(a[2], a[3])), "r"(pack2<kBF16>(a[4], a[5])),
                           "r"(pack2<kBF16>(a[6], a[7]))
                           : "memory");
            }
          }
          fence_proxy_async_smem();
#ifndef MG_DIAG_NO_EPI_BAR
          named_bar_sync(1, 128);
#endif
          if (threadIdx.x == 0) {
            tma_store_4d(&tmo, sO, 0, item.rowA, ubh % p.H, ubh / p.H);
            bulk_commit_group();
#ifndef MG_DIAG_NO_STORE_WAIT
            bulk_wait_group_read0();   // the buffer is reloaded with a later item's Q after q_empty
#endif
          }
        } else if (pad_row) {
          const int bb = ubh / p.H, hh = ubh % p.H;
          uint4* orow = reinterpret_cast<uint4*>(p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)r_out * p.o.sl);
  #pragma unroll
          for (int i = 0; i < 8; ++i) orow[i] = make_uint4(0u, 0u, 0u, 0u);
        } else if (r_out >= 0 && mt != -INFINITY && !skip) {
          const float inv = __frcp_rn(den);
          const int bb = ubh / p.H, hh = ubh % p.H;
          uint16_t* orow = p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)r_out * p.o.sl;
  #pragma unroll
          for (int h = 0; h < 2; ++h) {
  #pragma unroll
            for (int q8 = 0; q8 < 4; ++q8) {
              float a[8];
  #pragma unroll
              for (int i = 0; i < 8; ++i) a[i] = __uint_as_float(o[h][q8 * 8 + i]) * ac;
              if (accf) {
                const float4 f0 = __ldcg(accf + h * 8 + q8 * 2), f1 = __ldcg(accf + h * 8 + q8 * 2 + 1);
                a[0] = fmaf(f0.x, af, a[0]);
                a[1] = fmaf(f0.y, af, a[1]);
                a[2] = fmaf(f0.z, af, a[2]);
                a[3] = fmaf(f0.w, af, a[3]);
                a[4] = fmaf(f1.x, af, a[4]);
                a[5] = fmaf(f1.y, af, a[5]);
                a[6] = fmaf(f1.z, af, a[6]);
                a[7] = fmaf(f1.w, af, a[7]);
              }
              uint4 o4;
              o4.x = pack2<kBF16>(a[0] * inv, a[1] * inv);
              o4.y = pack2<kBF16>(a[2] * inv, a[3] * inv);
              o4.z = pack2<kBF16>(a[4] * inv, a[5] * inv);
              o4.w = pack2<kBF16>(a[6] * inv, a[7] * inv);
              *reinterpret_cast<uint4*>(orow + h * 32 + q8 * 8) = o4;
            }
          }
        }
      } else {
        // O is processed in kD / 64 halves of 64 columns (d = 64: one, read once up front)
        float mf = -INFINITY, lf = 0.f;
        const float4* accf = nullptr;
        const size_t fidx = (size_t)(kBatched ? ubh % p.H : ubh) * p.n_fine_rows + slot_f;
        if (slot_f >= 0 && !p.concurrent) {
          const float2 ml = p.part_ml[fidx];
          mf = ml.x;
          lf = ml.y;
          accf = reinterpret_cast<const float4*>(p.part_acc + fidx * kD);
        }
        if (threadIdx.x == 0) tl_rec(p, n - 1, 11);
        mbar_wait(bar(ctl->pv_done), (n - 1) & 1);          // the item's last P.V
        tc_fence_after();
        uint32_t o[2][32];
        auto load_o = [&](int sb) {
          tmem_ld32(tl + kTO + 64 * sb, o[0]);
          tmem_ld32(tl + kTO + 64 * sb + 32, o[1]);
          tmem_wait_ld();
        };
        if (kNSub == 1) load_o(0);
        if (threadIdx.x == 0) tl_rec(p, n - 1, 12);
        bool skip = false;
        // split dense-row item whose chunk finishes its group last: O is merged from the chunk partials
        bool merge_chunks = false;
        const float* chunk_base = nullptr;
        float mu0 = 0.f;
        constexpr int kPartStride = kD + 4;                 // acc[kD], m, l, pad (16-byte rows)
        if (kSplit && item.kind == 1 && item.nrowsB > 1) {
          // split dense-row item: publish this chunk's (m, l, acc) per row; the chunk that finishes
          // its row group last merges all chunks by log-sum-exp and writes O (a-4 over column chunks)
          const size_t gidx = (size_t)ubh * p.n_dense_groups + item.rowB;
          float* part = p.dense_part + ((gidx * p.dense_nsplit + item.turns) * 128 + t) * kPartStride;
          // (tcgen05.ld is warp-collective: every lane loads, only valid rows store)
  #pragma unroll
          for (int sb = 0; sb < kNSub; ++sb) {
            if (kNSub > 1) load_o(sb);
            if (t < item.nrowsA) {
              float4* dst = reinterpret_cast<float4*>(part + 64 * sb);
  #pragma unroll
              for (int i = 0; i < 16; ++i)
                __stcg(dst + i, make_float4(__uint_as_float(o[i >> 3][(i & 7) * 4]), __uint_as_float(o[i >> 3][(i & 7) * 4 + 1]),
                                            __uint_as_float(o[i >> 3][(i & 7) * 4 + 2]),
                                            __uint_as_float(o[i >> 3][(i & 7) * 4 + 3])));
            }
          }
          if (t < item.nrowsA) __stcg(reinterpret_cast<float2*>(part + kD), make_float2(m, l));
          __threadfence();
          named_bar_sync(1, 128);
          // per-group chunk counter in [0, nrowsB): atomicInc wraps it back to 0 on the last chunk, so it
          // is ready for the next forward and never overflows
          if (threadIdx.x == 0)
            ctl->dense_last = atomicInc(reinterpret_cast<unsigned*>(p.dense_ctr) + gidx, (unsigned)item.nrowsB - 1u) ==
                              (unsigned)item.nrowsB - 1u;
          named_bar_sync(1, 128);
          skip = !ctl->dense_last;
          if (!skip && t < item.nrowsA) {
            __threadfence();
            chunk_base = p.dense_part + (gidx * p.dense_nsplit * 128 + t) * kPartStride;
            float mm = -INFINITY;
            for (int k = 0; k < item.nrowsB; ++k) mm = fmaxf(mm, __ldcg(chunk_base + (size_t)k * 128 * kPartStride + kD));
            mu0 = mm == -INFINITY ? 0.f : mm;
            float den0 = 0.f;
            for (int k = 0; k < item.nrowsB; ++k)
              den0 += __ldcg(chunk_base + (size_t)k * 128 * kPartStride + kD + 1) *
                      ex2((__ldcg(chunk_base + (size_t)k * 128 * kPartStride + kD) - mu0) * c);
            // the merged row goes through the common store below: O = merged (scale 1), l = den0, m = mm
            merge_chunks = true;
            m = mm;
            l = den0;
          }
        }
        if (kNSub > 1 && p.concurrent) {
          // (tcgen05.ld is warp-collective: the d = 128 halves are loaded by every lane, stored below
          // by the rows with a CUDA-core CSR part)
  #pragma unroll
          for (int sb = 0; sb < kNSub; ++sb) {
            load_o(sb);
            if (slot_f >= 0) {
              float4* dst = reinterpret_cast<float4*>(p.part_c_acc + fidx * kD + 64 * sb);
  #pragma unroll
              for (int i = 0; i < 16; ++i)
                __stcg(dst + i, make_float4(__uint_as_float(o[i >> 3][(i & 7) * 4]), __uint_as_float(o[i >> 3][(i & 7) * 4 + 1]),
                                            __uint_as_float(o[i >> 3][(i & 7) * 4 + 2]), __uint_as_float(o[i >> 3][(i & 7) * 4 + 3])));
            }
          }
        }
        if (slot_f >= 0 && p.concurrent) {
          // publish this row's coarse partial; the side that finishes the row second merges both
          if (kNSub == 1) {
            float4* dst = reinterpret_cast<float4*>(p.part_c_acc + fidx * kD);
  #pragma unroll
            for (int i = 0; i < 16; ++i)
              __stcg(dst + i, make_float4(__uint_as_float(o[i >> 3][(i & 7) * 4]), __uint_as_float(o[i >> 3][(i & 7) * 4 + 1]),
                                          __uint_as_float(o[i >> 3][(i & 7) * 4 + 2]), __uint_as_float(o[i >> 3][(i & 7) * 4 + 3])));
          }
          __stcg(p.part_c_ml + fidx, make_float2(m, l));
          __threadfence();
          const int old = atomicAdd(p.part_flags + fidx, 1);
          if (old & 1) {
            __threadfence();
            const float2 ml = __ldcg(p.part_ml + fidx);
            mf = ml.x;
            lf = ml.y;
            accf = reinterpret_cast<const float4*>(p.part_acc + fidx * kD);
          } else {
            skip = true;
          }
        }
        const float mt = fmaxf(m, mf);
        const float mu = mt == -INFINITY ? 0.f : mt;
        const float ac = ex2((m - mu) * c), af = ex2((mf - mu) * c);
        const float den = l * ac + lf * af;
        // normalised row -> 16-bit, 8 x 16-byte stores per 64 columns of this thread's row. A row with
        // no valid element in this item (a global row inside a band row block: it is owned by the
        // dense-row part, A5) is not written. (Staging the tile through shared memory for 4-rows-per-
        // instruction stores measured 10% slower: tools/experiments/.)
        // padding (A18): rows at or beyond the batch element's valid length are written as 0 by
        // every item that holds them (whatever the merge protocol decided)
        const bool pad_row = kPad && r_out >= 0 &&
                             r_out >= min(max(__ldg(p.valid_len + ubh / p.H), 0), (int)p.L);
        // (only blocks without global rows and without CUDA-core CSR rows: no other writer, no partial
        // to merge; measured: merging partials in this path costs C2 3% and gains nothing on C4)
        tma_out = !kPad && p.tma_store && item.kind == 0 && (item.useA & 3) == 3;   // uniform per item
        const bool write_row = !tma_out && !pad_row && r_out >= 0 && mt != -INFINITY && !skip;
        const int bb = ubh / p.H, hh = ubh % p.H;
        uint16_t* orow = p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)max(r_out, 0) * p.o.sl;
        const uint32_t sO = sQ + (it & 1) * kTileBytes;
  #pragma unroll
        for (int sb = 0; sb < kNSub; ++sb) {
          if (kNSub > 1) load_o(sb);   // (warp-collective: every lane, before any per-row choice)
          if (merge_chunks) {
  #pragma unroll
            for (int i = 0; i < 64; ++i) o[i >> 5][i & 31] = 0u;
            for (int k = 0; k < item.nrowsB; ++k) {
              const float* pk = chunk_base + (size_t)k * 128 * kPartStride;
              const float a = ex2((__ldcg(pk + kD) - mu0) * c);
              const float4* src = reinterpret_cast<const float4*>(pk + 64 * sb);
  #pragma unroll
              for (int i = 0; i < 16; ++i) {
                const float4 v = __ldcg(src + i);
                uint32_t* q4 = &o[i >> 3][(i & 7) * 4];
                q4[0] = __float_as_uint(fmaf(v.x, a, __uint_as_float(q4[0])));
                q4[1] = __float_as_uint(fmaf(v.y, a, __uint_as_float(q4[1])));
                q4[2] = __float_as_uint(fmaf(v.z, a, __uint_as_float(q4[2])));
                q4[3] = __float_as_uint(fmaf(v.w, a, __uint_as_float(q4[3])));
              }
            }
          }
          if (tma_out) {
            // normalised rows into the item's Q buffer (SWIZZLE_128B layout of the O tensor map), then one
            // TMA store per 128 x 64 sub-tile (rows beyond L are clipped by the map)
            const float inv = (r_out >= 0 && mt != -INFINITY) ? __frcp_rn(den) : 0.f;
  #pragma unroll
            for (int h = 0; h < 2; ++h) {
  #pragma unroll
              for (int q8 = 0; q8 < 4; ++q8) {
                float a[8];
  #pragma unroll
                for (int i = 0; i < 8; ++i) a[i] = __uint_as_float(o[h][q8 * 8 + i]) * (ac * inv);
                const int ch = h * 4 + q8;
                asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(sO + sb * kSub + t * 128 + ((ch ^ (t & 7)) << 4)),
                             "r"(pack2<kBF16>(a[0], a[1])), "r"(pack2<kBF16>(a[2], a[3])), "r"(pack2<kBF16>(a[4], a[5])),
                             "r"(pack2<kBF16>(a[6], a[7]))
                             : "memory");
              }
            }
          } else if (pad_row) {
            uint4* o16 = reinterpret_cast<uint4*>(orow + 64 * sb);
  #pragma unroll
            for (int i = 0; i < 8; ++i) o16[i] = make_uint4(0u, 0u, 0u, 0u);
          } else if (write_row) {
            const float inv = __frcp_rn(den);
  #pragma unroll
            for (int h = 0; h < 2; ++h) {
  #pragma unroll
              for (int q8 = 0; q8 < 4; ++q8) {
                float a[8];
  #pragma unroll
                for (int i = 0; i < 8; ++i) a[i] = __uint_as_float(o[h][q8 * 8 + i]) * ac;
                if (accf) {
                  const float4 f0 = __ldcg(accf + 16 * sb + h * 8 + q8 * 2), f1 = __ldcg(accf + 16 * sb + h * 8 + q8 * 2 + 1);
                  a[0] = fmaf(f0.x, af, a[0]);
                  a[1] = fmaf(f0.y, af, a[1]);
                  a[2] = fmaf(f0.z, af, a[2]);
                  a[3] = fmaf(f0.w, af, a[3]);
                  a[4] = fmaf(f1.x, af, a[4]);
                  a[5] = fmaf(f1.y, af, a[5]);
                  a[6] = fmaf(f1.z, af, a[6]);
                  a[7] = fmaf(f1.w, af, a[7]);
                }
                uint4 o4;
                o4.x = pack2<kBF16>(a[0] * inv, a[1] * inv);
                o4.y = pack2<kBF16>(a[2] * inv, a[3] * inv);
                o4.z = pack2<kBF16>(a[4] * inv, a[5] * inv);
                o4.w = pack2<kBF16>(a[6] * inv, a[7] * inv);
                *reinterpret_cast<uint4*>(orow + 64 * sb + h * 32 + q8 * 8) = o4;
              }
            }
          }
        }
        if (tma_out) {
          fence_proxy_async_smem();
          named_bar_sync(1, 128);
          if (threadIdx.x == 0) {
  #pragma unroll
            for (int sb = 0; sb < kNSub; ++sb) tma_store_4d(&tmo, sO + sb * kSub, 64 * sb, item.rowA, hh, bb);
            bulk_commit_group();
#ifndef MG_DIAG_NO_STORE_WAIT
            bulk_wait_group_read0();   // the buffer is reloaded with a later item's Q after q_empty
#endif
          }
        }
        tc_fence_before();
      }
      // the item's Q buffer is free (its last S MMA has completed: pv_done above; its O tile, if
      // staged there, has been read by the TMA store)
      if (threadIdx.x == 0) {
        mbar_arrive(bar(ctl->q_empty[it & 1]));
        tl_rec(p, n - 1, 13);
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == W::kWMma) tmem_dealloc(tmem, kTmemCols);
  // the last CTA to finish resets the work counter for the next launch (every CTA's scheduler has
  // claimed its final, out-of-range unit before its CTA gets here), so no memset precedes a launch
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(p.counter + 1, 1) == (int)gridDim.x - 1) {
      atomicExch(p.counter, 0);
      atomicExch(p.counter + 1, 0);
    }
  }
}

cudaError_t launch_coarse_pp(const CoarseParams& p, const CUtensorMap& tmq, const CUtensorMap& tmk,
                             const CUtensorMap& tmv, const CUtensorMap& tmq2, const CUtensorMap& tmk2,
                             const CUtensorMap& tmv2, const CUtensorMap& tmo, bool bf16, bool split_dense, int grid,
                             cudaStream_t stream) {
  // the split-dense-item epilogue and the padding masks are compiled only into the instantiations
  // that need them (their code costs the common path registers)
  using K = void (*)(const CUtensorMap, const CUtensorMap, const CUtensorMap, const CUtensorMap, const CUtensorMap,
                     const CUtensorMap, const CUtensorMap, const CoarseParams);
#define MG_PP_ROW(D)                                                                                            \
  coarse_pp_kernel<false, 0, false, D>, coarse_pp_kernel<false, 0, true, D>, coarse_pp_kernel<false, 1, false, D>, \
      coarse_pp_kernel<false, 1, true, D>, coarse_pp_kernel<false, 2, false, D>, coarse_pp_kernel<false, 2, true, D>, \
      coarse_pp_kernel<false, 3, false, D>, coarse_pp_kernel<false, 3, true, D>, coarse_pp_kernel<true, 0, false, D>, \
      coarse_pp_kernel<true, 0, true, D>, coarse_pp_kernel<true, 1, false, D>, coarse_pp_kernel<true, 1, true, D>,    \
      coarse_pp_kernel<true, 2, false, D>, coarse_pp_kernel<true, 2, true, D>, coarse_pp_kernel<true, 3, false, D>,   \
      coarse_pp_kernel<true, 3, true, D>
  static const K table[32] = {MG_PP_ROW(64), MG_PP_ROW(128)};
#undef MG_PP_ROW
  if (p.d != 64 && p.d != 128) return cudaErrorInvalidValue;
  const int mode = p.batched ? 2 : (split_dense ? 1 : (p.n_fine_rows == 0 ? 3 : 0));
  const K kern = table[(p.d == 128 ? 16 : 0) + (bf16 ? 8 : 0) + 2 * mode + (p.valid_len ? 1 : 0)];
  const int smem = (int)(p.d == 128 ? smem_bytes<128>() : smem_bytes<64>());
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  const int threads = p.d == 128 ? WCfg<128>::kThreads : WCfg<64>::kThreads;
  kern<<<grid, threads, smem, stream>>>(tmq, tmk, tmv, tmq2, tmk2, tmv2, tmo, p);
  return cudaGetLastError();
}

// CTAs per SM of the persistent grid for head dimension d
int coarse_pp_ctas_per_sm(int d) { return d == 128 ? DCfg<128>::kMinBlocks : DCfg<64>::kMinBlocks; }

}  // namespace mg
