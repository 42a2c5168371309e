// Coarse-grained fused kernel for sm_100a. One work item = two 128-row Q tiles ("streams" A and
// B: two adjacent row blocks, or two groups of gathered global rows) of one (batch, head) and the
// union of their K/V tiles, each K/V tile loaded once and used by both streams:
//   SDDMM   S_X = Q_X K_j^T          tcgen05.mma (SS), S in TMEM          (§3.2)
//   scale + mask + online SpSoftmax  thread t of WG X owns row t of Q_X   (§3.3)
//   SpMM    O_X = P_X V_j            tcgen05.mma (TS: P from TMEM)       (§3.2)
// The per-row running (max, sum) is carried across the row's tiles instead of re-reading S
// (A14: the paper's 3-sweep SpSoftmax becomes an online softmax; same result).
//   kind 0 items: band row blocks with their BSR tiles (+ a gathered "strip" tile carrying the
//     blocks' CSR residual on the tensor cores); the epilogue merges the fp32 partial statistics
//     written by the CUDA-core fine kernel for any remaining CSR rows (compound SpSoftmax);
//   kind 1 items: gathered global rows against every column tile (dense-row part).
// Warp roles (one 384-thread CTA per SM, persistent, dynamic work counter):
//   warp 0      producer: work fetch, TMA of Q/K/V tiles (SWIZZLE_128B), bulk copies of tile
//               bitmasks, row gathers (global rows, strip columns)
//   warps 1, 3  MMA issuers for streams A and B (lane 0): S half tiles two ahead, P.V behind
//   warp 2      TMEM allocator, then scheduler: publishes work items, L2-prefetches their tiles
//   warps 4..7  softmax WG A, warps 8..11 softmax WG B: two independent streams, so one WG's
//               waits overlap the other's exp work (MUFU is the bound)
// TMEM (512 columns): per stream, three 64-column half-tile buffers (S_h, then P_h over it as
// 16-bit pairs) and a 64-column O accumulator. The pipeline unit is a half tile (64 keys): the MMA
// runs S two halves ahead; O accumulates in TMEM across the item (P.V with accumulate) with lazy
// rescaling by the softmax warps (FA4-style).
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "kernels.cuh"
#include "sm100_ptx.cuh"

namespace mg {

using namespace ptx;

namespace {

constexpr int kStages = 4;
constexpr int kThreads = 384;
constexpr uint32_t kTileBytes = 128 * 128;  // 128 rows x 64 x 16-bit
constexpr uint32_t kMaskBytes = 128 * 16;   // 128 rows x 2 x u64
// TMEM per stream w (256 columns at w*256): S [0,128), P (16-bit pairs) [128,192), O [192,256).
constexpr uint32_t kTmemPOff = 128, kTmemOOff = 192;

struct __align__(16) ItemSlot {
  Item item;
  int32_t u, bh, pad0, pad1;
};

// does stream w use tile j of the item (without touching the stage)
__device__ __forceinline__ bool item_uses(const Item& it, int w, int j) {
  if ((w == 0 ? it.nrowsA : it.nrowsB) == 0) return false;
  if (it.kind == 2) return (j & 1) == w;
  if (j >= 64) return true;
  return (((w == 0 ? it.useA : it.useB) >> j) & 1ull) != 0;
}

struct __align__(16) SmemCtl {
  TileRef tref[kStages];
  ItemSlot slot[2];
  uint64_t q_full[2], q_empty[2];
  uint64_t k_full[kStages], v_full[kStages], kv_empty[kStages];
  uint64_t s_full[2], s_free[2], p_full[2], pv_done[2];  // per stream
  uint64_t item_full[2], item_empty[2];
  uint32_t tmem_base;
};

constexpr size_t kSmemBytes =
    1024 + kTileBytes * (4 + 2 * kStages) + 2 * kMaskBytes * kStages + sizeof(SmemCtl);
static_assert(kSmemBytes <= 227 * 1024, "shared memory budget");
// setmaxnreg.inc draws from the CTA's pool (168 x 384 = 64512 registers at launch):
// 128 x kRegsCtl + 256 x kRegsSoftmax must not exceed it, or the inc blocks forever.
constexpr int kRegsCtl = 48, kRegsSoftmax = 224;
static_assert(128 * kRegsCtl + 256 * kRegsSoftmax <= 168 * 384, "register pool");

struct UnitInfo {
  int item, bh;
};

__device__ __forceinline__ UnitInfo decode_unit(const CoarseParams& p, int u) {
  const int dense_units = p.n_dense_items * p.BH;
  if (u < dense_units) return {u % p.n_dense_items, u / p.n_dense_items};
  const int v = u - dense_units;
  const int nband = p.n_items - p.n_dense_items;
  return {p.n_dense_items + v % nband, v / nband};
}

// Copy rows idx[0..nvalid) (idx < 0 -> zeros) of a [*, 64] 16-bit matrix into a K-major
// SWIZZLE_128B tile (row r at r*128 B, 16-byte chunk c at (c ^ (r & 7)) * 16); rows
// [nvalid, nfill) are zero-filled. Executed by one warp.
__device__ __forceinline__ void gather_rows(uint32_t dst, const uint16_t* base, int64_t sl, const int32_t* idx,
                                            int nvalid, int nfill, int lane) {
  for (int e = lane; e < nfill * 8; e += 32) {
    const int r = e >> 3, c = e & 7;
    int4 val = make_int4(0, 0, 0, 0);
    if (r < nvalid) {
      const int src = __ldg(idx + r);
      if (src >= 0) val = ld_nc_v4(base + (int64_t)src * sl + c * 8);
    }
    const uint32_t a = dst + r * 128 + ((c ^ (r & 7)) << 4);
    asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(val.x), "r"(val.y), "r"(val.z),
                 "r"(val.w)
                 : "memory");
  }
}

template <bool kBF16>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  return kBF16 ? pack_bf16(lo, hi) : pack_f16(lo, hi);
}

template <bool kBF16>
__device__ __forceinline__ void unpack2(uint32_t v, float& lo, float& hi) {
  if (kBF16) {
    lo = __uint_as_float(v << 16);
    hi = __uint_as_float(v & 0xffff0000u);
  } else {
    const float2 f = __half22float2(*reinterpret_cast<const __half2*>(&v));
    lo = f.x;
    hi = f.y;
  }
}

__device__ __forceinline__ int4 ld_shared_v4(uint32_t a) {
  int4 v;
  asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}

// One 16-column chunk of this thread's S row (r), validity bits in the low 16 bits of `bits`.
template <bool kMasked>
__device__ __forceinline__ void chunk_max(const uint32_t (&r)[16], uint32_t bits, float& mx0, float& mx1) {
#pragma unroll
  for (int i = 0; i < 16; i += 4) {
    float a[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) a[e] = (!kMasked || ((bits >> (i + e)) & 1u)) ? __uint_as_float(r[i + e]) : -INFINITY;
    mx0 = fmax3(mx0, a[0], a[1]);
    mx1 = fmax3(mx1, a[2], a[3]);
  }
}

template <bool kMasked, bool kBF16>
__device__ __forceinline__ void chunk_exp(const uint32_t (&r)[16], uint32_t bits, float2 c2, float2 nb2, float2& rs0,
                                          float2& rs1, uint32_t tP) {
  uint32_t pk[8];
#pragma unroll
  for (int i = 0; i < 16; i += 2) {
    const float s0 = (!kMasked || ((bits >> i) & 1u)) ? __uint_as_float(r[i]) : -INFINITY;
    const float s1 = (!kMasked || ((bits >> (i + 1)) & 1u)) ? __uint_as_float(r[i + 1]) : -INFINITY;
    const float2 x = __ffma2_rn(make_float2(s0, s1), c2, nb2);
    const float p0 = ex2(x.x), p1 = ex2(x.y);
    if (i & 2)
      rs1 = __fadd2_rn(rs1, make_float2(p0, p1));
    else
      rs0 = __fadd2_rn(rs0, make_float2(p0, p1));
    pk[i >> 1] = pack2<kBF16>(p0, p1);
  }
  tmem_st8(tP, pk);
}

__device__ __forceinline__ uint32_t chunk_bits16(uint64_t w0, uint64_t w1, int ch) {
  return (uint32_t)((ch < 4 ? w0 : w1) >> ((ch & 3) * 16)) & 0xffffu;
}

// Diagnostics: CTA 0 appends (clock64, role<<56 | event<<48 | arg) to its role's private segment
// of p.trace (4 segments of trace_cap/4 pairs; pair 0 of a segment holds the count). Plain
// stores only. Roles: 0 producer, 1 MMA, 2 softmax warp 4 (stream A), 3 softmax warp 8 (B).
struct Tracer {
  unsigned long long* seg = nullptr;
  uint32_t n = 0, cap = 0;
  __device__ __forceinline__ Tracer(const CoarseParams& p, uint32_t role) {
    if (p.trace != nullptr && blockIdx.x == 0) {
      cap = (uint32_t)(p.trace_cap / 4);
      seg = p.trace + 2ull * role * cap;
    }
  }
  __device__ __forceinline__ void operator()(uint32_t role, uint32_t ev, uint32_t arg) {
#ifndef MG_TRACE
    return;  // built without tracing: the hooks compile away
#endif
    if (seg == nullptr || n + 2 >= cap) return;
    ++n;
    seg[2 * n] = clock64();
    seg[2 * n + 1] = ((unsigned long long)role << 56) | ((unsigned long long)ev << 48) | arg;
    seg[0] = n;
  }
};

}  // namespace

template <bool kBF16>
__global__ void __launch_bounds__(kThreads, 1)
    coarse_kernel(const __grid_constant__ CUtensorMap tmq, const __grid_constant__ CUtensorMap tmk,
                  const __grid_constant__ CUtensorMap tmv, const CoarseParams p) {
  extern __shared__ uint8_t smem_raw[];
  // all shared-memory addresses are handled as 32-bit shared-window offsets
  const uint32_t sbase = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const uint32_t sQ = sbase;                              // [unit parity][stream] Q tiles
  const uint32_t sK = sQ + 4 * kTileBytes;
  const uint32_t sV = sK + kStages * kTileBytes;
  const uint32_t sM = sV + kStages * kTileBytes;           // [stage][stream] tile bitmasks
  SmemCtl* ctl = reinterpret_cast<SmemCtl*>(smem_raw + (sM + 2 * kStages * kMaskBytes - smem_u32(smem_raw)));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  auto bar = [&](const uint64_t& b) { return smem_u32(&b); };

  if (threadIdx.x == 0) {
    for (int b = 0; b < 2; ++b) {
      mbar_init(bar(ctl->q_full[b]), 1);
      mbar_init(bar(ctl->q_empty[b]), 2);           // one commit per MMA warp
      mbar_init(bar(ctl->s_full[b]), 1);
      mbar_init(bar(ctl->s_free[b]), 4);
      mbar_init(bar(ctl->p_full[b]), 4);
      mbar_init(bar(ctl->pv_done[b]), 1);
      mbar_init(bar(ctl->item_full[b]), 1);
      mbar_init(bar(ctl->item_empty[b]), 11);       // producer + 2 MMA warps + 8 softmax warps
    }
    for (int s = 0; s < kStages; ++s) {
      mbar_init(bar(ctl->k_full[s]), 1);
      mbar_init(bar(ctl->v_full[s]), 1);
      mbar_init(bar(ctl->kv_empty[s]), 2);          // one release per stream
    }
    fence_barrier_init();
  }
  if (warp == 2 && lane == 0) {
    prefetch_tmap(&tmq);
    prefetch_tmap(&tmk);
    prefetch_tmap(&tmv);
  }
  if (warp == 2) {
    tmem_alloc(smem_u32(&ctl->tmem_base), 512);
    tmem_relinquish();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = ctl->tmem_base;

  if (warp < 4) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
    if (warp == 0) {
      // ========================================================== producer
      Tracer trace(p, 0);
      const uint64_t pol_kv = policy_evict_last();   // K/V tiles are re-read by neighbouring items
      const uint64_t pol_q = policy_evict_first();   // Q tiles are read once
      uint32_t it = 0, g = 0, qi = 0;
      while (true) {
        const uint32_t slot = it & 1, ph = (it >> 1) & 1;
        mbar_wait(bar(ctl->item_full[slot]), ph);
        const int u = ctl->slot[slot].u;
        const Item item = ctl->slot[slot].item;
        const int bh = ctl->slot[slot].bh;
        __syncwarp();
        if (lane == 0) mbar_arrive(bar(ctl->item_empty[slot]));
        ++it;
        if (u >= p.total_units) break;
        const int bb = bh / p.H, hh = bh % p.H;
        if (lane == 0) trace(0, 1, u);
        const uint32_t qs = qi & 1;
        const uint32_t dQ = sQ + qs * 2 * kTileBytes;
        mbar_wait(bar(ctl->q_empty[qs]), ((qi >> 1) & 1) ^ 1);
        if (item.kind == 0) {
          if (lane == 0) {
            mbar_arrive_expect_tx(bar(ctl->q_full[qs]), item.nrowsB ? 2 * kTileBytes : kTileBytes);
            tma_load_4d(dQ, &tmq, bar(ctl->q_full[qs]), 0, item.rowA, hh, bb, pol_q);
            if (item.nrowsB) tma_load_4d(dQ + kTileBytes, &tmq, bar(ctl->q_full[qs]), 0, item.rowB, hh, bb, pol_q);
          }
        } else {
          const uint16_t* qsrc = p.q.data + bb * p.q.sb + hh * p.q.sh;
          gather_rows(dQ, qsrc, p.q.sl, p.global_rows + item.rowA, item.nrowsA, 128, lane);
          if (item.nrowsB && item.kind == 1)
            gather_rows(dQ + kTileBytes, qsrc, p.q.sl, p.global_rows + item.rowB, item.nrowsB, 128, lane);
          fence_proxy_async_smem();
          __syncwarp();
          if (lane == 0) mbar_arrive(bar(ctl->q_full[qs]));
        }
        ++qi;
        for (int j = 0; j < item.ntiles; ++j, ++g) {
          const TileRef tr = p.trefs[item.tref_begin + j];
          const uint32_t st = g % kStages, sph = (g / kStages) & 1;
          mbar_wait(bar(ctl->kv_empty[st]), sph ^ 1);
          if (lane == 0) trace(0, 3, g);
          const uint32_t dK = sK + st * kTileBytes, dV = sV + st * kTileBytes;
          const uint32_t dM = sM + st * 2 * kMaskBytes;
          const uint32_t mbytes = (tr.maskA >= 0 ? kMaskBytes : 0) + (tr.maskB >= 0 ? kMaskBytes : 0);
          if (lane == 0) ctl->tref[st] = tr;   // published by the k_full arrive below
          auto load_masks = [&]() {
            if (tr.maskA >= 0) bulk_load(dM, p.masks + (size_t)tr.maskA * 256, kMaskBytes, bar(ctl->k_full[st]));
            if (tr.maskB >= 0)
              bulk_load(dM + kMaskBytes, p.masks + (size_t)tr.maskB * 256, kMaskBytes, bar(ctl->k_full[st]));
          };
          if (p.debug_flags & 4) {
            if (lane == 0) {
              mbar_arrive(bar(ctl->k_full[st]));
              mbar_arrive(bar(ctl->v_full[st]));
            }
          } else if (tr.kind == 0) {
            if (lane == 0) {
              mbar_arrive_expect_tx(bar(ctl->k_full[st]), kTileBytes + mbytes);
              tma_load_4d(dK, &tmk, bar(ctl->k_full[st]), 0, tr.arg, hh, bb, pol_kv);
              load_masks();
              mbar_arrive_expect_tx(bar(ctl->v_full[st]), kTileBytes);
              tma_load_4d(dV, &tmv, bar(ctl->v_full[st]), 0, tr.arg, hh, bb, pol_kv);
            }
          } else {
            const int32_t* idx = p.strip_cols + tr.arg;
            gather_rows(dK, p.k.data + bb * p.k.sb + hh * p.k.sh, p.k.sl, idx, tr.ncols, tr.ncols, lane);
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) {
              mbar_arrive_expect_tx(bar(ctl->k_full[st]), mbytes);
              load_masks();
            }
            gather_rows(dV, p.v.data + bb * p.v.sb + hh * p.v.sh, p.v.sl, idx, tr.ncols, tr.ncols, lane);
            fence_proxy_async_smem();
            __syncwarp();
            if (lane == 0) mbar_arrive(bar(ctl->v_full[st]));
          }
        }
      }
    } else if (warp == 2) {
      // ========================================================== scheduler
      // Publishes work items in a 2-deep ring (dynamic counter) as soon as a slot frees, i.e. up
      // to two items ahead of the slowest consumer, and warms L2 with each item's Q and K/V tiles
      // (TMA prefetch, one lane per tile) so the producer's later TMA loads hit L2.
      Tracer trace(p, 0);
      uint32_t it = 0;
      while (true) {
        const uint32_t slot = it & 1, ph = (it >> 1) & 1;
        int u = 0;
        if (lane == 0) {
          trace(0, 4, it);
          mbar_wait(bar(ctl->item_empty[slot]), ph ^ 1);
          trace(0, 5, it);
          u = atomicAdd(p.counter, 1);
          ItemSlot is;
          is.u = u;
          if (u < p.total_units) {
            const UnitInfo ui = decode_unit(p, u);
            is.item = p.items[ui.item];
            is.bh = ui.bh;
          }
          ctl->slot[slot] = is;
          mbar_arrive(bar(ctl->item_full[slot]));
        }
        ++it;
        u = __shfl_sync(0xffffffffu, u, 0);
        if (u >= p.total_units) break;
        __syncwarp();
        const Item item = ctl->slot[slot].item;
        const int bh = ctl->slot[slot].bh;
        const int bb = bh / p.H, hh = bh % p.H;
        if (lane == 0 && item.kind == 0) {
          tma_prefetch_4d(&tmq, 0, item.rowA, hh, bb);
          if (item.nrowsB) tma_prefetch_4d(&tmq, 0, item.rowB, hh, bb);
        }
        for (int j = lane; j < item.ntiles; j += 32) {
          const TileRef tr = p.trefs[item.tref_begin + j];
          if (tr.kind == 0) {
            tma_prefetch_4d(&tmk, 0, tr.arg, hh, bb);
            tma_prefetch_4d(&tmv, 0, tr.arg, hh, bb);
          }
        }
      }
    } else if (warp == 1 || warp == 3) {
      // ========================================================== MMA issuers (one warp per stream)
      // Per used tile j of the stream: S_{next} = Q K_{next}^T (N = tile width) as soon as the
      // softmax has read S_j into registers, then O += P_j V_j once P_j is stored. Streams never
      // wait on each other; each releases a K/V stage after its own P.V of the tile (kv_empty
      // counts 2); tiles a stream skips are released once loaded. Lane 0 issues.
      const int w = warp == 3 ? 1 : 0;
      const bool leader = lane == 0;
      Tracer trace(p, 1);
      uint32_t it = 0, g = 0, qi = 0, nS = 0, nP = 0;   // S / P.V issued (CTA lifetime)
      const uint32_t tbase = tmem + w * 256;
      while (true) {
        const uint32_t slot = it & 1, ph = (it >> 1) & 1;
        mbar_wait(bar(ctl->item_full[slot]), ph);
        const int u = ctl->slot[slot].u;
        const Item item = ctl->slot[slot].item;
        __syncwarp();
        if (leader) mbar_arrive(bar(ctl->item_empty[slot]));
        ++it;
        if (u >= p.total_units) break;
        const uint32_t qs = qi & 1;
        const uint32_t qa = sQ + qs * 2 * kTileBytes + (item.kind == 2 ? 0 : w * kTileBytes);
        mbar_wait(bar(ctl->q_full[qs]), (qi >> 1) & 1);
        ++qi;
        const int nt = item.ntiles;
        int rel = 0;                                       // next tile whose stage is not yet released
        auto release_skipped = [&](int upto) {             // skipped tiles in [rel, upto)
          for (; rel < upto; ++rel) {
            if (item_uses(item, w, rel)) break;
            const uint32_t gs = g + rel;
            mbar_wait(bar(ctl->k_full[gs % kStages]), (gs / kStages) & 1);
            if (leader) mbar_arrive(bar(ctl->kv_empty[gs % kStages]));
            __syncwarp();
          }
        };
        auto next_used = [&](int from) {
          while (from < nt && !item_uses(item, w, from)) ++from;
          return from;
        };
        auto issue_s = [&](int j) {
          const uint32_t gg = g + j, st = gg % kStages;
          mbar_wait(bar(ctl->k_full[st]), (gg / kStages) & 1);
          const int ncols = ctl->tref[st].ncols;
          if (nS > 0) mbar_wait(bar(ctl->s_free[w]), (nS - 1) & 1);
          tc_fence_after();
          if (leader) {
            const uint32_t idesc_s = idesc_f16(kBF16, 128, ncols, false, false);
            const uint32_t kA = sK + st * kTileBytes;
#pragma unroll
            for (int kk = 0; kk < ((p.debug_flags & 2) ? 0 : 4); ++kk)
              mma_ss(tbase, smem_desc_sw128(qa + kk * 32, 16, 1024), smem_desc_sw128(kA + kk * 32, 16, 1024),
                     idesc_s, kk > 0);
            mma_commit(bar(ctl->s_full[w]));
          }
          __syncwarp();
          ++nS;
        };
        bool first_pv = true;
        auto issue_pv = [&](int j) {
          const uint32_t gg = g + j, st = gg % kStages;
          const int ncols = ctl->tref[st].ncols;
          mbar_wait(bar(ctl->v_full[st]), (gg / kStages) & 1);
          mbar_wait(bar(ctl->p_full[w]), nP & 1);
          tc_fence_after();
          if (leader) {
            const uint32_t idesc_pv = idesc_f16(kBF16, 128, 64, false, true);
            const uint32_t vA = sV + st * kTileBytes;
            for (int kk = 0; kk < ((p.debug_flags & 2) ? 0 : (ncols >> 4)); ++kk)
              mma_ts(tbase + kTmemOOff, tbase + kTmemPOff + kk * 8, smem_desc_sw128(vA + kk * 2048, 8192, 1024),
                     idesc_pv, (first_pv && kk == 0) ? 0u : 1u);
            mma_commit(bar(ctl->pv_done[w]));
            mma_commit(bar(ctl->kv_empty[st]));
          }
          __syncwarp();
          first_pv = false;
          ++nP;
        };
        int j = next_used(0);
        if (j < nt) {
          release_skipped(j);
          issue_s(j);
        }
        while (j < nt) {
          const int jn = next_used(j + 1);
          rel = j + 1;
          release_skipped(jn);                             // tiles this stream skips before jn
          if (jn < nt) {
            issue_s(jn);
          } else if (leader) {
            mma_commit(bar(ctl->q_empty[qs]));             // last S of the item issued
          }
          __syncwarp();
          issue_pv(j);
          j = jn;
        }
        if (next_used(0) >= nt) {                          // the stream has no tile in this item
          release_skipped(nt);
          if (leader) mma_commit(bar(ctl->q_empty[qs]));
          __syncwarp();
        }
        if (leader) trace(1, 2, g + nt - 1);
        g += nt;
      }
    }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(kRegsSoftmax) : "memory");
    // ============================================================ softmax + epilogue
    const int w = (warp - 4) >> 2;                         // stream: 0 = A, 1 = B
    const int q4 = warp & 3;                               // TMEM lane quarter
    const int t = q4 * 32 + lane;                          // row of the stream's Q tile = TMEM lane
    const uint32_t lane_base = (uint32_t)(q4 * 32) << 16;
    const uint32_t tbase = tmem + lane_base + w * 256;
    const uint32_t tP = tbase + kTmemPOff;
    const uint32_t tO = tbase + kTmemOOff;
    const float c = p.scale_log2;
    const float2 c2 = make_float2(c, c);
    Tracer trace(p, 2 + w);
    const bool tr_on = (warp == 4 || warp == 8) && lane == 0;
    const bool dry = (p.debug_flags & 1) != 0;
    // lazy rescaling (O accumulates in TMEM): the exponent uses a stale row max m until a half
    // tile's max exceeds it by more than 2^8 in probability, so p <= 256 and O rarely needs a rescale
    const float thresh = 8.f / c;
    uint32_t it = 0, g = 0, n = 0;                         // n: tiles processed by this stream
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      mbar_wait(bar(ctl->item_full[slot]), ph);
      const int u = ctl->slot[slot].u;
      const Item item = ctl->slot[slot].item;
      const int ubh = ctl->slot[slot].bh;
      __syncwarp();
      if (lane == 0) mbar_arrive(bar(ctl->item_empty[slot]));
      ++it;
      if (u >= p.total_units) break;
      const int nrows = w == 0 ? item.nrowsA : item.nrowsB;
      const bool active = q4 * 32 < nrows;                 // this warp has real rows
      // epilogue metadata, loaded now so its latency hides behind the item's tiles
      int r_out = -1, slot_f = -1;
      if (t < nrows) {
        const int rbase = w == 0 ? item.rowA : item.rowB;
        r_out = item.kind == 0 ? rbase + t : __ldg(p.global_rows + rbase + t);
        if (item.kind == 2 && w == 1) r_out = -1;          // stream B hands its partial to A
        if (item.kind == 0) slot_f = __ldg(p.fine_slot + rbase + t);
      }
      float m = -INFINITY, l = 0.f;
      uint32_t n_item = 0;
      for (int j = 0; j < item.ntiles && nrows > 0; ++j) {
        // a skipped tile's stage may already be recycled: decide from the item's use bitmap
        if (!item_uses(item, w, j)) continue;
        const uint32_t gg = g + j, st = gg % kStages;
        mbar_wait(bar(ctl->k_full[st]), (gg / kStages) & 1);   // tile descriptor + bitmask
        const TileRef tr = ctl->tref[st];
        const bool partial = (w == 0 ? tr.maskA : tr.maskB) >= 0;
        uint64_t w0 = ~0ull, w1 = ~0ull;
        if (partial && active) {
          const int4 mw = ld_shared_v4(sM + st * 2 * kMaskBytes + w * kMaskBytes + t * 16);
          w0 = ((uint64_t)(uint32_t)mw.y << 32) | (uint32_t)mw.x;
          w1 = ((uint64_t)(uint32_t)mw.w << 32) | (uint32_t)mw.z;
        }
        const int nh = tr.ncols > 64 ? 2 : 1;
        if (tr_on) trace(2 + w, 1, gg);
        mbar_wait(bar(ctl->s_full[w]), n & 1);
        if (tr_on) trace(2 + w, 2, gg);
        tc_fence_after();
        // S_j is read in two 64-column halves (four x16 loads in flight, one wait each); each half
        // runs max -> lazy rescale -> exp -> P store. The S buffer is released after the second
        // half's load so the MMA computes the next tile's S during this tile's exps.
        for (int hh = 0; hh < nh; ++hh) {
          const int nc = (tr.ncols - hh * 64 > 64 ? 64 : tr.ncols - hh * 64) >> 4;   // 16-col chunks
          const uint32_t tS = tbase + hh * 64;
          const uint64_t wd = hh ? w1 : w0;
          uint32_t r0[16], r1[16], r2[16], r3[16];
          if (active && !(p.debug_flags & 16)) {
            tmem_ld16(tS, r0);
            if (nc > 1) tmem_ld16(tS + 16, r1);
            if (nc > 2) tmem_ld16(tS + 32, r2);
            if (nc > 3) tmem_ld16(tS + 48, r3);
            tmem_wait_ld();
          }
          if (hh == nh - 1) {                              // S buffer free for the next tile
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(bar(ctl->s_free[w]));
          }
          float tmax = -INFINITY;
          if (active && !dry) {
            float mx0 = -INFINITY, mx1 = -INFINITY;
            if (partial) {
              chunk_max<true>(r0, (uint32_t)wd & 0xffffu, mx0, mx1);
              if (nc > 1) chunk_max<true>(r1, (uint32_t)(wd >> 16) & 0xffffu, mx0, mx1);
              if (nc > 2) chunk_max<true>(r2, (uint32_t)(wd >> 32) & 0xffffu, mx0, mx1);
              if (nc > 3) chunk_max<true>(r3, (uint32_t)(wd >> 48) & 0xffffu, mx0, mx1);
            } else {
              chunk_max<false>(r0, 0xffffu, mx0, mx1);
              if (nc > 1) chunk_max<false>(r1, 0xffffu, mx0, mx1);
              if (nc > 2) chunk_max<false>(r2, 0xffffu, mx0, mx1);
              if (nc > 3) chunk_max<false>(r3, 0xffffu, mx0, mx1);
            }
            tmax = fmaxf(mx0, mx1);
          }
          // lazy rescale decision (warp-uniform for the TMEM accesses)
          const bool need = tmax > m + thresh || (m == -INFINITY && tmax != -INFINITY);
          float alpha = 1.f;
          if (need) {
            alpha = ex2((m - tmax) * c);                   // 0 when m = -inf
            m = tmax;
          }
          l *= alpha;
          const bool any_rescale = __any_sync(0xffffffffu, need && alpha != 0.f);
          if (hh == 0 && n_item > 0 && !(p.debug_flags & 32)) {
            // previous P.V done: P may be overwritten, O holds the earlier tiles
            mbar_wait(bar(ctl->pv_done[w]), (n - 1) & 1);
            tc_fence_after();
          }
          if (any_rescale && active) {
            if (n_item > 0) {
#pragma unroll
              for (int h2 = 0; h2 < 4; ++h2) {
                uint32_t r[16];
                tmem_ld16(tO + h2 * 16, r);
                tmem_wait_ld();
#pragma unroll
                for (int i = 0; i < 16; ++i) r[i] = __float_as_uint(__uint_as_float(r[i]) * alpha);
                tmem_st16(tO + h2 * 16, r);
              }
            }
            if (hh == 1) {                                 // first half's P (32 packed columns)
              tmem_wait_st();
#pragma unroll
              for (int h2 = 0; h2 < 2; ++h2) {
                uint32_t r[16];
                tmem_ld16(tP + h2 * 16, r);
                tmem_wait_ld();
#pragma unroll
                for (int i = 0; i < 16; ++i) {
                  float lo, hi;
                  unpack2<kBF16>(r[i], lo, hi);
                  r[i] = pack2<kBF16>(lo * alpha, hi * alpha);
                }
                tmem_st16(tP + h2 * 16, r);
              }
            }
          }
          // p = 2^(s*c - m*c) (masked -> 0), packed to 16-bit pairs (A operand of P.V)
          if (active && !dry) {
            const float mu = (m == -INFINITY) ? 0.f : m;
            const float2 nb2 = make_float2(-mu * c, -mu * c);
            float2 rs0 = make_float2(0.f, 0.f), rs1 = make_float2(0.f, 0.f);
            const uint32_t pb = tP + hh * 32;
            if (partial) {
              chunk_exp<true, kBF16>(r0, (uint32_t)wd & 0xffffu, c2, nb2, rs0, rs1, pb);
              if (nc > 1) chunk_exp<true, kBF16>(r1, (uint32_t)(wd >> 16) & 0xffffu, c2, nb2, rs0, rs1, pb + 8);
              if (nc > 2) chunk_exp<true, kBF16>(r2, (uint32_t)(wd >> 32) & 0xffffu, c2, nb2, rs0, rs1, pb + 16);
              if (nc > 3) chunk_exp<true, kBF16>(r3, (uint32_t)(wd >> 48) & 0xffffu, c2, nb2, rs0, rs1, pb + 24);
            } else {
              chunk_exp<false, kBF16>(r0, 0xffffu, c2, nb2, rs0, rs1, pb);
              if (nc > 1) chunk_exp<false, kBF16>(r1, 0xffffu, c2, nb2, rs0, rs1, pb + 8);
              if (nc > 2) chunk_exp<false, kBF16>(r2, 0xffffu, c2, nb2, rs0, rs1, pb + 16);
              if (nc > 3) chunk_exp<false, kBF16>(r3, 0xffffu, c2, nb2, rs0, rs1, pb + 24);
            }
            l += (rs0.x + rs0.y) + (rs1.x + rs1.y);
          }
        }
        if (active) tmem_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(bar(ctl->p_full[w]));
        if (tr_on) trace(2 + w, 3, gg);
        ++n;
        ++n_item;
      }
      g += item.ntiles;
      if (n_item == 0) continue;                           // stream unused in this item
      // the item's last P.V: O is complete in TMEM
      mbar_wait(bar(ctl->pv_done[w]), (n - 1) & 1);
      tc_fence_after();
      float oacc[64];
      if (active) {
#pragma unroll
        for (int h2 = 0; h2 < 4; ++h2) {
          uint32_t r[16];
          tmem_ld16(tO + h2 * 16, r);
#pragma unroll
          for (int i = 0; i < 16; ++i) oacc[h2 * 16 + i] = __uint_as_float(r[i]);
        }
        tmem_wait_ld();
      }
      tc_fence_before();
      if (tr_on) trace(2 + w, 5, g - 1);
      if (item.kind == 2) {
        // split dense item: B's partial (m, l, O) rows -> per-CTA scratch -> A merges (LSE)
        float* xr = p.dense_xch + ((size_t)blockIdx.x * 128 + t) * 68;
        if (w == 1) {
          if (active) {
            *reinterpret_cast<float2*>(xr) = make_float2(m, l);
#pragma unroll
            for (int i = 0; i < 64; i += 4)
              *reinterpret_cast<float4*>(xr + 4 + i) = make_float4(oacc[i], oacc[i + 1], oacc[i + 2], oacc[i + 3]);
          }
          __threadfence_block();
          asm volatile("bar.arrive 9, 256;" ::: "memory");
        } else {
          named_bar_sync(9, 256);
          if (active) {
            const float2 mlb = *reinterpret_cast<const float2*>(xr);
            const float mt = fmaxf(m, mlb.x);
            const float mu2 = mt == -INFINITY ? 0.f : mt;
            const float aa = ex2((m - mu2) * c), ab = ex2((mlb.x - mu2) * c);
            l = l * aa + mlb.y * ab;
#pragma unroll
            for (int i = 0; i < 64; i += 4) {
              const float4 ob = *reinterpret_cast<const float4*>(xr + 4 + i);
              oacc[i] = oacc[i] * aa + ob.x * ab;
              oacc[i + 1] = oacc[i + 1] * aa + ob.y * ab;
              oacc[i + 2] = oacc[i + 2] * aa + ob.z * ab;
              oacc[i + 3] = oacc[i + 3] * aa + ob.w * ab;
            }
            m = mt;
          }
        }
      }

      // ---- epilogue: merge the fine partial (if any), normalise, store the row's 64 outputs
      if (r_out >= 0) {
        const int r = r_out;
        float mf = -INFINITY, lf = 0.f;
        const float* accf = nullptr;
        {
          if (slot_f >= 0) {
            const size_t idx = (size_t)ubh * p.n_fine_rows + slot_f;
            const float2 ml = p.part_ml[idx];
            mf = ml.x;
            lf = ml.y;
            accf = p.part_acc + idx * 64;
          }
        }
        const float mt = fmaxf(m, mf);
        if (mt != -INFINITY) {
          const float as = ex2((m - mt) * c), af = ex2((mf - mt) * c);
          const float inv = 1.f / (l * as + lf * af);
          const int bb = ubh / p.H, hh = ubh % p.H;
          uint16_t* orow = p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)r * p.o.sl;
#pragma unroll
          for (int q8 = 0; q8 < 8; ++q8) {
            float v[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) v[e] = oacc[q8 * 8 + e] * as;
            if (accf) {
              const float4 f0 = reinterpret_cast<const float4*>(accf)[q8 * 2];
              const float4 f1 = reinterpret_cast<const float4*>(accf)[q8 * 2 + 1];
              v[0] = fmaf(f0.x, af, v[0]); v[1] = fmaf(f0.y, af, v[1]);
              v[2] = fmaf(f0.z, af, v[2]); v[3] = fmaf(f0.w, af, v[3]);
              v[4] = fmaf(f1.x, af, v[4]); v[5] = fmaf(f1.y, af, v[5]);
              v[6] = fmaf(f1.z, af, v[6]); v[7] = fmaf(f1.w, af, v[7]);
            }
            uint4 o4;
            o4.x = pack2<kBF16>(v[0] * inv, v[1] * inv);
            o4.y = pack2<kBF16>(v[2] * inv, v[3] * inv);
            o4.z = pack2<kBF16>(v[4] * inv, v[5] * inv);
            o4.w = pack2<kBF16>(v[6] * inv, v[7] * inv);
            *reinterpret_cast<uint4*>(orow + q8 * 8) = o4;
          }
        }
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 2) tmem_dealloc(tmem, 512);
}

cudaError_t launch_coarse(const CoarseParams& p, const CUtensorMap& tmq, const CUtensorMap& tmk,
                          const CUtensorMap& tmv, bool bf16, int grid, cudaStream_t stream) {
  auto kern = bf16 ? coarse_kernel<true> : coarse_kernel<false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemBytes);
  if (e != cudaSuccess) return e;
  kern<<<grid, kThreads, kSmemBytes, stream>>>(tmq, tmk, tmv, p);
  return cudaGetLastError();
}

}  // namespace mg
