// Coarse-grained fused kernel for sm_100a. One work item = one 128-row Q tile (a band row block,
// or up to 128 gathered global rows) of one (batch, head) and its list of K/V tiles:
//   SDDMM   S = Q K_j^T            tcgen05.mma (SS), S in TMEM            (§3.2)
//   scale + mask + online SpSoftmax  thread t owns row t of Q            (§3.3)
//   SpMM    O = P V_j              tcgen05.mma (TS: P from TMEM)         (§3.2)
// The per-row running (max, sum) is carried across the row's tiles instead of re-reading S
// (A14: the paper's 3-sweep SpSoftmax becomes an online softmax; same result).
//   kind 0 items: a band row block with its BSR tiles (+ a gathered "strip" tile carrying the
//     block's CSR residual on the tensor cores); the epilogue merges the fp32 partial statistics
//     written by the CUDA-core fine kernel for any remaining CSR rows (compound SpSoftmax);
//   kind 1 items: gathered global rows against every column tile (dense-row part).
// Column-group softmax: the 16-column chunks of every tile are dealt round-robin to four column
// groups (group cg owns chunks cg and cg + 4). 16 softmax warps = 4 groups x 4 TMEM lane quarters;
// each warp runs an independent online softmax over its group's columns for its 32 rows, with its
// own O accumulator in TMEM (O_cg = sum_j P_j,cg V_j,cg). The four partial rows (m, l, O_cg) are
// merged once per item in the epilogue. Four warps per SMSP hide each other's latencies; MUFU ex2
// throughput is the bound.
// P aliasing: a warp writes its packed P (16-bit pairs) over the S columns it has just read, and
// P.V(n) reads it from there. tcgen05.mma ops issued by one thread execute in order, so S(n+2),
// issued after P.V(n), cannot overwrite the buffer before P.V(n) has read it: no "S free" barrier.
// Warp roles (one 640-thread CTA per SM, persistent, dynamic work counter):
//   warp 0      producer: TMA of Q/K/V tiles (SWIZZLE_128B), bulk copies of tile bitmasks,
//               row gathers (global rows, strip columns)
//   warp 1      MMA issuer (lane 0): S(n), then P.V(n-1) of all groups
//   warp 2      TMEM allocator, then scheduler: publishes work items, L2-prefetches their tiles
//   warp 3      gatherer: row gathers (global-row Q tiles, strip K/V tiles) posted by the
//               producer through a job ring, so gathers never stall the TMA stream
//   warps 4..19 softmax: column group cg = (warp - 4) / 4, TMEM lane quarter = warp % 4
// TMEM (512 columns): S/P[b] at b*128 (b = tile parity), O_cg at 256 + cg*64.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "kernels.cuh"
#include "sm100_ptx.cuh"

namespace mg {

using namespace ptx;

namespace {

#ifndef MG_GROUPS
#define MG_GROUPS 4
#endif
// Column groups per tile (2 or 4): 4 * kGroups softmax warps; group cg owns the 16-column
// chunks c = cg, cg + kGroups, ... of every tile. TMEM holds kSbuf S/P buffers (128 columns each)
// and one 64-column O accumulator per group: 2 groups -> 3 buffers, 4 groups -> 2 buffers.
constexpr int kGroups = MG_GROUPS;
static_assert(kGroups == 2 || kGroups == 4, "column groups");
constexpr int kChunks = 8 / kGroups;          // chunks per group of a 128-column tile
constexpr int kSbuf = kGroups == 2 ? 3 : 2;   // S/P buffers
constexpr int kLag = kSbuf - 1;               // tiles the MMA issuer runs S ahead of P.V
constexpr int kStages = 5;
constexpr int kThreads = 128 + 128 * kGroups;
constexpr uint32_t kTileBytes = 128 * 128;  // 128 rows x 64 x 16-bit
constexpr uint32_t kMaskBytes = 128 * 16;   // 128 rows x 2 x u64
constexpr uint32_t kTmemO = 128 * kSbuf;
static_assert(kTmemO + 64 * kGroups <= 512, "TMEM columns");

struct __align__(16) ItemSlot {
  Item item;
  int32_t u, bh, pad0, pad1;
};

// A gather job for the gatherer warp: kind 0 = strip K/V tile into stage `dst`, 1 = Q rows into
// Q buffer `dst`, 2 = stop.
struct __align__(16) GatherJob {
  const uint16_t* kbase;
  const uint16_t* vbase;
  const int32_t* idx;
  int32_t kind, dst, nvalid, nfill, mask, pad;
};
constexpr int kJobs = 4;

struct __align__(16) SmemCtl {
  GatherJob job[kJobs];
  uint64_t job_full[kJobs], job_empty[kJobs];
  TileRef tref[kStages];
  ItemSlot slot[2];
  float2 xch[2][kGroups][128];               // [item parity][group][row] (m, l) for the merge
  uint64_t q_full[2], q_empty[2];
  uint64_t kv_full[kStages], kv_empty[kStages];
  uint64_t s_full[kSbuf], p_full[kSbuf], pv_done[kSbuf];  // per S/P buffer
  uint64_t o_free;
  uint64_t item_full[2], item_empty[2];
  uint32_t tmem_base;
};

constexpr size_t kSmemBytes = 1024 + kTileBytes * (2 + 2 * kStages) + kMaskBytes * kStages + sizeof(SmemCtl);
static_assert(kSmemBytes <= 227 * 1024, "shared memory budget");
// setmaxnreg.inc draws from the CTA's pool (launch registers x kThreads): 128 x kRegsCtl +
// (kThreads - 128) x kRegsSoftmax must not exceed it, or the inc blocks forever.
constexpr int kRegsLaunch = (65536 / kThreads) & ~7;
constexpr int kRegsCtl = 56, kRegsSoftmax = kGroups == 2 ? 224 : 104;
static_assert(128 * kRegsCtl + (kThreads - 128) * kRegsSoftmax <= kRegsLaunch * kThreads, "register pool");

struct UnitInfo {
  int item, bh;
};

// dense units first (long items start early), then band units
__device__ __forceinline__ UnitInfo decode_unit(const CoarseParams& p, int u) {
  const int dense_units = p.n_dense_items * p.BH;
  if (u < dense_units) return {u % p.n_dense_items, u / p.n_dense_items};
  const int v = u - dense_units;
  const int nband = p.n_items - p.n_dense_items;
  return {p.n_dense_items + v % nband, v / nband};
}

// Copy rows idx[0..nvalid) (idx < 0 -> zeros) of a [*, 64] 16-bit matrix into a K-major
// SWIZZLE_128B tile (row r at r*128 B, 16-byte chunk c at (c ^ (r & 7)) * 16); rows
// [nvalid, nfill) are zero-filled. Executed by one warp; each lane keeps kBatch 16-byte loads in
// flight before storing them (the loads are independent, so one memory latency per batch).
__device__ __forceinline__ void gather_rows(uint32_t dst, const uint16_t* base, int64_t sl, const int32_t* idx,
                                            int nvalid, int nfill, int lane) {
  constexpr int kBatch = 4;
  const int total = nfill * 8;
  for (int e0 = 0; e0 < total; e0 += 32 * kBatch) {
    int4 val[kBatch];
#pragma unroll
    for (int k = 0; k < kBatch; ++k) {
      const int e = e0 + k * 32 + lane, r = e >> 3;
      val[k] = make_int4(0, 0, 0, 0);
      if (e < total && r < nvalid) {
        const int src = __ldg(idx + r);
        if (src >= 0) val[k] = ld_nc_v4(base + (int64_t)src * sl + (e & 7) * 8);
      }
    }
#pragma unroll
    for (int k = 0; k < kBatch; ++k) {
      const int e = e0 + k * 32 + lane, r = e >> 3;
      if (e < total) {
        const uint32_t a = dst + r * 128 + (((e & 7) ^ (r & 7)) << 4);
        asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(val[k].x), "r"(val[k].y),
                     "r"(val[k].z), "r"(val[k].w)
                     : "memory");
      }
    }
  }
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

// Diagnostics (MG_TRACE builds only; compiled away otherwise): one lane of selected warps keeps
// per-phase cycle counters in registers -- mark(k) charges the cycles since the previous mark to
// phase k -- and adds them to p.trace[role * 16 + k] (summed over CTAs) at exit. No memory
// traffic while the kernel runs, so the timeline is not perturbed. Roles: 0 producer, 1 MMA,
// 2 softmax warp 4 (half 0), 3 softmax warp 8 (half 1).
struct Prof {
#ifdef MG_TRACE
  uint32_t acc[12];
  long long last;
  bool on;
  __device__ __forceinline__ explicit Prof(bool on_) : on(on_) {
#pragma unroll
    for (int k = 0; k < 12; ++k) acc[k] = 0;
    last = clock64();
  }
  __device__ __forceinline__ void mark(int k) {
    if (!on) return;
    const long long now = clock64();
    acc[k] += (uint32_t)(now - last);
    last = now;
  }
  __device__ __forceinline__ void flush(const CoarseParams& p, int role) {
    if (!on || p.trace == nullptr) return;
#pragma unroll
    for (int k = 0; k < 12; ++k) atomicAdd(p.trace + role * 16 + k, (unsigned long long)acc[k]);
    atomicAdd(p.trace + role * 16 + 15, 1ull);
  }
#else
  __device__ __forceinline__ explicit Prof(bool) {}
  __device__ __forceinline__ void mark(int) {}
  __device__ __forceinline__ void flush(const CoarseParams&, int) {}
#endif
};

// Diagnostics (MG_TIMELINE builds only): per-item event clocks (low 32 bits of clock64) of every
// CTA, 16 fields per item, written by single lanes to p.trace (as uint32, after 256 uint64s):
// 0 softmax item start, 1 first S ready, 2 last P stored, 3/4 epilogue start/end, 5 MMA Q ready,
// 6 MMA first S issued, 7 MMA first P.V issued, 8 epilogue after (m, l) exchange, 9 epilogue
// after last-P.V wait, 10 epilogue after O read. tools/timeline_coarse.py reads it.
__device__ __forceinline__ void tl_rec(const CoarseParams& p, uint32_t idx, int field) {
#ifdef MG_TIMELINE
  if (p.trace == nullptr || idx >= 64 || p.trace_cap < 256 + 8 * 64 * (int)gridDim.x) return;
  reinterpret_cast<uint32_t*>(p.trace + 256)[(blockIdx.x * 64 + idx) * 16 + field] = (uint32_t)clock64();
#endif
}

}  // namespace

template <bool kBF16>
__global__ void __launch_bounds__(kThreads, 1)
    coarse_kernel(const __grid_constant__ CUtensorMap tmq, const __grid_constant__ CUtensorMap tmk,
                  const __grid_constant__ CUtensorMap tmv, const CoarseParams p) {
  extern __shared__ uint8_t smem_raw[];
  // all shared-memory addresses are handled as 32-bit shared-window offsets
  const uint32_t sbase = (smem_u32(smem_raw) + 1023u) & ~1023u;
  const uint32_t sQ = sbase;                              // [item parity] Q tiles
  const uint32_t sK = sQ + 2 * kTileBytes;
  const uint32_t sV = sK + kStages * kTileBytes;
  const uint32_t sM = sV + kStages * kTileBytes;           // [stage] tile bitmasks
  SmemCtl* ctl = reinterpret_cast<SmemCtl*>(smem_raw + (sM + kStages * kMaskBytes - smem_u32(smem_raw)));
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  auto bar = [&](const uint64_t& b) { return smem_u32(&b); };

  if (threadIdx.x == 0) {
    for (int b = 0; b < 2; ++b) {
      mbar_init(bar(ctl->q_full[b]), 1);
      mbar_init(bar(ctl->q_empty[b]), 1);
      mbar_init(bar(ctl->item_full[b]), 1);
      mbar_init(bar(ctl->item_empty[b]), 2 + 4 * kGroups);   // producer + MMA + softmax warps
    }
    for (int b = 0; b < kSbuf; ++b) {
      mbar_init(bar(ctl->s_full[b]), 1);
      mbar_init(bar(ctl->p_full[b]), 4 * kGroups);  // every softmax warp stored its P
      mbar_init(bar(ctl->pv_done[b]), 1);
    }
    mbar_init(bar(ctl->o_free), 4 * kGroups);
    for (int j = 0; j < kJobs; ++j) {
      mbar_init(bar(ctl->job_full[j]), 1);
      mbar_init(bar(ctl->job_empty[j]), 1);
    }
    for (int s = 0; s < kStages; ++s) {
      mbar_init(bar(ctl->kv_full[s]), 1);
      mbar_init(bar(ctl->kv_empty[s]), 1);
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

  if (warp == 0) {
    // ============================================================ producer
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
    Prof prof(lane == 0 && blockIdx.x < 148);
    const uint64_t pol_kv = policy_evict_last();   // K/V tiles are re-read by neighbouring items
    const uint64_t pol_q = policy_evict_first();   // Q tiles are read once
    uint32_t it = 0, g = 0, jc = 0;
    auto post = [&](const GatherJob& jb) {             // hand a gather to the gatherer warp
      if (lane == 0) {
        const uint32_t js = jc % kJobs;
        mbar_wait(bar(ctl->job_empty[js]), ((jc / kJobs) & 1) ^ 1);
        ctl->job[js] = jb;
        mbar_arrive(bar(ctl->job_full[js]));
      }
      __syncwarp();
      ++jc;
    };
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      mbar_wait(bar(ctl->item_full[slot]), ph);
      const int u = ctl->slot[slot].u;
      const Item item = ctl->slot[slot].item;
      const int bh = ctl->slot[slot].bh;
      __syncwarp();
      if (lane == 0) mbar_arrive(bar(ctl->item_empty[slot]));
      if (u >= p.total_units) break;
      const int bb = bh / p.H, hh = bh % p.H;
      prof.mark(0);
      const uint32_t qs = it & 1;
      const uint32_t dQ = sQ + qs * kTileBytes;
      mbar_wait(bar(ctl->q_empty[qs]), ph ^ 1);
      prof.mark(1);
      if (item.kind == 0) {
        if (lane == 0) {
          mbar_arrive_expect_tx(bar(ctl->q_full[qs]), kTileBytes);
          tma_load_4d(dQ, &tmq, bar(ctl->q_full[qs]), 0, item.rowA, hh, bb, pol_q);
        }
      } else {
        post(GatherJob{p.q.data + bb * p.q.sb + hh * p.q.sh, nullptr, p.global_rows + item.rowA, 1, (int32_t)qs,
                       item.nrowsA, 128, -1, 0});
      }
      prof.mark(2);
      ++it;
      for (int j = 0; j < item.ntiles; ++j, ++g) {
        const TileRef tr = p.trefs[item.tref_begin + j];
        const uint32_t st = g % kStages, sph = (g / kStages) & 1;
        mbar_wait(bar(ctl->kv_empty[st]), sph ^ 1);
        prof.mark(3);
        const uint32_t dK = sK + st * kTileBytes, dV = sV + st * kTileBytes;
        const uint32_t dM = sM + st * kMaskBytes;
        const uint32_t mbytes = tr.maskA >= 0 ? kMaskBytes : 0;
        if (lane == 0) ctl->tref[st] = tr;   // published by the kv_full arrive below
        const uint32_t kvf = bar(ctl->kv_full[st]);
        if (p.debug_flags & 4) {
          if (lane == 0) mbar_arrive(kvf);
        } else if (tr.kind == 0) {
          if (lane == 0) {
            mbar_arrive_expect_tx(kvf, 2 * kTileBytes + mbytes);
            tma_load_4d(dK, &tmk, kvf, 0, tr.arg, hh, bb, pol_kv);
            tma_load_4d(dV, &tmv, kvf, 0, tr.arg, hh, bb, pol_kv);
            if (mbytes) bulk_load(dM, p.masks + (size_t)tr.maskA * 256, kMaskBytes, kvf);
          }
        } else {
          post(GatherJob{p.k.data + bb * p.k.sb + hh * p.k.sh, p.v.data + bb * p.v.sb + hh * p.v.sh,
                         p.strip_cols + tr.arg, 0, (int32_t)st, tr.ncols, tr.ncols, tr.maskA, 0});
        }
        prof.mark(tr.kind == 0 ? 4 : 5);
      }
    }
    post(GatherJob{nullptr, nullptr, nullptr, 2, 0, 0, 0, -1, 0});
    prof.flush(p, 0);
  } else if (warp == 2) {
    // ============================================================ scheduler
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
    // Publishes work items in a 2-deep ring (dynamic counter) as soon as a slot frees, i.e. up
    // to two items ahead of the slowest consumer, and warms L2 with each item's Q and K/V tiles
    // (TMA prefetch, one lane per tile) so the producer's later TMA loads hit L2.
    uint32_t it = 0;
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      int u = 0;
      if (lane == 0) {
        mbar_wait(bar(ctl->item_empty[slot]), ph ^ 1);
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
      if (lane == 0 && item.kind == 0) tma_prefetch_4d(&tmq, 0, item.rowA, hh, bb);
      for (int j = lane; j < item.ntiles; j += 32) {
        const TileRef tr = p.trefs[item.tref_begin + j];
        if (tr.kind == 0) {
          tma_prefetch_4d(&tmk, 0, tr.arg, hh, bb);
          tma_prefetch_4d(&tmv, 0, tr.arg, hh, bb);
        }
      }
    }
  } else if (warp == 1) {
    // ============================================================ MMA issuer (lane 0)
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
    // Tile sequence over the CTA's lifetime: n = 0, 1, 2, ...; S(n) -> S/P[n % kSbuf]. Iteration n
    // issues S(n), then P.V(n - kLag) once every softmax warp stored that tile's P. S(n) reuses
    // the buffer of tile n - kSbuf, whose P.V this thread issued earlier (in-order execution).
    // The first P.V of an item (accumulate = 0) also waits until the previous item's epilogue has
    // read O (o_free).
    const bool leader = lane == 0;
    Prof prof(leader && blockIdx.x < 148);
    uint32_t it = 0, g = 0, n = 0, items_done = 0;
    struct Pend {
      uint32_t st, n;
      int ncols;
      bool first, valid;
    };
    Pend q[kLag];                                      // pending P.V, oldest first
#pragma unroll
    for (int i = 0; i < kLag; ++i) q[i].valid = false;
    auto issue_pv = [&](const Pend& e) {
      const uint32_t b = e.n % kSbuf, st = e.st;
      if (e.first) {
        if (items_done > 0 && !(p.debug_flags & 64)) mbar_wait(bar(ctl->o_free), (items_done - 1) & 1);
        if (leader) tl_rec(p, items_done, 7);
        ++items_done;
      }
      prof.mark(5);
      mbar_wait(bar(ctl->p_full[b]), (e.n / kSbuf) & 1);
      prof.mark(6);
      tc_fence_after();
      if (leader && !(p.debug_flags & 2)) {
        const uint32_t vA = sV + st * kTileBytes;
        const uint32_t idesc_pv = idesc_f16(kBF16, 128, 64, false, true);
        // chunk c (16 keys): P at S/P[b] columns [16c, 16c + 8) (packed), V rows [16c, 16c + 16);
        // group c % kGroups accumulates into its O; the first chunk of a group in an item
        // overwrites (the item's first tile has all groups: tiles are >= 2 * kGroups chunks wide
        // except strips, which come last)
        for (int c = 0; c < (e.ncols >> 4); ++c) {
          const int cg = c % kGroups;
          mma_ts(tmem + kTmemO + cg * 64, tmem + b * 128 + c * 16, smem_desc_sw128(vA + c * 2048, 8192, 1024),
                 idesc_pv, (e.first && c < kGroups) ? 0u : 1u);
        }
      }
      if (leader) {
        mma_commit(bar(ctl->pv_done[b]));
        mma_commit(bar(ctl->kv_empty[st]));
      }
      __syncwarp();
      prof.mark(7);
    };
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      mbar_wait(bar(ctl->item_full[slot]), ph);
      const int u = ctl->slot[slot].u;
      const int ntiles = ctl->slot[slot].item.ntiles;
      __syncwarp();
      if (leader) mbar_arrive(bar(ctl->item_empty[slot]));
      if (u >= p.total_units) break;
      prof.mark(0);
      const uint32_t qs = it & 1;
      const uint32_t qa = sQ + qs * kTileBytes;
      mbar_wait(bar(ctl->q_full[qs]), ph);
      prof.mark(1);
      if (leader) tl_rec(p, it, 5);
      ++it;
      for (int j = 0; j < ntiles; ++j, ++g, ++n) {
        const uint32_t st = g % kStages, b = n % kSbuf;
        mbar_wait(bar(ctl->kv_full[st]), (g / kStages) & 1);
        prof.mark(2);
        const int ncols = ctl->tref[st].ncols;
        tc_fence_after();
        if (leader) {
          const uint32_t idesc_s = idesc_f16(kBF16, 128, ncols, false, false);
          const uint32_t kA = sK + st * kTileBytes;
#pragma unroll
          for (int kk = 0; kk < ((p.debug_flags & 2) ? 0 : 4); ++kk)
            mma_ss(tmem + b * 128, smem_desc_sw128(qa + kk * 32, 16, 1024), smem_desc_sw128(kA + kk * 32, 16, 1024),
                   idesc_s, kk > 0);
          mma_commit(bar(ctl->s_full[b]));
          if (j == ntiles - 1) mma_commit(bar(ctl->q_empty[qs]));   // last S of the item
        }
        __syncwarp();
        prof.mark(4);
        if (leader && j == 0) tl_rec(p, it - 1, 6);
        if (q[0].valid) issue_pv(q[0]);               // P.V of tile n - kLag
#pragma unroll
        for (int i = 0; i + 1 < kLag; ++i) q[i] = q[i + 1];
        q[kLag - 1] = Pend{st, n, ncols, j == 0, true};
      }
    }
#pragma unroll
    for (int i = 0; i < kLag; ++i)
      if (q[i].valid) issue_pv(q[i]);
    prof.flush(p, 1);
  } else if (warp == 3) {
    // ============================================================ gatherer
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kRegsCtl) : "memory");
    for (uint32_t jc = 0;; ++jc) {
      const uint32_t js = jc % kJobs;
      mbar_wait(bar(ctl->job_full[js]), (jc / kJobs) & 1);
      const GatherJob jb = ctl->job[js];
      __syncwarp();
      if (lane == 0) mbar_arrive(bar(ctl->job_empty[js]));
      if (jb.kind == 2) break;
      if (jb.kind == 0) {                                  // strip K/V tile (+ its bitmask)
        gather_rows(sK + jb.dst * kTileBytes, jb.kbase, p.k.sl, jb.idx, jb.nvalid, jb.nfill, lane);
        gather_rows(sV + jb.dst * kTileBytes, jb.vbase, p.v.sl, jb.idx, jb.nvalid, jb.nfill, lane);
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          const uint32_t kvf = bar(ctl->kv_full[jb.dst]);
          mbar_arrive_expect_tx(kvf, jb.mask >= 0 ? kMaskBytes : 0);
          if (jb.mask >= 0) bulk_load(sM + jb.dst * kMaskBytes, p.masks + (size_t)jb.mask * 256, kMaskBytes, kvf);
        }
      } else {                                             // gathered global-row Q tile
        gather_rows(sQ + jb.dst * kTileBytes, jb.kbase, p.q.sl, jb.idx, jb.nvalid, jb.nfill, lane);
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(bar(ctl->q_full[jb.dst]));
      }
    }
  } else {
    // ============================================================ softmax + epilogue
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(kRegsSoftmax) : "memory");
    const int cg = (warp - 4) >> 2;                        // column group: chunks cg + kGroups*i
    const int q4 = warp & 3;                               // TMEM lane quarter
    const int t = q4 * 32 + lane;                          // row of the Q tile = TMEM lane
    const uint32_t tl = tmem + ((uint32_t)(q4 * 32) << 16);
    const float c = p.scale_log2;
    const float2 c2 = make_float2(c, c);
    Prof prof((warp == 4 || warp == 8) && lane == 0 && blockIdx.x < 148);
    const bool dry = (p.debug_flags & 1) != 0;
    // lazy rescaling (O accumulates in TMEM): the exponent uses a stale row max m until a tile's
    // max exceeds it by more than 2^8 in probability, so p <= 256 and O rarely needs a rescale
    const float thresh = 8.f / c;
    constexpr int W = 64 / kGroups;                        // output columns written per warp

    // An item's epilogue runs after the NEXT item's first tile, by which time the item's last P.V
    // (issued by the MMA warp after the next item's first S) has normally completed; the next
    // item's first P.V (accumulate = 0) waits for it through o_free.
    struct Epi {
      float m, l;
      int r_out, slot_f, ubh;
      uint32_t n_last, ipar, idx;
      bool active, valid;
    };
    Epi pend{0.f, 0.f, -1, -1, 0, 0, 0, 0, false, false};
    const bool tlw = warp == 4 && lane == 0;
    auto epilogue = [&](const Epi& e) {
      if (tlw) tl_rec(p, e.idx, 3);
      // the groups' partial rows are merged; warp (cg, q4) writes output columns [W*cg, W*cg + W)
      // of its rows from every group's O (same TMEM lane), plus the fine partial if any. (m, l)
      // are final after the item's last tile: exchange them first, so that the only wait between
      // the item's last P.V and o_free is the O read itself.
      ctl->xch[e.ipar][cg][t] = make_float2(e.m, e.l);
      named_bar_sync(1 + q4, 32 * kGroups);                // (m, l) of the row's groups visible
      float mg[kGroups], lg[kGroups];
#pragma unroll
      for (int k = 0; k < kGroups; ++k) {
        const float2 v = ctl->xch[e.ipar][k][t];
        mg[k] = v.x;
        lg[k] = v.y;
      }
      float mf = -INFINITY, lf = 0.f;
      const float* accf = nullptr;
      if (e.slot_f >= 0) {
        const size_t idx = (size_t)e.ubh * p.n_fine_rows + e.slot_f;
        const float2 ml = p.part_ml[idx];
        mf = ml.x;
        lf = ml.y;
        accf = p.part_acc + idx * 64 + cg * W;
      }
      float mt = mf;
#pragma unroll
      for (int k = 0; k < kGroups; ++k) mt = fmaxf(mt, mg[k]);
      const float mu = mt == -INFINITY ? 0.f : mt;
      float a[kGroups], den = 0.f;
#pragma unroll
      for (int k = 0; k < kGroups; ++k) {
        a[k] = ex2((mg[k] - mu) * c);                      // 0 for a group with no valid column
        den += lg[k] * a[k];
      }
      const float af = ex2((mf - mu) * c);
      den += lf * af;
      prof.mark(9);
      if (tlw) tl_rec(p, e.idx, 8);
      mbar_wait(bar(ctl->pv_done[e.n_last % kSbuf]), (e.n_last / kSbuf) & 1);   // the item's last P.V
      tc_fence_after();
      if (tlw) tl_rec(p, e.idx, 9);
      float acc[W];
#pragma unroll
      for (int i = 0; i < W; ++i) acc[i] = 0.f;
      if (e.active) {
#pragma unroll
        for (int k = 0; k < kGroups; ++k) {
#pragma unroll
          for (int s16 = 0; s16 < W / 16; ++s16) {
            uint32_t o[16];
            tmem_ld16(tl + kTmemO + k * 64 + cg * W + s16 * 16, o);
            tmem_wait_ld();
#pragma unroll
            for (int i = 0; i < 16; ++i) acc[s16 * 16 + i] = fmaf(__uint_as_float(o[i]), a[k], acc[s16 * 16 + i]);
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(bar(ctl->o_free));        // O may be overwritten by the next item
      prof.mark(10);
      if (tlw) tl_rec(p, e.idx, 10);
      if (e.r_out >= 0 && mt != -INFINITY) {
        if (accf) {
#pragma unroll
          for (int q = 0; q < W / 4; ++q) {
            const float4 f = reinterpret_cast<const float4*>(accf)[q];
            acc[4 * q] = fmaf(f.x, af, acc[4 * q]);
            acc[4 * q + 1] = fmaf(f.y, af, acc[4 * q + 1]);
            acc[4 * q + 2] = fmaf(f.z, af, acc[4 * q + 2]);
            acc[4 * q + 3] = fmaf(f.w, af, acc[4 * q + 3]);
          }
        }
        const float inv = __frcp_rn(den);
        const int bb = e.ubh / p.H, hh = e.ubh % p.H;
        uint16_t* orow = p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)e.r_out * p.o.sl + cg * W;
#pragma unroll
        for (int q8 = 0; q8 < W / 8; ++q8) {
          uint4 o4;
          o4.x = pack2<kBF16>(acc[q8 * 8 + 0] * inv, acc[q8 * 8 + 1] * inv);
          o4.y = pack2<kBF16>(acc[q8 * 8 + 2] * inv, acc[q8 * 8 + 3] * inv);
          o4.z = pack2<kBF16>(acc[q8 * 8 + 4] * inv, acc[q8 * 8 + 5] * inv);
          o4.w = pack2<kBF16>(acc[q8 * 8 + 6] * inv, acc[q8 * 8 + 7] * inv);
          *reinterpret_cast<uint4*>(orow + q8 * 8) = o4;
        }
      }
      prof.mark(11);
      if (tlw) tl_rec(p, e.idx, 4);
    };

    uint32_t it = 0, g = 0, n = 0;                         // n: tiles processed (CTA lifetime)
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      mbar_wait(bar(ctl->item_full[slot]), ph);
      const int u = ctl->slot[slot].u;
      const int ntiles = ctl->slot[slot].item.ntiles;
      const int kind = ctl->slot[slot].item.kind;
      const int row0 = ctl->slot[slot].item.rowA;
      const int nrows = ctl->slot[slot].item.nrowsA;
      const int ubh = ctl->slot[slot].bh;
      __syncwarp();
      if (lane == 0) mbar_arrive(bar(ctl->item_empty[slot]));
      if (u >= p.total_units) break;
      const uint32_t ipar = it & 1;
      ++it;
      const bool active = q4 * 32 < nrows;                 // this warp has real rows
      // epilogue metadata, loaded now so its latency hides behind the item's tiles
      int r_out = -1, slot_f = -1;
      if (t < nrows) {
        r_out = kind == 0 ? row0 + t : __ldg(p.global_rows + row0 + t);
        if (kind == 0) slot_f = __ldg(p.fine_slot + row0 + t);
      }
      prof.mark(0);
      if (tlw) tl_rec(p, it - 1, 0);
      float m = -INFINITY, l = 0.f;
      for (int j = 0; j < ntiles; ++j, ++g, ++n) {
        const uint32_t st = g % kStages, b = n % kSbuf;
        // S(n) complete implies (tcgen05.commit tracks all earlier tcgen05 ops of the MMA thread)
        // that the MMA warp had observed kv_full for this stage: tile descriptor and bitmask landed
        mbar_wait(bar(ctl->s_full[b]), (n / kSbuf) & 1);
        prof.mark(2);
        if (tlw && j == 0) tl_rec(p, it - 1, 1);
        tc_fence_after();
        const int4 tri = ld_shared_v4(smem_u32(&ctl->tref[st]));   // {arg, kind, ncols, maskA}
        const int4 mw = ld_shared_v4(sM + st * kMaskBytes + t * 16);
        const int nchunk = tri.z >> 4;                     // 16-column chunks of the tile: 2..8
        const bool partial = tri.w >= 0;
        const uint32_t tSb = tl + b * 128 + cg * 16;       // this group's first chunk
        bool has[kChunks];
#pragma unroll
        for (int i = 0; i < kChunks; ++i) has[i] = cg + kGroups * i < nchunk;
        uint32_t r[kChunks][16];
        const bool ld = active && has[0] && !(p.debug_flags & 16);
        if (ld) {
#pragma unroll
          for (int i = 0; i < kChunks; ++i)
            if (has[i]) tmem_ld16(tSb + kGroups * 16 * i, r[i]);
        }
        // validity bits of the group's chunks
        uint32_t mk[kChunks];
#pragma unroll
        for (int i = 0; i < kChunks; ++i) {
          const int ch = cg + kGroups * i;
          const uint32_t word = (uint32_t)((ch & 4) ? (ch & 2 ? mw.w : mw.z) : (ch & 2 ? mw.y : mw.x));
          mk[i] = partial ? (word >> (16 * (ch & 1))) & 0xffffu : 0xffffu;
        }
        if (ld) tmem_wait_ld();
        prof.mark(3);
        float tmax = -INFINITY;
        if (active && has[0] && !dry) {
          float mx0 = -INFINITY, mx1 = -INFINITY;
          if (partial) {
#pragma unroll
            for (int i = 0; i < kChunks; ++i)
              if (has[i]) chunk_max<true>(r[i], mk[i], mx0, mx1);
          } else {
#pragma unroll
            for (int i = 0; i < kChunks; ++i)
              if (has[i]) chunk_max<false>(r[i], 0xffffu, mx0, mx1);
          }
          tmax = fmaxf(mx0, mx1);
        }
        // lazy rescale decision (warp-uniform for the TMEM accesses)
        const bool need = tmax > m + thresh || (m == -INFINITY && tmax != -INFINITY);
        float alpha = 1.f;
        if (need) {
          alpha = ex2((m - tmax) * c);                     // 0 when m = -inf
          m = tmax;
        }
        l *= alpha;
        prof.mark(4);
        if (j > 0 && __any_sync(0xffffffffu, need && alpha != 0.f)) {
          // O_cg holds tiles < n once P.V(n-1) is done; P.V(n) is not issued before p_full
          mbar_wait(bar(ctl->pv_done[(n - 1) % kSbuf]), ((n - 1) / kSbuf) & 1);
          tc_fence_after();
          if (active) {
#pragma unroll
            for (int h2 = 0; h2 < 4; ++h2) {
              uint32_t rr[16];
              tmem_ld16(tl + kTmemO + cg * 64 + h2 * 16, rr);
              tmem_wait_ld();
#pragma unroll
              for (int i = 0; i < 16; ++i) rr[i] = __float_as_uint(__uint_as_float(rr[i]) * alpha);
              tmem_st16(tl + kTmemO + cg * 64 + h2 * 16, rr);
            }
          }
        }
        prof.mark(5);
        // p = 2^(s*c - m*c) (masked -> 0), packed to 16-bit pairs over the chunk's first 8 columns
        if (active && has[0] && !dry) {
          const float mu = (m == -INFINITY) ? 0.f : m;
          const float2 nb2 = make_float2(-mu * c, -mu * c);
          float2 rs0 = make_float2(0.f, 0.f), rs1 = make_float2(0.f, 0.f);
          if (partial) {
#pragma unroll
            for (int i = 0; i < kChunks; ++i)
              if (has[i]) chunk_exp<true, kBF16>(r[i], mk[i], c2, nb2, rs0, rs1, tSb + kGroups * 16 * i);
          } else {
#pragma unroll
            for (int i = 0; i < kChunks; ++i)
              if (has[i]) chunk_exp<false, kBF16>(r[i], 0xffffu, c2, nb2, rs0, rs1, tSb + kGroups * 16 * i);
          }
          l += (rs0.x + rs0.y) + (rs1.x + rs1.y);
          tmem_wait_st();
        }
        prof.mark(7);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(bar(ctl->p_full[b]));
        prof.mark(8);
        if (tlw && j == ntiles - 1) tl_rec(p, it - 1, 2);
        if (j == 0 && pend.valid) {                        // previous item's epilogue
          epilogue(pend);
          pend.valid = false;
        }
      }
      pend = Epi{m, l, r_out, slot_f, ubh, n - 1, ipar, it - 1, active, true};
    }
    if (pend.valid) epilogue(pend);
    prof.flush(p, 2 + (warp == 8));
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
