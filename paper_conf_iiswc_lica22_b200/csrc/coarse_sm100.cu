// Coarse-grained fused kernel for sm_100a: per work item (a 128-row block of one (batch, head)),
//   SDDMM   S_j = Q_I K_j^T             tcgen05.mma (SS), S in TMEM        (§3.2)
//   scale + mask + online SpSoftmax     thread per (row, column half)      (§3.3)
//   SpMM    O_j = P_j V_j               tcgen05.mma (TS: P from TMEM)     (§3.2)
// with the per-row running (max, sum) carried across the row's tiles instead of re-reading S
// (A14: the paper's 3-sweep SpSoftmax becomes an online softmax; same result).
// Work items:
//   kind 0: a band row block with its BSR tiles (+ an optional gathered "strip" tile carrying the
//           row block's CSR residual on the tensor cores); the epilogue merges the fp32 partial
//           statistics written by the CUDA-core fine kernel for any remaining CSR rows;
//   kind 1: up to 128 gathered global rows against every column tile (the dense-row part,
//           P:103 / P:133 — CUTLASS + TensorRT in the paper).
// Warp roles (one 384-thread CTA per SM, persistent, dynamic work counter):
//   warp 0       producer: work fetch, TMA loads of Q/K/V tiles (SWIZZLE_128B), row gathers
//   warp 1       MMA issuer (lane 0): S_j = Q K_j^T; O_j = P_j V_j as two K-halves (one per softmax WG)
//   warp 2       TMEM allocator
//   warps 4..7   softmax WG0: thread t owns row t, columns [0, n/2) of every tile
//   warps 8..11  softmax WG1: thread t owns row t, columns [n/2, n) of every tile
// Each WG keeps its own online (m, l, O) over its column half — two disjoint parts of the row —
// and the halves are merged by log-sum-exp in the epilogue together with the fine partial
// (compound SpSoftmax over coarse and fine parts).
// TMEM (512 columns): S/O triple buffer [0, 384): S_j is overwritten by O_j = (O_A | O_B) once
// both WGs have stored P_j; P double buffer (16-bit pairs) [384, 512).
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
constexpr uint32_t kTmemP = 384;
constexpr int kXchStride = 36;              // floats per row in the WG exchange buffer

struct __align__(16) ItemSlot {
  Item item;
  int32_t u, bh, pad0, pad1;
};

struct __align__(16) SmemCtl {
  TileRef tref[kStages];                    // tile descriptor of each K/V stage
  ItemSlot slot[2];                         // work item broadcast to the MMA and softmax warps
  uint64_t q_full[2], q_empty[2];
  uint64_t k_full[kStages], v_full[kStages], kv_empty[kStages];
  uint64_t s_full[3], o_full[3], o_empty[3];
  uint64_t p_full[2];
  uint64_t item_full[2], item_empty[2];
  uint32_t tmem_base;
};

constexpr uint32_t kMaskBytes = 128 * 16;  // 128 rows x 2 x u64 per tile bitmask
constexpr size_t kXchBytes = 2 * 128 * kXchStride * sizeof(float);
constexpr size_t kSmemBytes =
    1024 + kTileBytes * (2 + 2 * kStages) + kMaskBytes * kStages + kXchBytes + sizeof(SmemCtl);
static_assert(kSmemBytes <= 227 * 1024, "shared memory budget");

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
__device__ __forceinline__ void gather_rows(uint8_t* dst, const uint16_t* base, int64_t sl, const int32_t* idx,
                                            int nvalid, int nfill, int lane) {
  const uint32_t d0 = smem_u32(dst);
  for (int e = lane; e < nfill * 8; e += 32) {
    const int r = e >> 3, c = e & 7;
    int4 val = make_int4(0, 0, 0, 0);
    if (r < nvalid) {
      const int src = __ldg(idx + r);
      if (src >= 0) val = ld_nc_v4(base + (int64_t)src * sl + c * 8);
    }
    const uint32_t a = d0 + r * 128 + ((c ^ (r & 7)) << 4);
    asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(val.x), "r"(val.y), "r"(val.z),
                 "r"(val.w)
                 : "memory");
  }
}

template <bool kBF16>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  return kBF16 ? pack_bf16(lo, hi) : pack_f16(lo, hi);
}

// 64-bit window of a 128-bit mask row starting at bit `off` (off in {0, 16, 32, 64}; the window
// never straddles the two words because off + h <= 64 whenever off < 64).
__device__ __forceinline__ uint64_t mask_window(uint64_t w0, uint64_t w1, int off) {
  return off >= 64 ? w1 : (w0 >> off);
}

// Diagnostics: CTA 0 appends (clock64, role<<56 | event<<48 | arg) to its role's private segment
// of p.trace (4 segments of trace_cap/4 pairs; pair 0 of a segment holds the count). Plain
// stores only, so the timeline is not perturbed by atomics. Roles: 0 producer, 1 MMA, 2 softmax
// warp 4, 3 softmax warp 8.
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
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;                              // 2 Q buffers
  uint8_t* sK = smem + 2 * kTileBytes;
  uint8_t* sV = sK + kStages * kTileBytes;
  uint8_t* sM = sV + kStages * kTileBytes;          // tile bitmasks, one per stage
  float* xch = reinterpret_cast<float*>(sM + kStages * kMaskBytes);
  SmemCtl* ctl = reinterpret_cast<SmemCtl*>(reinterpret_cast<uint8_t*>(xch) + kXchBytes);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  auto q_full = [&](uint32_t b) { return smem_u32(&ctl->q_full[b]); };
  auto q_empty = [&](uint32_t b) { return smem_u32(&ctl->q_empty[b]); };
  auto k_full = [&](uint32_t s) { return smem_u32(&ctl->k_full[s]); };
  auto v_full = [&](uint32_t s) { return smem_u32(&ctl->v_full[s]); };
  auto kv_empty = [&](uint32_t s) { return smem_u32(&ctl->kv_empty[s]); };
  auto s_full = [&](uint32_t b) { return smem_u32(&ctl->s_full[b]); };
  auto o_full = [&](uint32_t b) { return smem_u32(&ctl->o_full[b]); };
  auto o_empty = [&](uint32_t b) { return smem_u32(&ctl->o_empty[b]); };
  auto p_full = [&](uint32_t b) { return smem_u32(&ctl->p_full[b]); };
  auto item_full = [&](uint32_t b) { return smem_u32(&ctl->item_full[b]); };
  auto item_empty = [&](uint32_t b) { return smem_u32(&ctl->item_empty[b]); };

  if (threadIdx.x == 0) {
    for (int b = 0; b < 2; ++b) {
      mbar_init(q_full(b), 1);
      mbar_init(q_empty(b), 1);
    }
    for (int s = 0; s < kStages; ++s) {
      mbar_init(k_full(s), 1);
      mbar_init(v_full(s), 1);
      mbar_init(kv_empty(s), 1);
    }
    for (int b = 0; b < 3; ++b) {
      mbar_init(s_full(b), 1);
      mbar_init(o_full(b), 1);
      mbar_init(o_empty(b), 8);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(p_full(b), 8);
      mbar_init(item_full(b), 1);
      mbar_init(item_empty(b), 9);
    }
    fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
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
  // Register rebalancing per warpgroup: the producer/MMA warpgroup needs few registers, the
  // softmax warpgroups hold a 64-column S slice and a 64-column O accumulator per thread.
  // setmaxnreg.inc draws from the CTA's own pool (168 x 384 = 64512 registers at launch), so
  // 128 x 88 + 256 x 208 must not exceed it (it equals it) or the inc blocks forever.
  if (warp < 4) {
  asm volatile("setmaxnreg.dec.sync.aligned.u32 88;" ::: "memory");
  if (warp == 0) {
    // ============================================================ producer
    Tracer trace(p, 0);
    const uint64_t pol_kv = policy_evict_last();   // K/V tiles are re-read by neighbouring row blocks
    const uint64_t pol_q = policy_evict_first();   // Q tile is read once
    uint32_t it = 0, g = 0, qi = 0;
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      int u = 0;
      if (lane == 0) {
        mbar_wait(item_empty(slot), ph ^ 1);
        u = atomicAdd(p.counter, 1);
        ItemSlot is;
        is.u = u;
        if (u < p.total_units) {
          const UnitInfo ui = decode_unit(p, u);
          is.item = p.items[ui.item];
          is.bh = ui.bh;
        }
        ctl->slot[slot] = is;
        mbar_arrive(item_full(slot));
      }
      u = __shfl_sync(0xffffffffu, u, 0);
      ++it;
      if (u >= p.total_units) break;
      __syncwarp();
      const Item item = ctl->slot[slot].item;
      const int bh = ctl->slot[slot].bh;
      const int bb = bh / p.H, hh = bh % p.H;
      const uint32_t qb = qi & 1;
      uint8_t* dQ = sQ + qb * kTileBytes;
      if (lane == 0) trace(0, 1, u);                       // item fetched
      mbar_wait(q_empty(qb), ((qi >> 1) & 1) ^ 1);
      if (lane == 0) trace(0, 2, qi);                      // Q buffer free
      if (item.kind == 0) {
        if (lane == 0) {
          mbar_arrive_expect_tx(q_full(qb), kTileBytes);
          tma_load_4d(smem_u32(dQ), &tmq, q_full(qb), 0, item.row0, hh, bb, pol_q);
        }
      } else {
        const uint16_t* qsrc = p.q.data + bb * p.q.sb + hh * p.q.sh;
        gather_rows(dQ, qsrc, p.q.sl, p.global_rows + item.row0, min(128, p.n_global - item.row0), 128, lane);
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(q_full(qb));
      }
      ++qi;
      for (int j = 0; j < item.ntiles; ++j, ++g) {
        const TileRef tr = p.trefs[item.tref_begin + j];
        const uint32_t st = g % kStages, sph = (g / kStages) & 1;
        mbar_wait(kv_empty(st), sph ^ 1);
        if (lane == 0) trace(0, 3, g);                     // stage free, loads issued
        uint8_t* dK = sK + st * kTileBytes;
        uint8_t* dV = sV + st * kTileBytes;
        const uint32_t dM = smem_u32(sM + st * kMaskBytes);
        const uint32_t mbytes = tr.mask >= 0 ? kMaskBytes : 0;
        if (lane == 0) ctl->tref[st] = tr;   // published by the k_full arrive below
        if (tr.kind == 0) {
          if (lane == 0) {
            mbar_arrive_expect_tx(k_full(st), kTileBytes + mbytes);
            tma_load_4d(smem_u32(dK), &tmk, k_full(st), 0, tr.arg, hh, bb, pol_kv);
            if (mbytes) bulk_load(dM, p.masks + (size_t)tr.mask * 256, kMaskBytes, k_full(st));
            mbar_arrive_expect_tx(v_full(st), kTileBytes);
            tma_load_4d(smem_u32(dV), &tmv, v_full(st), 0, tr.arg, hh, bb, pol_kv);
          }
        } else {
          const int32_t* idx = p.strip_cols + tr.arg;
          gather_rows(dK, p.k.data + bb * p.k.sb + hh * p.k.sh, p.k.sl, idx, tr.ncols, tr.ncols, lane);
          fence_proxy_async_smem();
          __syncwarp();
          if (lane == 0) {
            if (mbytes) {
              mbar_arrive_expect_tx(k_full(st), mbytes);
              bulk_load(dM, p.masks + (size_t)tr.mask * 256, kMaskBytes, k_full(st));
            } else {
              mbar_arrive(k_full(st));
            }
          }
          gather_rows(dV, p.v.data + bb * p.v.sb + hh * p.v.sh, p.v.sl, idx, tr.ncols, tr.ncols, lane);
          fence_proxy_async_smem();
          __syncwarp();
          if (lane == 0) mbar_arrive(v_full(st));
        }
      }
    }
  } else if (warp == 1) {
    // ============================================================ MMA issuer
    // The whole warp walks the schedule (waits are warp-wide); lane 0 issues tcgen05.mma/commit.
    // Within an item S_{j+1} is issued before P_j V_j; the last P.V of an item is issued at once
    // and the next item's S_0 follows it (its Q is already in the other Q buffer).
    const bool leader = lane == 0;
    Tracer trace(p, 1);
    uint32_t it = 0, g = 0, qi = 0;
    auto issue_pv = [&](uint32_t x, int ncols, uint32_t st) {
      const uint32_t buf = x & 1, xs = x % 3;
      mbar_wait(p_full(buf), (x >> 1) & 1);
      if (leader) trace(1, 4, x);                          // P ready
      mbar_wait(v_full(st), (x / kStages) & 1);
      if (leader) trace(1, 5, x);                          // V ready, PV issued
      tc_fence_after();
      if (leader) {
        const int h = ncols >> 1, nk = h >> 4;
        const uint32_t idesc = idesc_f16(kBF16, 128, 64, false, true);
        const uint32_t aP = tmem + kTmemP + buf * 64;
        const uint32_t vA = smem_u32(sV + st * kTileBytes);
        for (int half = 0; half < 2; ++half) {
          const uint32_t dO = tmem + xs * 128 + half * 64;
          for (int kk = 0; kk < nk; ++kk) {
            const int k = half * nk + kk;
            mma_ts(dO, aP + k * 8, smem_desc_sw128(vA + k * 2048, 8192, 1024), idesc, kk > 0);
          }
        }
        mma_commit(o_full(xs));
        mma_commit(kv_empty(st));
      }
      __syncwarp();
    };
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      mbar_wait(item_full(slot), ph);
      const int u = ctl->slot[slot].u;
      const Item item = ctl->slot[slot].item;
      __syncwarp();
      if (leader) mbar_arrive(item_empty(slot));
      ++it;
      if (u >= p.total_units) break;
      const uint32_t qb = qi & 1;
      const uint32_t sQa = smem_u32(sQ + qb * kTileBytes);
      mbar_wait(q_full(qb), (qi >> 1) & 1);
      if (leader) trace(1, 0, qi);                         // Q ready
      ++qi;
      tc_fence_after();
      int prev_n = 0;
      uint32_t prev_st = 0;
      for (int j = 0; j < item.ntiles; ++j) {
        const uint32_t gg = g + j, xs = gg % 3;
        const uint32_t st = gg % kStages;
        mbar_wait(k_full(st), (gg / kStages) & 1);
        if (leader) trace(1, 1, gg);                       // K ready
        const int ncols = ctl->tref[st].ncols;
        if (gg >= 3) mbar_wait(o_empty(xs), ((gg / 3) - 1) & 1);
        if (leader) trace(1, 2, gg);                       // S buffer free, S issued
        tc_fence_after();
        if (leader) {
          const uint32_t idesc_s = idesc_f16(kBF16, 128, ncols, false, false);
          const uint32_t dS = tmem + xs * 128;
          const uint32_t kA = smem_u32(sK + st * kTileBytes);
#pragma unroll
          for (int kk = 0; kk < 4; ++kk)
            mma_ss(dS, smem_desc_sw128(sQa + kk * 32, 16, 1024), smem_desc_sw128(kA + kk * 32, 16, 1024), idesc_s,
                   kk > 0);
          mma_commit(s_full(xs));
          if (j == item.ntiles - 1) mma_commit(q_empty(qb));
        }
        __syncwarp();
        if (j >= 1) issue_pv(gg - 1, prev_n, prev_st);
        prev_n = ncols;
        prev_st = st;
      }
      issue_pv(g + item.ntiles - 1, prev_n, prev_st);
      g += item.ntiles;
    }
  }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 208;" ::: "memory");
    // ============================================================ softmax + epilogue (2 WGs)
    const int wg = (warp - 4) >> 2;                        // column half
    const int q4 = warp & 3;                               // TMEM lane quarter
    const int t = q4 * 32 + lane;                          // row within the tile = TMEM lane
    const uint32_t lane_base = (uint32_t)(q4 * 32) << 16;
    const float c = p.scale_log2;
    const float2 c2 = make_float2(c, c);
    Tracer trace(p, 2 + (warp >> 3));
    const bool tr_on_item = (warp == 4 || warp == 8) && lane == 0;
    uint32_t it = 0, g = 0;
    float oacc[64];
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      mbar_wait(item_full(slot), ph);
      const int u = ctl->slot[slot].u;
      const Item item = ctl->slot[slot].item;
      const int ubh = ctl->slot[slot].bh;
      __syncwarp();
      if (lane == 0) mbar_arrive(item_empty(slot));
      ++it;
      if (u >= p.total_units) break;
      // rows of this warp that exist (dense items carry up to 128 gathered rows)
      const int nrows = item.kind == 0 ? (int)(p.L - item.row0 < 128 ? p.L - item.row0 : 128) : min(128, p.n_global - item.row0);
      const bool active = q4 * 32 < nrows;
      float m = -INFINITY, l = 0.f, alpha_prev = 0.f;
#pragma unroll
      for (int i = 0; i < 64; ++i) oacc[i] = 0.f;
      auto consume = [&](uint32_t x, float a) {
        const uint32_t xs = x % 3;
        mbar_wait(o_full(xs), (x / 3) & 1);
        tc_fence_after();
        if (active) {
          const uint32_t tO = tmem + lane_base + xs * 128 + wg * 64;
#pragma unroll
          for (int h2 = 0; h2 < 2; ++h2) {
            uint32_t r[32];
            tmem_ld32(tO + h2 * 32, r);
            tmem_wait_ld();
            const float2 a2 = make_float2(a, a);
#pragma unroll
            for (int i = 0; i < 32; i += 2) {
              const float2 o = __ffma2_rn(make_float2(oacc[h2 * 32 + i], oacc[h2 * 32 + i + 1]), a2,
                                          make_float2(__uint_as_float(r[i]), __uint_as_float(r[i + 1])));
              oacc[h2 * 32 + i] = o.x;
              oacc[h2 * 32 + i + 1] = o.y;
            }
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(o_empty(xs));
      };
      for (int j = 0; j < item.ntiles; ++j) {
        const uint32_t gg = g + j, xs = gg % 3, buf = gg & 1, st = gg % kStages;
        // the stage's tile descriptor and bitmask landed with its K tile
        mbar_wait(k_full(st), (gg / kStages) & 1);
        const TileRef tr = ctl->tref[st];
        const int h = tr.ncols >> 1;                       // columns of this WG: [wg*h, wg*h + h)
        const int nch = h >> 4;                            // 16-column chunks (1..4)
        const bool partial = tr.mask >= 0;
        uint64_t bits = ~0ull;
        if (partial && active) {
          const ulonglong2 mw = *reinterpret_cast<const ulonglong2*>(sM + st * kMaskBytes + t * 16);
          bits = mask_window(mw.x, mw.y, wg * h);
        }
        const bool tr_on = (warp == 4 || warp == 8) && lane == 0;
        if (tr_on) trace(2 + (warp >> 3), 1, gg);                         // tile start
        mbar_wait(s_full(xs), (gg / 3) & 1);
        if (tr_on) trace(2 + (warp >> 3), 2, gg);                         // S ready
        tc_fence_after();
        float alpha = 1.f;
        if (active) {
          const uint32_t tS = tmem + lane_base + xs * 128 + wg * h;
          float s[64];
#pragma unroll
          for (int ch = 0; ch < 4; ++ch) {
            if (ch < nch) {
              uint32_t r[16];
              tmem_ld16(tS + ch * 16, r);
#pragma unroll
              for (int i = 0; i < 16; ++i) s[ch * 16 + i] = __uint_as_float(r[i]);
            }
          }
          tmem_wait_ld();
          if (partial) {
#pragma unroll
            for (int ch = 0; ch < 4; ++ch)
              if (ch < nch) {
#pragma unroll
                for (int i = 0; i < 16; ++i)
                  s[ch * 16 + i] = ((bits >> (ch * 16 + i)) & 1ull) ? s[ch * 16 + i] : -INFINITY;
              }
          }
          // masked row max over this WG's columns (3-input max, two independent chains)
          float mx0 = -INFINITY, mx1 = -INFINITY;
#pragma unroll
          for (int ch = 0; ch < 4; ++ch) {
            if (ch < nch) {
#pragma unroll
              for (int i = 0; i < 16; i += 4) {
                mx0 = fmax3(mx0, s[ch * 16 + i], s[ch * 16 + i + 1]);
                mx1 = fmax3(mx1, s[ch * 16 + i + 2], s[ch * 16 + i + 3]);
              }
            }
          }
          const float m_new = fmaxf(m, fmaxf(mx0, mx1));
          const float mu = (m_new == -INFINITY) ? 0.f : m_new;
          alpha = ex2((m - mu) * c);
          const float nb = -mu * c;
          const float2 nb2 = make_float2(nb, nb);
          float2 rs0 = make_float2(0.f, 0.f), rs1 = make_float2(0.f, 0.f);
          const uint32_t tP = tmem + lane_base + kTmemP + buf * 64 + ((wg * h) >> 1);
#pragma unroll
          for (int ch = 0; ch < 4; ++ch) {
            if (ch < nch) {
              uint32_t pk[8];
#pragma unroll
              for (int i = 0; i < 16; i += 2) {
                const float2 x = __ffma2_rn(make_float2(s[ch * 16 + i], s[ch * 16 + i + 1]), c2, nb2);
                const float p0 = ex2(x.x), p1 = ex2(x.y);
                if (i & 2)
                  rs1 = __fadd2_rn(rs1, make_float2(p0, p1));
                else
                  rs0 = __fadd2_rn(rs0, make_float2(p0, p1));
                pk[i >> 1] = pack2<kBF16>(p0, p1);
              }
              tmem_st8(tP + ch * 8, pk);
            }
          }
          tmem_wait_st();
          l = l * alpha + ((rs0.x + rs0.y) + (rs1.x + rs1.y));
          m = m_new;
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(p_full(buf));
        if (tr_on) trace(2 + (warp >> 3), 3, gg);                         // P stored
        if (j >= 1) consume(gg - 1, alpha_prev);
        if (tr_on) trace(2 + (warp >> 3), 4, gg);                         // O_{j-1} consumed
        alpha_prev = alpha;
      }
      consume(g + item.ntiles - 1, alpha_prev);
      if (tr_on_item) trace(2 + (warp >> 3), 5, g + item.ntiles - 1);   // item O complete
      g += item.ntiles;

      // ---- epilogue: merge the two column halves (+ the fine partial), normalise, store O
      // WG w finalises output columns [32w, 32w + 32); it sends the other WG's 32 columns.
      float* mine = xch + (wg * 128 + t) * kXchStride;
      // (register arrays are only indexed with compile-time constants: select by wg)
      float keep[32];
      {
#pragma unroll
        for (int i = 0; i < 32; i += 4) {
          const float a0 = wg ? oacc[i] : oacc[32 + i], a1 = wg ? oacc[i + 1] : oacc[33 + i];
          const float a2 = wg ? oacc[i + 2] : oacc[34 + i], a3 = wg ? oacc[i + 3] : oacc[35 + i];
          *reinterpret_cast<float4*>(mine + i) = make_float4(a0, a1, a2, a3);
        }
#pragma unroll
        for (int i = 0; i < 32; ++i) keep[i] = wg ? oacc[32 + i] : oacc[i];
        *reinterpret_cast<float2*>(mine + 32) = make_float2(m, l);
      }
      named_bar_sync(1, 256);
      if (tr_on_item) trace(2 + (warp >> 3), 6, 0);           // halves exchanged
      const float* other = xch + ((1 - wg) * 128 + t) * kXchStride;
      int r = -1;
      if (item.kind == 0) {
        if (t < nrows) r = item.row0 + t;
      } else if (t < nrows) {
        r = __ldg(p.global_rows + item.row0 + t);
      }
      if (r >= 0) {
        const float2 mlo = *reinterpret_cast<const float2*>(other + 32);
        float mf = -INFINITY, lf = 0.f;
        const float* accf = nullptr;
        if (item.kind == 0) {
          const int slot_f = __ldg(p.fine_slot + r);
          if (slot_f >= 0) {
            const size_t idx = (size_t)ubh * p.n_fine_rows + slot_f;
            const float2 ml = p.part_ml[idx];
            mf = ml.x;
            lf = ml.y;
            accf = p.part_acc + idx * 64 + wg * 32;
          }
        }
        const float mt = fmaxf(fmaxf(m, mlo.x), mf);
        if (mt != -INFINITY) {
          const float as = ex2((m - mt) * c), ao = ex2((mlo.x - mt) * c), af = ex2((mf - mt) * c);
          const float inv = 1.f / (l * as + mlo.y * ao + lf * af);
          const int bb = ubh / p.H, hh = ubh % p.H;
          uint16_t* orow = p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)r * p.o.sl + wg * 32;
#pragma unroll
          for (int q8 = 0; q8 < 4; ++q8) {
            float v[8];
            const float4 x0 = *reinterpret_cast<const float4*>(other + q8 * 8);
            const float4 x1 = *reinterpret_cast<const float4*>(other + q8 * 8 + 4);
            const float xo[8] = {x0.x, x0.y, x0.z, x0.w, x1.x, x1.y, x1.z, x1.w};
#pragma unroll
            for (int e = 0; e < 8; ++e) v[e] = fmaf(keep[q8 * 8 + e], as, xo[e] * ao);
            if (accf) {
              const float4 f0 = reinterpret_cast<const float4*>(accf)[q8 * 2];
              const float4 f1 = reinterpret_cast<const float4*>(accf)[q8 * 2 + 1];
              const float xf[8] = {f0.x, f0.y, f0.z, f0.w, f1.x, f1.y, f1.z, f1.w};
#pragma unroll
              for (int e = 0; e < 8; ++e) v[e] = fmaf(xf[e], af, v[e]);
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
