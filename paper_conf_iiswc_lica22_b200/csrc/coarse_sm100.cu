// Coarse-grained fused kernel for sm_100a: per work item (a 128-row block of one (batch, head)),
//   SDDMM   S_j = Q_I K_j^T             tcgen05.mma (SS), S in TMEM        (§3.2)
//   scale + mask + online SpSoftmax     one thread per row, bits per tile  (§3.3)
//   SpMM    O_j = P_j V_j               tcgen05.mma (TS: P from TMEM)     (§3.2)
// with the per-row running (max, sum) carried across the row's tiles instead of re-reading S
// (the paper's 3-sweep SpSoftmax is replaced by an online softmax; the result is
// the same masked softmax). Work items are
//   kind 0: a band row block with its BSR tiles (+ an optional gathered "strip" tile that carries
//           the row block's CSR residual on the tensor cores), merged in the epilogue with the
//           fp32 partial statistics written by the CUDA-core fine kernel for any remaining CSR rows;
//   kind 1: up to 128 gathered global rows against every column tile (the dense-row part,
//           P:103 / P:133 — CUTLASS + TensorRT in the paper).
// Warp roles (one CTA per SM, persistent, dynamic work counter):
//   warp 0      producer: work fetch, TMA loads of Q/K/V tiles (SWIZZLE_128B), row gathers
//   warp 1      MMA issuer (one thread): S_j = Q K_j^T, O_j = P_j V_j
//   warp 2      TMEM allocator
//   warps 4..7  softmax / correction / epilogue, thread t owns row t (TMEM lane t)
// TMEM (512 columns): S double buffer [0,256), P double buffer (bf16x2) [256,384),
// O double buffer [384,512). O_j is accumulated into registers with the running rescale.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "kernels.cuh"
#include "sm100_ptx.cuh"

namespace mg {

using namespace ptx;

namespace {

constexpr int kStages = 4;
constexpr int kThreads = 256;
constexpr uint32_t kTileBytes = 128 * 128;  // 128 rows x 64 x 16-bit
constexpr uint32_t kTmemS = 0;
constexpr uint32_t kTmemP = 256;
constexpr uint32_t kTmemO = 384;

struct __align__(8) SmemCtl {
  uint64_t q_full, q_empty;
  uint64_t k_full[kStages], v_full[kStages], kv_empty[kStages];
  uint64_t s_full[2], p_full[2], o_full[2];
  uint64_t item_full[2], item_empty[2];
  int32_t item_id[2];
  uint32_t tmem_base;
};

constexpr size_t kSmemBytes = 1024 + kTileBytes * (1 + 2 * kStages) + sizeof(SmemCtl);

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
  for (int e = lane; e < nfill * 8; e += 32) {
    const int r = e >> 3, c = e & 7;
    int4 val = make_int4(0, 0, 0, 0);
    if (r < nvalid) {
      const int src = __ldg(idx + r);
      if (src >= 0) val = ld_nc_v4(base + (int64_t)src * sl + c * 8);
    }
    *reinterpret_cast<int4*>(dst + r * 128 + ((c ^ (r & 7)) << 4)) = val;
  }
}

__device__ __forceinline__ uint32_t chunk_bits(uint64_t w0, uint64_t w1, int ch) {
  const uint64_t w = ch < 2 ? w0 : w1;
  return (uint32_t)(w >> ((ch & 1) * 32));
}

template <bool kBF16>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  return kBF16 ? pack_bf16(lo, hi) : pack_f16(lo, hi);
}

}  // namespace

template <bool kBF16>
__global__ void __launch_bounds__(kThreads, 1)
    coarse_kernel(const __grid_constant__ CUtensorMap tmq, const __grid_constant__ CUtensorMap tmk,
                  const __grid_constant__ CUtensorMap tmv, const CoarseParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = smem + kTileBytes;
  uint8_t* sV = sK + kStages * kTileBytes;
  SmemCtl* ctl = reinterpret_cast<SmemCtl*>(sV + kStages * kTileBytes);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  const uint32_t q_full = smem_u32(&ctl->q_full), q_empty = smem_u32(&ctl->q_empty);
  auto k_full = [&](uint32_t s) { return smem_u32(&ctl->k_full[s]); };
  auto v_full = [&](uint32_t s) { return smem_u32(&ctl->v_full[s]); };
  auto kv_empty = [&](uint32_t s) { return smem_u32(&ctl->kv_empty[s]); };
  auto s_full = [&](uint32_t b) { return smem_u32(&ctl->s_full[b]); };
  auto p_full = [&](uint32_t b) { return smem_u32(&ctl->p_full[b]); };
  auto o_full = [&](uint32_t b) { return smem_u32(&ctl->o_full[b]); };
  auto item_full = [&](uint32_t b) { return smem_u32(&ctl->item_full[b]); };
  auto item_empty = [&](uint32_t b) { return smem_u32(&ctl->item_empty[b]); };

  if (threadIdx.x == 0) {
    mbar_init(q_full, 1);
    mbar_init(q_empty, 1);
    for (int s = 0; s < kStages; ++s) {
      mbar_init(k_full(s), 1);
      mbar_init(v_full(s), 1);
      mbar_init(kv_empty(s), 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(s_full(b), 1);
      mbar_init(p_full(b), 4);
      mbar_init(o_full(b), 1);
      mbar_init(item_full(b), 1);
      mbar_init(item_empty(b), 5);
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

  if (warp == 0) {
    // ============================================================ producer
    const uint64_t pol_kv = policy_evict_last();   // K/V tiles are re-read by neighbouring row blocks
    const uint64_t pol_q = policy_evict_first();   // Q tile is read once
    uint32_t it = 0, g = 0, qi = 0;
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      int u = 0;
      if (lane == 0) {
        mbar_wait(item_empty(slot), ph ^ 1);
        u = atomicAdd(p.counter, 1);
        ctl->item_id[slot] = u;
        mbar_arrive(item_full(slot));
      }
      u = __shfl_sync(0xffffffffu, u, 0);
      ++it;
      if (u >= p.total_units) break;
      const UnitInfo ui = decode_unit(p, u);
      const Item item = p.items[ui.item];
      const int bb = ui.bh / p.H, hh = ui.bh % p.H;
      mbar_wait(q_empty, (qi & 1) ^ 1);
      if (item.kind == 0) {
        if (lane == 0) {
          mbar_arrive_expect_tx(q_full, kTileBytes);
          tma_load_4d(smem_u32(sQ), &tmq, q_full, 0, item.row0, hh, bb, pol_q);
        }
      } else {
        const uint16_t* qb = p.q.data + bb * p.q.sb + hh * p.q.sh;
        gather_rows(sQ, qb, p.q.sl, p.global_rows + item.row0, min(128, p.n_global - item.row0), 128, lane);
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(q_full);
      }
      ++qi;
      for (int j = 0; j < item.ntiles; ++j, ++g) {
        const TileRef tr = p.trefs[item.tref_begin + j];
        const uint32_t st = g % kStages, sph = (g / kStages) & 1;
        mbar_wait(kv_empty(st), sph ^ 1);
        uint8_t* dK = sK + st * kTileBytes;
        uint8_t* dV = sV + st * kTileBytes;
        if (tr.kind == 0) {
          if (lane == 0) {
            mbar_arrive_expect_tx(k_full(st), kTileBytes);
            tma_load_4d(smem_u32(dK), &tmk, k_full(st), 0, tr.arg, hh, bb, pol_kv);
            mbar_arrive_expect_tx(v_full(st), kTileBytes);
            tma_load_4d(smem_u32(dV), &tmv, v_full(st), 0, tr.arg, hh, bb, pol_kv);
          }
        } else {
          const int32_t* idx = p.strip_cols + tr.arg;
          gather_rows(dK, p.k.data + bb * p.k.sb + hh * p.k.sh, p.k.sl, idx, tr.ncols, tr.ncols, lane);
          fence_proxy_async_smem();
          __syncwarp();
          if (lane == 0) mbar_arrive(k_full(st));
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
    const bool leader = lane == 0;
    const uint32_t idesc_pv = idesc_f16(kBF16, 128, 64, false, true);
    const uint32_t sQa = smem_u32(sQ);
    uint32_t it = 0, g = 0, qi = 0;
    auto issue_pv = [&](uint32_t x, int ncols, uint32_t st) {
      const uint32_t buf = x & 1;
      mbar_wait(p_full(buf), (x >> 1) & 1);
      mbar_wait(v_full(st), (x / kStages) & 1);
      tc_fence_after();
      if (leader) {
        const uint32_t dO = tmem + kTmemO + buf * 64;
        const uint32_t aP = tmem + kTmemP + buf * 64;
        const uint32_t vA = smem_u32(sV + st * kTileBytes);
        for (int kk = 0; kk < (ncols >> 4); ++kk)
          mma_ts(dO, aP + kk * 8, smem_desc_sw128(vA + kk * 2048, 8192, 1024), idesc_pv, kk > 0);
        mma_commit(o_full(buf));
        mma_commit(kv_empty(st));
      }
      __syncwarp();
    };
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      mbar_wait(item_full(slot), ph);
      const int u = ctl->item_id[slot];
      __syncwarp();
      if (leader) mbar_arrive(item_empty(slot));
      ++it;
      if (u >= p.total_units) break;
      const Item item = p.items[decode_unit(p, u).item];
      mbar_wait(q_full, qi & 1);
      ++qi;
      tc_fence_after();
      int prev_ncols = 0;
      uint32_t prev_st = 0;
      for (int j = 0; j < item.ntiles; ++j) {
        const uint32_t gg = g + j;
        const TileRef tr = p.trefs[item.tref_begin + j];
        const uint32_t st = gg % kStages;
        mbar_wait(k_full(st), (gg / kStages) & 1);
        tc_fence_after();
        if (leader) {
          const uint32_t idesc_s = idesc_f16(kBF16, 128, tr.ncols, false, false);
          const uint32_t dS = tmem + kTmemS + (gg & 1) * 128;
          const uint32_t kA = smem_u32(sK + st * kTileBytes);
#pragma unroll
          for (int kk = 0; kk < 4; ++kk)
            mma_ss(dS, smem_desc_sw128(sQa + kk * 32, 16, 1024), smem_desc_sw128(kA + kk * 32, 16, 1024), idesc_s,
                   kk > 0);
          mma_commit(s_full(gg & 1));
          if (j == item.ntiles - 1) mma_commit(q_empty);
        }
        __syncwarp();
        if (j >= 1) issue_pv(gg - 1, prev_ncols, prev_st);
        prev_ncols = tr.ncols;
        prev_st = st;
      }
      issue_pv(g + item.ntiles - 1, prev_ncols, prev_st);
      g += item.ntiles;
    }
  } else if (warp >= 4) {
    // ============================================================ softmax + epilogue
    const int t = threadIdx.x - 128;                       // row within the tile = TMEM lane
    const uint32_t lane_base = (uint32_t)((warp & 3) * 32) << 16;
    const float c = p.scale_log2;
    uint32_t it = 0, g = 0;
    float oacc[64];
    auto consume = [&](uint32_t x, float a) {
      const uint32_t buf = x & 1;
      mbar_wait(o_full(buf), (x >> 1) & 1);
      tc_fence_after();
      const uint32_t tO = tmem + lane_base + kTmemO + buf * 64;
#pragma unroll
      for (int h2 = 0; h2 < 2; ++h2) {
        uint32_t r[32];
        tmem_ld32(tO + h2 * 32, r);
        tmem_wait_ld();
#pragma unroll
        for (int i = 0; i < 32; ++i) oacc[h2 * 32 + i] = fmaf(oacc[h2 * 32 + i], a, __uint_as_float(r[i]));
      }
    };
    while (true) {
      const uint32_t slot = it & 1, ph = (it >> 1) & 1;
      mbar_wait(item_full(slot), ph);
      const int u = ctl->item_id[slot];
      __syncwarp();
      if (lane == 0) mbar_arrive(item_empty(slot));
      ++it;
      if (u >= p.total_units) break;
      const UnitInfo ui = decode_unit(p, u);
      const Item item = p.items[ui.item];
      float m = -INFINITY, l = 0.f, alpha_prev = 0.f;
#pragma unroll
      for (int i = 0; i < 64; ++i) oacc[i] = 0.f;
      for (int j = 0; j < item.ntiles; ++j) {
        const uint32_t gg = g + j, buf = gg & 1;
        const TileRef tr = p.trefs[item.tref_begin + j];
        uint64_t w0 = ~0ull, w1 = ~0ull;
        if (tr.mask >= 0) {
          const ulonglong2 mw = __ldg(reinterpret_cast<const ulonglong2*>(p.masks + ((size_t)tr.mask * 128 + t) * 2));
          w0 = mw.x;
          w1 = mw.y;
        }
        const int nch = tr.ncols >> 5;
        mbar_wait(s_full(buf), (gg >> 1) & 1);
        tc_fence_after();
        const uint32_t tS = tmem + lane_base + kTmemS + buf * 128;
        // pass 1: masked row max of this tile
        float tmax = -INFINITY;
#pragma unroll
        for (int ch = 0; ch < 4; ++ch) {
          if (ch < nch) {
            uint32_t r[32];
            tmem_ld32(tS + ch * 32, r);
            tmem_wait_ld();
            const uint32_t bits = chunk_bits(w0, w1, ch);
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if ((bits >> i) & 1u) tmax = fmaxf(tmax, __uint_as_float(r[i]));
          }
        }
        const float m_new = fmaxf(m, tmax);
        const float mu = (m_new == -INFINITY) ? 0.f : m_new;
        const float alpha = ex2((m - mu) * c);
        const float nbias = -mu * c;
        // pass 2: p = 2^(s*c - m*c), packed to 16-bit into TMEM as the A operand of P.V
        float rs = 0.f;
        const uint32_t tP = tmem + lane_base + kTmemP + buf * 64;
#pragma unroll
        for (int ch = 0; ch < 4; ++ch) {
          if (ch < nch) {
            uint32_t r[32];
            tmem_ld32(tS + ch * 32, r);
            tmem_wait_ld();
            const uint32_t bits = chunk_bits(w0, w1, ch);
            uint32_t pk[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) {
              const float p0 = ((bits >> (2 * i)) & 1u) ? ex2(fmaf(__uint_as_float(r[2 * i]), c, nbias)) : 0.f;
              const float p1 = ((bits >> (2 * i + 1)) & 1u) ? ex2(fmaf(__uint_as_float(r[2 * i + 1]), c, nbias)) : 0.f;
              rs += p0 + p1;
              pk[i] = pack2<kBF16>(p0, p1);
            }
            tmem_st16(tP + ch * 16, pk);
          }
        }
        tmem_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(p_full(buf));
        l = l * alpha + rs;
        if (j >= 1) consume(gg - 1, alpha_prev);
        alpha_prev = alpha;
        m = m_new;
      }
      consume(g + item.ntiles - 1, alpha_prev);
      g += item.ntiles;

      // ---- epilogue: merge the fine partial (if any), normalise, store 16-bit O
      int r = -1;
      if (item.kind == 0) {
        const int64_t rr = (int64_t)item.row0 + t;
        if (rr < p.L) r = (int)rr;
      } else if (item.row0 + t < p.n_global) {
        r = __ldg(p.global_rows + item.row0 + t);
      }
      if (r >= 0) {
        float mf = -INFINITY, lf = 0.f;
        const float* accf = nullptr;
        if (item.kind == 0) {
          const int slot_f = __ldg(p.fine_slot + r);
          if (slot_f >= 0) {
            const size_t idx = (size_t)ui.bh * p.n_fine_rows + slot_f;
            const float2 ml = p.part_ml[idx];
            mf = ml.x;
            lf = ml.y;
            accf = p.part_acc + idx * 64;
          }
        }
        const float mt = fmaxf(m, mf);
        if (mt != -INFINITY) {
          const float ac = ex2((m - mt) * c);
          const float af = ex2((mf - mt) * c);
          const float inv = 1.f / (l * ac + lf * af);
          const int bb = ui.bh / p.H, hh = ui.bh % p.H;
          uint16_t* orow = p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)r * p.o.sl;
#pragma unroll
          for (int q8 = 0; q8 < 8; ++q8) {
            float v[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) v[e] = oacc[q8 * 8 + e] * ac;
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
