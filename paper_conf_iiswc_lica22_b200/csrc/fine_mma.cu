// Fine-grained CSR kernel on the warp-level tensor cores (mma.sync m16n8k16), the default for the
// CUDA-core CSR rows of the plan (the low-locality residual). Same contract as
// fine_rows.cu (one warp per (CSR row, batch*head); SDDMM -> online softmax -> SpMM fused; final
// row or fp32 partial for the coarse epilogue's merge), but the two dot-product phases
// run as small MMAs instead of per-element FMAs and shuffle reductions: the CUDA-core kernel is
// issue-bound (73% issue-active, 27 warp instructions per nnz, profiles/r01c_ncu_full_c4_fine.txt),
// while the gathers alone would run at ~22 TB/s from L2 (tools/microbench/gather_bw.cu).
//
// A step handles 16 nnz of the row, as two chunks A and B of 8. Lane = 4g + t.
//   SDDMM  s^T = q . K_c^T as mma(M=16 x N=8 x K=16) x 4 per chunk (64 dims): A = q broadcast to
//          all 16 rows (lane registers from the q slot of the row's first ring stage), B column n = gathered K row
//          of chunk nnz n (ldmatrix from the swizzled stage). D: lane (g,t) gets the scores of
//          chunk nnz 2t and 2t+1.
//   SpMM   O^T = V_c^T . p as mma(M=16 dims x N=8 x K=16 nnz) x 4 (64 dims): k = nnz (chunk A
//          nnz 2t,2t+1 -> k 2t,2t+1; chunk B -> k 2t+8, 2t+9), which is exactly where the SDDMM
//          left each lane's p, so P never moves between lanes; A = V^T from ldmatrix.trans. D:
//          lane (g,t) holds output dims 16j+g, 16j+g+8 (all N columns equal), and writes j = t.
// p is rounded to the operand dtype for the SpMM (as in the coarse kernel, A9); s, the
// running max/sum and O accumulate in fp32. Lazy rescaling: the exponent keeps a stale max until
// a step's max exceeds it by 8/c (p <= 256), warp-uniform because all lanes see the same max.
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <utility>

#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "kernels.cuh"
#include "sm100_ptx.cuh"

namespace mg {

using namespace ptx;

namespace {

template <bool kBF16>
__device__ __forceinline__ void mma16816(float (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                         uint32_t b0, uint32_t b1) {
  if (kBF16)
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
  else
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

template <bool kBF16>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  return kBF16 ? pack_bf16(lo, hi) : pack_f16(lo, hi);
}

__device__ __forceinline__ void cp_async16(uint32_t dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async16a(uint32_t dst, uint64_t src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
// base + a * b (64-bit result, one IMAD.WIDE.U32)
__device__ __forceinline__ uint64_t mad_wide(uint32_t a, uint32_t b, uint64_t base) {
  uint64_t r;
  asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(r) : "r"(a), "r"(b), "l"(base));
  return r;
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void ldsm_x4(uint32_t (&r)[4], uint32_t addr) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(addr));
}
__device__ __forceinline__ void ldsm_x4_t(uint32_t (&r)[4], uint32_t addr) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(addr));
}

#ifndef MG_FINE_STAGES
#define MG_FINE_STAGES 2
#endif
#ifndef MG_FINE_MINB
#define MG_FINE_MINB 5
#endif
#ifndef MG_FINE_PAIRS
#define MG_FINE_PAIRS 1
#endif
#ifndef MG_FINE_WARPS
#define MG_FINE_WARPS 4
#endif
#ifndef MG_FINE_IDX_AHEAD
#define MG_FINE_IDX_AHEAD 1
#endif
constexpr bool kIdxAhead = MG_FINE_IDX_AHEAD;   // column-index window prefetched one step ahead
constexpr int kWarps = MG_FINE_WARPS;       // warps per block, each a persistent row sequence
constexpr int kP = MG_FINE_PAIRS;           // 16-nnz pairs of 8-nnz chunks per step (1 or 2)
constexpr int kS = 16 * kP;                 // nnz per step
constexpr int kStages = MG_FINE_STAGES;     // smem ring stages per warp (kStages - 1 steps in flight)
// Head dimension kD = 64 or 128: a gathered row is kD * 2 bytes, copied by kD / 8 lanes
// (16 B each), 32 / (kD / 8) rows per cp.async instruction.
template <int kD>
struct FCfg {
  static constexpr int kRowBytes = kD * 2;
  static constexpr int kLPR = kD / 8;                   // lanes per gathered row
  static constexpr int kRPI = 32 / kLPR;                // rows per cp.async instruction
  static constexpr int kQOff = 2 * kS * kRowBytes;      // the q row of a row's first step follows its K and V rows
  static constexpr int kStageBytes = kQOff + kRowBytes; // kS K rows + kS V rows + q
  static constexpr int kSmemBytes = kWarps * kStages * kStageBytes;
  static constexpr int kMinB = kD == 64 ? MG_FINE_MINB : 3;
};

}  // namespace

// The 16 K rows and 16 V rows of a step are gathered with cp.async into a warp-private shared-memory
// ring, kStages - 1 steps ahead of the computation: 8 lanes copy one full 128-byte row per
// instruction (the pattern the L2 serves at ~15 TB/s through cp.async; partial-line pieces are 6x
// slower, tools/microbench/gather_bw.cu), and the copies hold no registers while in flight. Rows
// are stored with the 16-byte-chunk XOR swizzle (chunk c of row r at (c ^ (r & 7)) * 16), and the
// MMA fragments come from ldmatrix: non-transposed for the SDDMM's B operand (K rows = columns n,
// dims = k), transposed for the SpMM's A operand (V^T: dims = rows m, nnz = k).
// Persistent warps: warp w processes the rows w, w + W, w + 2W, ... of the (b*h, CSR row) space (W =
// warps in the grid; neighbouring warps stay on neighbouring rows of the same head, so the head's
// K/V stay in L2), and the gather pointer runs ahead across row boundaries, so a row's first gathers
// are in flight while the previous row is computed (one row is only ~11 steps).
// (b*h, CSR row) of a global row index: 32-bit division whenever the row space fits 32 bits (a
// 64-bit division is a ~100-instruction software routine, run twice per row)
__device__ __forceinline__ void split_row(int64_t g, int n, bool r32, int& u0, int& fi) {
  if (r32) {
    const uint32_t g32 = (uint32_t)g, q = g32 / (uint32_t)n;
    u0 = (int)q;
    fi = (int)(g32 - q * (uint32_t)n);
  } else {
    u0 = (int)(g / n);
    fi = (int)(g % n);
  }
}

template <bool kBF16, bool kPad, int kD>
__global__ void __launch_bounds__(kWarps * 32, FCfg<kD>::kMinB) fine_mma_kernel(const FineParams p) {
  using F = FCfg<kD>;
  constexpr int kRowBytes = F::kRowBytes, kLPR = F::kLPR, kRPI = F::kRPI, kQOff = F::kQOff;
  constexpr int kStageBytes = F::kStageBytes;
  constexpr int kJ = kD / 16;                           // k16 steps of the SDDMM = m16 blocks of the SpMM
  extern __shared__ __align__(128) uint8_t fsm[];
  const int lane = threadIdx.x & 31;
  const int g = lane >> 2, t = lane & 3;
  const float c = p.scale_log2;
  const float thresh = 8.f / c;
  const int64_t nrows = (int64_t)p.BH * p.n_fine_rows;
  const bool r32 = nrows <= (int64_t)0xffffffffLL;   // (split_row is only called with an index < nrows)
  const int64_t W = (int64_t)gridDim.x * kWarps;
  const int64_t w0 = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5);
  const uint32_t ring = (uint32_t)__cvta_generic_to_shared(fsm) + (threadIdx.x >> 5) * (kStages * kStageBytes);
  // row strides fit 32 bits (checked by the forward's validation: (L - 1) * stride_l < 2^32)
  const uint32_t ksl = (uint32_t)p.k.sl, vsl = (uint32_t)p.v.sl;
  constexpr int kIters = kS / kRPI;   // cp.async instructions per lane per step (each of K and V)
  uint32_t doff[kIters];   // swizzled destination of this lane's chunk in rows R_i = lane / kLPR + kRPI i
#pragma unroll
  for (int i = 0; i < kIters; ++i) {
    const int R = lane / kLPR + kRPI * i;
    doff[i] = R * kRowBytes + (((lane % kLPR) ^ (R & 7)) << 4);
  }

  // ---- gather pointer: row gi (global work index), step is of [ibeg, iend)
  int64_t gi = w0;
  int ibeg = 0, iend = 0, is = 0, icol = -1, icol_next = -1;
  const uint16_t *iK = nullptr, *iV = nullptr, *iQ = nullptr;
  auto open_issue_row = [&]() {
    if (gi < nrows) {
      int u0, fi;
      split_row(gi, p.n_fine_rows, r32, u0, fi);
      const int bh = p.fine_sample ? __ldg(p.fine_sample + fi) * p.H + u0 : u0;
      ibeg = __ldg(p.row_ptr + fi);
      iend = __ldg(p.row_ptr + fi + 1);
      const int bb = bh / p.H, hh = bh % p.H;
      iK = p.k.data + bb * p.k.sb + hh * p.k.sh + (lane % kLPR) * 8;
      iV = p.v.data + bb * p.v.sb + hh * p.v.sh + (lane % kLPR) * 8;
      const int rq = __ldg(p.fine_rows + fi) & 0x7fffffff;
      iQ = p.q.data + bb * p.q.sb + hh * p.q.sh + (int64_t)rq * p.q.sl + (lane % kLPR) * 8;
    }
    is = 0;
  };
  // issue the gathers of the pointer's step into ring stage `stg` and advance the pointer. Every
  // fine row has at least one entry (checked at plan upload, api.cu), so each row start issues
  // exactly the ceil(nnz / kS) steps the computing side consumes, the first carrying q. Indices
  // come from `icol` (lane i holds index ibeg + 32 w + i of window w; steps 2w, 2w + 1 use it); past
  // the row's end they are -1 and read row 0 (masked scores, p = 0).
  auto issue_step = [&](uint32_t stg) {
    if (gi < nrows) {   // warp-uniform
      const int nb0 = ibeg + kS * is;
      // column indices: a row's first window is loaded here; later windows of the row were
      // prefetched one step earlier (MG_FINE_IDX_AHEAD), so the index load latency overlaps a step
      if (kP == 2 || (is & 1) == 0)
        icol = (kIdxAhead && kP == 1 && is > 0) ? icol_next : (nb0 + lane < iend ? __ldg(p.cols + nb0 + lane) : -1);
      const int off = (kP == 2 ? 0 : (is & 1) * 16) + lane / kLPR;
      const uint32_t st = ring + stg * kStageBytes;
      // a row's first step also carries its q row (lanes 0 .. kLPR-1, 16 B each), so the computing
      // side never waits on a dependent q load at a row start
      if (is == 0 && lane < kLPR) cp_async16(st + kQOff + (lane << 4), iQ);
#pragma unroll
      for (int i = 0; i < kIters; ++i) {
        const uint32_t cc = (uint32_t)max(__shfl_sync(0xffffffffu, icol, off + kRPI * i), 0);
        cp_async16(st + doff[i], iK + cc * ksl);
        cp_async16(st + doff[i] + kS * kRowBytes, iV + cc * vsl);
      }
      if (kIdxAhead && kP == 1 && (is & 1) == 1 && nb0 + kS < iend)
        icol_next = nb0 + kS + lane < iend ? __ldg(p.cols + nb0 + kS + lane) : -1;
      if (nb0 + kS < iend) {
        ++is;
      } else {
        gi += W;
        open_issue_row();
      }
    }
    cp_async_commit();   // (an empty group past the end keeps the wait count uniform)
  };

  open_issue_row();
#pragma unroll
  for (int s = 0; s < kStages - 1; ++s) issue_step(s);
  uint32_t stage = 0, istage = kStages - 1;
  const uint32_t a_row = (lane & 7) * kRowBytes, b_row = a_row + 8 * kRowBytes;
  const uint32_t vr = (lane & 7) + 8 * (lane >> 4);

  for (int64_t gw = w0; gw < nrows; gw += W) {
    int u0, fi;
    split_row(gw, p.n_fine_rows, r32, u0, fi);
    const int bh = p.fine_sample ? __ldg(p.fine_sample + fi) * p.H + u0 : u0;   // (batched plans)
    const int enc = __ldg(p.fine_rows + fi);
    const int r = enc & 0x7fffffff;
    const bool final_out = enc < 0;
    const int bb = bh / p.H, hh = bh % p.H;
    // q as the SDDMM's A operand (every row = q): k16 step j uses dims 16j + 2t (+1), 16j + 8 + 2t (+1);
    // read from the q slot of the row's first ring stage
    uint32_t qa[kJ], qb[kJ];
    const int beg = __ldg(p.row_ptr + fi), end = __ldg(p.row_ptr + fi + 1);
    // padding (A18): columns >= n_b are masked; a row >= n_b is written as 0 if it is final (a row
    // with a coarse part is zeroed by the coarse kernel)
    const int nvalid = kPad ? max(__ldg(p.valid_len + bb), 0) : 0x7fffffff;
    const bool pad_row = kPad && r >= nvalid;

    float m = -INFINITY, l = 0.f;
    float acc[kJ][4];
#pragma unroll
    for (int j = 0; j < kJ; ++j)
#pragma unroll
      for (int e = 0; e < 4; ++e) acc[j][e] = 0.f;

    for (int base = beg; base < end; base += kS) {
      issue_step(istage);
      istage = istage == kStages - 1 ? 0 : istage + 1;
      cp_async_wait<kStages - 1>();
      __syncwarp();
      const uint32_t st = ring + stage * kStageBytes;
      stage = stage == kStages - 1 ? 0 : stage + 1;
      if (base == beg) {
#pragma unroll
        for (int j = 0; j < kJ; ++j) {
          asm volatile("ld.shared.u32 %0, [%1];" : "=r"(qa[j]) : "r"(st + kQOff + 32 * j + 4 * t));
          asm volatile("ld.shared.u32 %0, [%1];" : "=r"(qb[j]) : "r"(st + kQOff + 32 * j + 16 + 4 * t));
        }
      }

      // ---- SDDMM per pair: chunk A (rows 16pr + 0-7) and chunk B (rows 16pr + 8-15); lane holds
      // nnz 2t, 2t+1 of each chunk; two independent accumulators per chunk (dims 0-31, 32-63)
      float s[kP][4];
#pragma unroll
      for (int pr = 0; pr < kP; ++pr) {
        float sa[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
        float sb[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
#pragma unroll
        for (int h = 0; h < kD / 32; ++h) {   // dims 32h .. 32h + 31 = k16 steps 2h, 2h + 1
          uint32_t ka[4], kb[4];
          const uint32_t sw = ((uint32_t)(((lane >> 3) + 4 * h) ^ (lane & 7))) << 4;
          ldsm_x4(ka, st + pr * 16 * kRowBytes + a_row + sw);
          ldsm_x4(kb, st + pr * 16 * kRowBytes + b_row + sw);
          mma16816<kBF16>(sa[h & 1], qa[2 * h], qa[2 * h], qb[2 * h], qb[2 * h], ka[0], ka[1]);
          mma16816<kBF16>(sb[h & 1], qa[2 * h], qa[2 * h], qb[2 * h], qb[2 * h], kb[0], kb[1]);
          mma16816<kBF16>(sa[h & 1], qa[2 * h + 1], qa[2 * h + 1], qb[2 * h + 1], qb[2 * h + 1], ka[2], ka[3]);
          mma16816<kBF16>(sb[h & 1], qa[2 * h + 1], qa[2 * h + 1], qb[2 * h + 1], qb[2 * h + 1], kb[2], kb[3]);
        }
        // this lane's positions: nnz base + 16pr + {2t, 2t+1} (chunk A), + {8 + 2t, 9 + 2t} (chunk B)
        const int rem = end - base - 16 * pr - 2 * t;
        s[pr][0] = rem > 0 ? sa[0][0] + sa[1][0] : -INFINITY;
        s[pr][1] = rem > 1 ? sa[0][1] + sa[1][1] : -INFINITY;
        s[pr][2] = rem > 8 ? sb[0][0] + sb[1][0] : -INFINITY;
        s[pr][3] = rem > 9 ? sb[0][1] + sb[1][1] : -INFINITY;
        if (kPad) {   // padding: mask the columns at or beyond n_b (index loads hit L1)
          const int o4[4] = {0, 1, 8, 9};
#pragma unroll
          for (int i = 0; i < 4; ++i)
            if (rem > o4[i] && __ldg(p.cols + base + 16 * pr + 2 * t + o4[i]) >= nvalid) s[pr][i] = -INFINITY;
        }
      }
      // ---- online softmax over the step (warp-uniform max: lanes with equal t hold equal values)
      float mx = -INFINITY;
#pragma unroll
      for (int pr = 0; pr < kP; ++pr) mx = fmaxf(mx, fmaxf(fmaxf(s[pr][0], s[pr][1]), fmaxf(s[pr][2], s[pr][3])));
      mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 1));
      mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 2));
      // (mx = -inf only when padding masked the whole step: nothing to add)
      if (mx > m + thresh) {   // also taken on the first step (m = -inf) unless mx = -inf
        const float alpha = ex2((m - mx) * c);
        l *= alpha;
#pragma unroll
        for (int j = 0; j < kJ; ++j)
#pragma unroll
          for (int e = 0; e < 4; ++e) acc[j][e] *= alpha;
        m = mx;
      }
      const float nbias = m == -INFINITY ? 0.f : -m * c;   // (all-masked steps: every p is 0)
#pragma unroll
      for (int pr = 0; pr < kP; ++pr) {
        float pv[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          pv[i] = ex2(fmaf(s[pr][i], c, nbias));
          l += pv[i];
        }
        const uint32_t pb0 = pack2<kBF16>(pv[0], pv[1]), pb1 = pack2<kBF16>(pv[2], pv[3]);
        // ---- SpMM: O^T[dims 16j + g, 16j + g + 8] += V^T . p (A = V^T from ldmatrix.trans)
#pragma unroll
        for (int j = 0; j < kJ; ++j) {
          uint32_t a[4];
          const uint32_t ch = 2 * j + ((lane >> 3) & 1);
          const uint32_t row = vr + 16 * pr;
          ldsm_x4_t(a, st + kS * kRowBytes + row * kRowBytes + ((ch ^ (row & 7)) << 4));
          mma16816<kBF16>(acc[j], a[0], a[1], a[2], a[3], pb0, pb1);
        }
      }
      __syncwarp();   // every lane has read this stage before it is refilled
    }
    // ---- row epilogue. Row sum: lanes with the same g hold disjoint nnz subsets (t).
    l += __shfl_xor_sync(0xffffffffu, l, 1);
    l += __shfl_xor_sync(0xffffffffu, l, 2);
    // lane (g, t) owns output dims 16j + g and 16j + g + 8 of the blocks j = t (+ 4 at d = 128):
    // acc[j][0] and acc[j][2]
    constexpr int kOwn = kJ / 4;
    float v[kOwn][2];
    int dd[kOwn];
#pragma unroll
    for (int w = 0; w < kOwn; ++w) {
      v[w][0] = acc[4 * w][0];
      v[w][1] = acc[4 * w][2];
#pragma unroll
      for (int j = 1; j < 4; ++j)
        if (t == j) {
          v[w][0] = acc[4 * w + j][0];
          v[w][1] = acc[4 * w + j][2];
        }
      dd[w] = 16 * (4 * w + t) + g;
    }
    float inv = l > 0.f ? 1.f / l : 0.f;
    bool write_o = final_out;
    if (!final_out) {
      const size_t idx = (size_t)u0 * p.n_fine_rows + fi;
#pragma unroll
      for (int w = 0; w < kOwn; ++w) {
        __stcg(p.part_acc + idx * kD + dd[w], v[w][0]);
        __stcg(p.part_acc + idx * kD + dd[w] + 8, v[w][1]);
      }
      if (lane == 0) __stcg(p.part_ml + idx, make_float2(m, l));
      if (p.concurrent) {
        // concurrent coarse || fine: the side that finishes the row second merges (a-8)
        __threadfence();
        __syncwarp();
        int old = 0;
        if (lane == 0) old = atomicAdd(p.part_flags + idx, 1);
        old = __shfl_sync(0xffffffffu, old, 0);
        if (old & 1) {
          __threadfence();
          const float2 mlc = __ldcg(p.part_c_ml + idx);
          const float mt = fmaxf(m, mlc.x);
          const float mu = mt == -INFINITY ? 0.f : mt;
          const float af = ex2((m - mu) * c), ac = ex2((mlc.x - mu) * c);
          const float den = l * af + mlc.y * ac;
          inv = den > 0.f ? 1.f / den : 0.f;
#pragma unroll
          for (int w = 0; w < kOwn; ++w) {
            v[w][0] = v[w][0] * af + __ldcg(p.part_c_acc + idx * kD + dd[w]) * ac;
            v[w][1] = v[w][1] * af + __ldcg(p.part_c_acc + idx * kD + dd[w] + 8) * ac;
          }
          write_o = true;
        }
      }
    }
    if (pad_row) {
      write_o = final_out;   // rows with a coarse part are zeroed by the coarse kernel
#pragma unroll
      for (int w = 0; w < kOwn; ++w) v[w][0] = v[w][1] = 0.f;
    }
    if (write_o) {
      uint16_t* orow = p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)r * p.o.sl;
#pragma unroll
      for (int w = 0; w < kOwn; ++w) {
        const uint32_t pk = pack2<kBF16>(v[w][0] * inv, v[w][1] * inv);
        orow[dd[w]] = (uint16_t)(pk & 0xffffu);
        orow[dd[w] + 8] = (uint16_t)(pk >> 16);
      }
    }
  }
  cp_async_wait<0>();
}

// ---------------------------------------------------------------------------------------------
// Two heads per warp (d = 64, even head count): heads 2u and 2u + 1 of one batch element share the
// CSR row's column indices (the plan is shared across heads, A8), so one index window, one set of
// shuffles / gather offsets and one row's bookkeeping serve both heads, and each warp runs two
// independent SDDMM -> softmax -> SpMM chains (instruction-level parallelism for the mma.sync ->
// softmax -> mma.sync latency chain). Stage layout: [K_h0 kS rows][V_h0 kS rows][K_h1][V_h1][q_h0][q_h1].
#ifndef MG_FINE_MINB2
#define MG_FINE_MINB2 3
#endif
// SDDMM operand order of the two-head kernel: 1 = gathered K rows as the M operand (one 4-MMA chain
// per 16 nnz), 0 = q broadcast as the M operand (two chains, twice the MMAs)
#ifndef MG_FINE_SWAP
#define MG_FINE_SWAP 1
#endif
// p to the SpMM's B fragment by two movmatrix transposes (1) or two shuffles + byte permutes (0)
#ifndef MG_FINE_MOVM
#define MG_FINE_MOVM 1
#endif
// rows (head-pair rows) per dynamic claim of the two-head kernel: longer runs of one head pair's rows
// per warp (K/V locality, fewer claims); measured on C4: 2 / 4 / 8 / 16 / 32 / 64 ->
// 2.06 / 2.03 / 1.99 / 1.95 / 1.87 / 1.98 ms
#ifndef MG_FINE_CHUNK
#define MG_FINE_CHUNK 32
#endif
// lazy-rescale test by a warp vote before the max reduction (1) or after it (0)
#ifndef MG_FINE_VOTE
#define MG_FINE_VOTE 1
#endif
namespace {
constexpr int kHB = 2 * kS * 128;                 // K + V rows of one head in a stage
constexpr int kQOff2 = 2 * kHB;
constexpr int kStageBytes2 = kQOff2 + 2 * 128;
constexpr int kSmemBytes2 = kWarps * kStages * kStageBytes2;
}  // namespace

// kDyn (SM-split mode): the (head pair, CSR row) sequence of a warp comes from a global counter in
// chunks of kChunk consecutive rows instead of the static stride; the issue side claims, the compute
// side follows it one step behind (so it finds the chunk the issue side is in when it leaves its own).
template <bool kBF16, bool kPad, bool kDyn>
__global__ void __launch_bounds__(kWarps * 32, MG_FINE_MINB2) fine_mma2_kernel(const FineParams p) {
  constexpr int kChunk = MG_FINE_CHUNK;   // rows per dynamic claim
  constexpr int kD = 64, kRowBytes = 128, kLPR = 8, kRPI = 4, kJ = 4;
  extern __shared__ __align__(128) uint8_t fsm[];
  const int lane = threadIdx.x & 31;
  const int g = lane >> 2, t = lane & 3;
  const float c = p.scale_log2;
  const float thresh = 8.f / c;
  const int nhp = p.BH >> 1;                           // head pairs per fine row
  const int64_t nrows = (int64_t)nhp * p.n_fine_rows;
  const bool r32 = nrows <= (int64_t)0xffffffffLL;
  const int64_t W = (int64_t)gridDim.x * kWarps;
  const int64_t w0 = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5);
  const uint32_t ring = (uint32_t)__cvta_generic_to_shared(fsm) + (threadIdx.x >> 5) * (kStages * kStageBytes2);
  // row strides in bytes (fit 32 bits: (L - 1) * stride_l < 2^32, checked by the forward's validation)
  const uint32_t kslb = 2u * (uint32_t)p.k.sl, vslb = 2u * (uint32_t)p.v.sl;
  // head strides fit 32 bits (checked by the launcher)
  const uint32_t qsh = (uint32_t)p.q.sh;
  constexpr int kIters = kS / kRPI;
  uint32_t doff[kIters];
#pragma unroll
  for (int i = 0; i < kIters; ++i) {
    const int R = lane / kLPR + kRPI * i;
    doff[i] = R * kRowBytes + (((lane % kLPR) ^ (R & 7)) << 4);
  }

  // dynamic rows: claim a chunk (warp-uniform), -> its first row, or nrows when exhausted
  auto claim = [&]() -> int64_t {
    int c = 0;
    if (lane == 0) c = atomicAdd(p.row_ctr, 1);
    c = __shfl_sync(0xffffffffu, c, 0);
    const int64_t g = (int64_t)c * kChunk;
    return g < nrows ? g : nrows;
  };
  // Chunks claimed by the issue side for the compute side (the same warp, one step behind): the
  // issue side is never more than the next chunk (plus the final exhausted claim) ahead, so two
  // entries suffice.
  int64_t fq0 = nrows, fq1 = nrows;
  int fn = 0;
  // the row after g in the issue side's sequence
  auto next_row = [&](int64_t g) -> int64_t {
    if (!kDyn) return g + W;
    if ((g + 1) % kChunk != 0 && g + 1 < nrows) return g + 1;
    const int64_t c = claim();
    if (fn == 0) fq0 = c;
    else fq1 = c;
    ++fn;
    return c;
  };
  int64_t gi = kDyn ? claim() : w0;
  const int64_t g_first = gi;   // the compute side's first row (the prologue below may move gi on)
  int ibeg = 0, iend = 0, is = 0, icol = -1, icol_next = -1;
  // byte addresses of this lane's 16-byte chunk of row 0 of K / V of both heads of the issuing row: a
  // gathered row's address is one mad.wide.u32 (column x row stride + base) per copy
  uint64_t kb0 = 0, kb1 = 0, vb0 = 0, vb1 = 0;
  const uint16_t* iQ = nullptr;
  auto open_issue_row = [&]() {
    if (gi < nrows) {
      int u0, fi;
      split_row(gi, p.n_fine_rows, r32, u0, fi);
      const int bh = (p.fine_sample ? __ldg(p.fine_sample + fi) * p.H : 0) + 2 * u0;   // first head of the pair
      ibeg = __ldg(p.row_ptr + fi);
      iend = __ldg(p.row_ptr + fi + 1);
      const int bb = bh / p.H, hh = bh % p.H;
      kb0 = reinterpret_cast<uint64_t>(p.k.data + bb * p.k.sb + hh * p.k.sh + (lane % kLPR) * 8);
      vb0 = reinterpret_cast<uint64_t>(p.v.data + bb * p.v.sb + hh * p.v.sh + (lane % kLPR) * 8);
      kb1 = kb0 + 2 * (uint64_t)p.k.sh;
      vb1 = vb0 + 2 * (uint64_t)p.v.sh;
      const int rq = __ldg(p.fine_rows + fi) & 0x7fffffff;
      // lanes 0-7: q of the first head, lanes 8-15: q of the second
      iQ = p.q.data + bb * p.q.sb + hh * p.q.sh + (int64_t)rq * p.q.sl + (lane % kLPR) * 8 + ((lane >> 3) & 1) * qsh;
    }
    is = 0;
  };
  auto issue_step = [&](uint32_t stg) {
    if (gi < nrows) {
      const int nb0 = ibeg + kS * is;
      if ((is & 1) == 0) icol = is > 0 ? icol_next : (nb0 + lane < iend ? __ldg(p.cols + nb0 + lane) : -1);
      const int off = (is & 1) * 16 + lane / kLPR;
      const uint32_t st = ring + stg * kStageBytes2;
      if (is == 0 && lane < 2 * kLPR) cp_async16(st + kQOff2 + (lane << 4), iQ);
#pragma unroll
      for (int i = 0; i < kIters; ++i) {
        const uint32_t cc = (uint32_t)max(__shfl_sync(0xffffffffu, icol, off + kRPI * i), 0);
        cp_async16a(st + doff[i], mad_wide(cc, kslb, kb0));
        cp_async16a(st + doff[i] + kS * kRowBytes, mad_wide(cc, vslb, vb0));
        cp_async16a(st + kHB + doff[i], mad_wide(cc, kslb, kb1));
        cp_async16a(st + kHB + doff[i] + kS * kRowBytes, mad_wide(cc, vslb, vb1));
      }
      if ((is & 1) == 1 && nb0 + kS < iend) icol_next = nb0 + kS + lane < iend ? __ldg(p.cols + nb0 + kS + lane) : -1;
      if (nb0 + kS < iend) {
        ++is;
      } else {
        gi = next_row(gi);
        open_issue_row();
      }
    }
    cp_async_commit();
  };

  open_issue_row();
#pragma unroll
  for (int s0 = 0; s0 < kStages - 1; ++s0) issue_step(s0);
  uint32_t stage = 0, istage = kStages - 1;
  const uint32_t a_row = (lane & 7) * kRowBytes, b_row = a_row + 8 * kRowBytes;
  const uint32_t vr = (lane & 7) + 8 * (lane >> 4);

  auto next_compute_row = [&](int64_t g) -> int64_t {
    if (!kDyn) return g + W;
    if ((g + 1) % kChunk != 0 && g + 1 < nrows) return g + 1;
    const int64_t c = fn > 0 ? fq0 : nrows;
    fq0 = fq1;
    fn = fn > 0 ? fn - 1 : 0;
    return c;
  };
  for (int64_t gw = g_first; gw < nrows; gw = next_compute_row(gw)) {
    int u0, fi;
    split_row(gw, p.n_fine_rows, r32, u0, fi);
    const int bh = (p.fine_sample ? __ldg(p.fine_sample + fi) * p.H : 0) + 2 * u0;
    const int enc = __ldg(p.fine_rows + fi);
    const int r = enc & 0x7fffffff;
    const bool final_out = enc < 0;
    const int bb = bh / p.H, hh = bh % p.H;
    // q fragments as the SDDMM's A quads {q, q, q', q'} (rows g and g + 8 of the broadcast q: the
    // rows g + 8 of the product are never read), kept for the whole row so no step re-packs them
    uint32_t qq[2][kJ][4];
    const int beg = __ldg(p.row_ptr + fi), end = __ldg(p.row_ptr + fi + 1);
    const int nvalid = kPad ? max(__ldg(p.valid_len + bb), 0) : 0x7fffffff;
    const bool pad_row = kPad && r >= nvalid;

    float m[2] = {-INFINITY, -INFINITY}, l[2] = {0.f, 0.f};
    float acc[2][kJ][4];
#pragma unroll
    for (int hd = 0; hd < 2; ++hd)
#pragma unroll
      for (int j = 0; j < kJ; ++j)
#pragma unroll
        for (int e = 0; e < 4; ++e) acc[hd][j][e] = 0.f;

    for (int base = beg; base < end; base += kS) {
      issue_step(istage);
      istage = istage == kStages - 1 ? 0 : istage + 1;
      cp_async_wait<kStages - 1>();
      __syncwarp();
      const uint32_t st = ring + stage * kStageBytes2;
      stage = stage == kStages - 1 ? 0 : stage + 1;
      if (base == beg) {
#pragma unroll
        for (int hd = 0; hd < 2; ++hd)
#pragma unroll
          for (int j = 0; j < kJ; ++j) {
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(qq[hd][j][0]) : "r"(st + kQOff2 + hd * 128 + 32 * j + 4 * t));
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(qq[hd][j][2]) : "r"(st + kQOff2 + hd * 128 + 32 * j + 16 + 4 * t));
            qq[hd][j][1] = qq[hd][j][0];
            qq[hd][j][3] = qq[hd][j][2];
          }
      }
#if MG_FINE_SWAP
      // SDDMM with the gathered K rows as the M operand: s = K_c q for the step's 16 nnz in one
      // m16n8k16 chain over the 4 k16 steps (A = 16 K rows x 16 dims by ldmatrix, B = q broadcast to
      // the 8 columns), half the MMAs of the q-broadcast form; lane (g, t) gets the scores of nnz g
      // and g + 8 (the same in its 4 t-lanes).
      const int remg = end - base - g;
      float s[2][2];
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
        const uint32_t sk = st + hd * kHB;
        float sd[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int j = 0; j < kJ; ++j) {
          // matrices: rows 0-7 / 8-15 of chunk 2j, then of chunk 2j + 1 (lane -> row address)
          uint32_t ka[4];
          const uint32_t R = (lane & 7) + 8 * ((lane >> 3) & 1), ch = 2 * j + (lane >> 4);
          ldsm_x4(ka, sk + R * kRowBytes + ((ch ^ (R & 7)) << 4));
          mma16816<kBF16>(sd, ka[0], ka[1], ka[2], ka[3], qq[hd][j][0], qq[hd][j][2]);
        }
        s[hd][0] = sd[0];
        s[hd][1] = sd[2];
        if (end - base < kS) {   // the row's last, partial step (warp-uniform): entries past the row
          s[hd][0] = remg > 0 ? s[hd][0] : -INFINITY;
          s[hd][1] = remg > 8 ? s[hd][1] : -INFINITY;
        }
      }
      if (kPad) {   // padding: mask the columns at or beyond n_b (same columns for both heads)
        if (remg > 0 && __ldg(p.cols + base + g) >= nvalid) s[0][0] = s[1][0] = -INFINITY;
        if (remg > 8 && __ldg(p.cols + base + g + 8) >= nvalid) s[0][1] = s[1][1] = -INFINITY;
      }
      // lazy rescale: the step's row max is only reduced across the warp when some lane's scores
      // exceed the running max by the threshold (the same decision as comparing the full max, without
      // the three dependent shuffles on the common path)
      float mx[2];
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) mx[hd] = fmaxf(s[hd][0], s[hd][1]);
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
#if MG_FINE_VOTE
        if (__any_sync(0xffffffffu, mx[hd] > m[hd] + thresh)) {
#pragma unroll
          for (int o = 4; o < 32; o <<= 1) mx[hd] = fmaxf(mx[hd], __shfl_xor_sync(0xffffffffu, mx[hd], o));
#else
#pragma unroll
        for (int o = 4; o < 32; o <<= 1) mx[hd] = fmaxf(mx[hd], __shfl_xor_sync(0xffffffffu, mx[hd], o));
        if (mx[hd] > m[hd] + thresh) {
#endif
          const float alpha = ex2((m[hd] - mx[hd]) * c);
          l[hd] *= alpha;
#pragma unroll
          for (int j = 0; j < kJ; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[hd][j][e] *= alpha;
          m[hd] = mx[hd];
        }
      }
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
        const float nbias = m[hd] == -INFINITY ? 0.f : -m[hd] * c;
        const float p0 = ex2(fmaf(s[hd][0], c, nbias)), p1 = ex2(fmaf(s[hd][1], c, nbias));
        l[hd] += p0 + p1;
        // the SpMM's B fragment wants nnz 2t, 2t + 1 (b0) and 2t + 8, 2t + 9 (b1): from the lanes of
        // groups 2t and 2t + 1, which hold (p_2t, p_2t+8) and (p_2t+1, p_2t+9)
#if MG_FINE_MOVM
        // as 8 x 8 16-bit matrices M[g][c] = p_g (resp. p_g+8) for every column c, held one register
        // per lane (row g, columns 2t, 2t + 1): their transposes put p_2t, p_2t+1 (resp. p_2t+8,
        // p_2t+9) in lane (g, t), the SpMM's B fragment
        uint32_t pb0, pb1;
        asm("movmatrix.sync.aligned.m8n8.trans.b16 %0, %1;" : "=r"(pb0) : "r"(pack2<kBF16>(p0, p0)));
        asm("movmatrix.sync.aligned.m8n8.trans.b16 %0, %1;" : "=r"(pb1) : "r"(pack2<kBF16>(p1, p1)));
#else
        const uint32_t pk = pack2<kBF16>(p0, p1);
        const uint32_t x = __shfl_sync(0xffffffffu, pk, 8 * t), y = __shfl_sync(0xffffffffu, pk, 8 * t + 4);
        const uint32_t pb0 = __byte_perm(x, y, 0x5410), pb1 = __byte_perm(x, y, 0x7632);
#endif
        const uint32_t sv = st + hd * kHB + kS * kRowBytes;
#pragma unroll
        for (int j = 0; j < kJ; ++j) {
          uint32_t a[4];
          const uint32_t ch = 2 * j + ((lane >> 3) & 1);
          ldsm_x4_t(a, sv + vr * kRowBytes + ((ch ^ (vr & 7)) << 4));
          mma16816<kBF16>(acc[hd][j], a[0], a[1], a[2], a[3], pb0, pb1);
        }
      }
      __syncwarp();
#else
      const int rem = end - base - 2 * t;
      float s[2][4];
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
        const uint32_t sk = st + hd * kHB;
        // chunk A (nnz 0-7) and chunk B (nnz 8-15): one accumulator chain each over the 4 k16 steps
        float sa[4] = {0.f, 0.f, 0.f, 0.f}, sb[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          uint32_t ka[4], kb[4];
          const uint32_t sw = ((uint32_t)(((lane >> 3) + 4 * h) ^ (lane & 7))) << 4;
          ldsm_x4(ka, sk + a_row + sw);
          ldsm_x4(kb, sk + b_row + sw);
          const uint32_t(&q0)[4] = qq[hd][2 * h];
          const uint32_t(&q1)[4] = qq[hd][2 * h + 1];
          mma16816<kBF16>(sa, q0[0], q0[1], q0[2], q0[3], ka[0], ka[1]);
          mma16816<kBF16>(sb, q0[0], q0[1], q0[2], q0[3], kb[0], kb[1]);
          mma16816<kBF16>(sa, q1[0], q1[1], q1[2], q1[3], ka[2], ka[3]);
          mma16816<kBF16>(sb, q1[0], q1[1], q1[2], q1[3], kb[2], kb[3]);
        }
        s[hd][0] = sa[0];
        s[hd][1] = sa[1];
        s[hd][2] = sb[0];
        s[hd][3] = sb[1];
        if (end - base < kS) {   // the row's last, partial step (warp-uniform): entries past the row
          s[hd][0] = rem > 0 ? s[hd][0] : -INFINITY;
          s[hd][1] = rem > 1 ? s[hd][1] : -INFINITY;
          s[hd][2] = rem > 8 ? s[hd][2] : -INFINITY;
          s[hd][3] = rem > 9 ? s[hd][3] : -INFINITY;
        }
      }
      if (kPad) {   // padding: mask the columns at or beyond n_b (same columns for both heads)
        const int o4[4] = {0, 1, 8, 9};
#pragma unroll
        for (int i = 0; i < 4; ++i)
          if (rem > o4[i] && __ldg(p.cols + base + 2 * t + o4[i]) >= nvalid) s[0][i] = s[1][i] = -INFINITY;
      }
      float mx[2];
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) mx[hd] = fmaxf(fmaxf(s[hd][0], s[hd][1]), fmaxf(s[hd][2], s[hd][3]));
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) mx[hd] = fmaxf(mx[hd], __shfl_xor_sync(0xffffffffu, mx[hd], 1));
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) mx[hd] = fmaxf(mx[hd], __shfl_xor_sync(0xffffffffu, mx[hd], 2));
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
        if (mx[hd] > m[hd] + thresh) {
          const float alpha = ex2((m[hd] - mx[hd]) * c);
          l[hd] *= alpha;
#pragma unroll
          for (int j = 0; j < kJ; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[hd][j][e] *= alpha;
          m[hd] = mx[hd];
        }
      }
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
        const float nbias = m[hd] == -INFINITY ? 0.f : -m[hd] * c;
        float pv[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          pv[i] = ex2(fmaf(s[hd][i], c, nbias));
          l[hd] += pv[i];
        }
        const uint32_t pb0 = pack2<kBF16>(pv[0], pv[1]), pb1 = pack2<kBF16>(pv[2], pv[3]);
        const uint32_t sv = st + hd * kHB + kS * kRowBytes;
#pragma unroll
        for (int j = 0; j < kJ; ++j) {
          uint32_t a[4];
          const uint32_t ch = 2 * j + ((lane >> 3) & 1);
          ldsm_x4_t(a, sv + vr * kRowBytes + ((ch ^ (vr & 7)) << 4));
          mma16816<kBF16>(acc[hd][j], a[0], a[1], a[2], a[3], pb0, pb1);
        }
      }
      __syncwarp();
#endif
    }
    // ---- row epilogue of both heads
#pragma unroll
    for (int hd = 0; hd < 2; ++hd) {
      float lh = l[hd];
#if MG_FINE_SWAP
      // (each group g holds the sums of its own nnz, the same in its four t-lanes)
      lh += __shfl_xor_sync(0xffffffffu, lh, 4);
      lh += __shfl_xor_sync(0xffffffffu, lh, 8);
      lh += __shfl_xor_sync(0xffffffffu, lh, 16);
#else
      lh += __shfl_xor_sync(0xffffffffu, lh, 1);
      lh += __shfl_xor_sync(0xffffffffu, lh, 2);
#endif
      float v0 = acc[hd][0][0], v1 = acc[hd][0][2];
#pragma unroll
      for (int j = 1; j < 4; ++j)
        if (t == j) {
          v0 = acc[hd][j][0];
          v1 = acc[hd][j][2];
        }
      const int d0 = 16 * t + g;
      float inv = lh > 0.f ? 1.f / lh : 0.f;
      bool write_o = final_out;
      if (!final_out) {
        const size_t idx = (size_t)(2 * u0 + hd) * p.n_fine_rows + fi;
        __stcg(p.part_acc + idx * kD + d0, v0);
        __stcg(p.part_acc + idx * kD + d0 + 8, v1);
        if (lane == 0) __stcg(p.part_ml + idx, make_float2(m[hd], lh));
        if (p.concurrent) {
          __threadfence();
          __syncwarp();
          int old = 0;
          if (lane == 0) old = atomicAdd(p.part_flags + idx, 1);
          old = __shfl_sync(0xffffffffu, old, 0);
          if (old & 1) {
            __threadfence();
            const float2 mlc = __ldcg(p.part_c_ml + idx);
            const float mt = fmaxf(m[hd], mlc.x);
            const float mu = mt == -INFINITY ? 0.f : mt;
            const float af = ex2((m[hd] - mu) * c), ac = ex2((mlc.x - mu) * c);
            const float den = lh * af + mlc.y * ac;
            inv = den > 0.f ? 1.f / den : 0.f;
            v0 = v0 * af + __ldcg(p.part_c_acc + idx * kD + d0) * ac;
            v1 = v1 * af + __ldcg(p.part_c_acc + idx * kD + d0 + 8) * ac;
            write_o = true;
          }
        }
      }
      if (pad_row) {
        write_o = final_out;
        v0 = v1 = 0.f;
      }
      if (write_o) {
        uint16_t* orow = p.o.data + bb * p.o.sb + (hh + hd) * p.o.sh + (int64_t)r * p.o.sl;
        const uint32_t pk = pack2<kBF16>(v0 * inv, v1 * inv);
        orow[d0] = (uint16_t)(pk & 0xffffu);
        orow[d0 + 8] = (uint16_t)(pk >> 16);
      }
    }
  }
  cp_async_wait<0>();
  if (kDyn) {
    // the last block to finish resets the row counter for the next launch
    __syncthreads();
    if (threadIdx.x == 0) {
      __threadfence();
      if (atomicAdd(p.row_ctr + 1, 1) == (int)gridDim.x - 1) {
        atomicExch(p.row_ctr, 0);
        atomicExch(p.row_ctr + 1, 0);
      }
    }
  }
}

// ---------------------------------------------------------------------------------------------
// Two heads per warp with TMA row gathers (tile::gather4): per step, lanes 0-15 each issue one
// gather of 4 rows (K and V of both heads, 16 rows each) and, at a row start, lane 16 gathers the
// two q rows, all completing on the stage's mbarrier; one warp instruction replaces the 16 cp.async
// per lane of fine_mma2_kernel. Stage (1024-byte aligned, SWIZZLE_128B = the ring's XOR layout):
// [K_h0 16 rows][V_h0][K_h1][V_h1][q_h0, q_h1, 2 zero rows] = 8.5 KB, padded to 9 KB.
namespace {
constexpr int kStageBytesT = 9216;
constexpr int kQOffT = 4 * kS * 128;
constexpr int kSmemBytesT = 1024 + kWarps * kStages * kStageBytesT + kWarps * kStages * 8;
}  // namespace

template <bool kBF16, bool kPad>
__global__ void __launch_bounds__(kWarps * 32, MG_FINE_MINB2)
    fine_tma2_kernel(const __grid_constant__ CUtensorMap tmq2, const __grid_constant__ CUtensorMap tmk2,
                     const __grid_constant__ CUtensorMap tmv2, const FineParams p) {
  constexpr int kD = 64, kRowBytes = 128, kJ = 4;
  extern __shared__ __align__(128) uint8_t fsm[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int g = lane >> 2, t = lane & 3;
  const float c = p.scale_log2;
  const float thresh = 8.f / c;
  const int nhp = p.BH >> 1;
  const int64_t nrows = (int64_t)nhp * p.n_fine_rows;
  const bool r32 = nrows <= (int64_t)0xffffffffLL;
  const int64_t W = (int64_t)gridDim.x * kWarps;
  const int64_t w0 = (int64_t)blockIdx.x * kWarps + wid;
  const uint32_t base = ((uint32_t)__cvta_generic_to_shared(fsm) + 1023u) & ~1023u;
  const uint32_t ring = base + wid * (kStages * kStageBytesT);
  const uint32_t bars = base + kWarps * kStages * kStageBytesT + wid * (kStages * 8);
  if (lane == 0) {
    for (int s0 = 0; s0 < kStages; ++s0) mbar_init(bars + 8 * s0, 1);
    fence_barrier_init();
  }
  __syncwarp();
  if (threadIdx.x == 0) {
    prefetch_tmap(&tmk2);
    prefetch_tmap(&tmv2);
    prefetch_tmap(&tmq2);
  }
  const uint64_t pol = policy_evict_last();
  // lane j < 16 gathers rows 4 (j % 4) .. + 3 of the step into block j / 4: K_h0, V_h0, K_h1, V_h1
  const int gblk = (lane >> 2) & 3, gq = lane & 3;
  const CUtensorMap* gmap = (gblk & 1) ? &tmv2 : &tmk2;
  const int64_t rstep = (gblk & 1) ? p.rv.z : p.rk.z;

  int64_t gi = w0;
  int ibeg = 0, iend = 0, is = 0, icol = -1, icol_next = -1;
  int64_t grow0 = 0;          // this lane's gather: row of (b, head of its block, column 0)
  int qrow0 = 0, qrow1 = 0;   // the row's q rows in the Q view
  auto open_issue_row = [&]() {
    if (gi < nrows) {
      int u0, fi;
      split_row(gi, p.n_fine_rows, r32, u0, fi);
      const int bh = (p.fine_sample ? __ldg(p.fine_sample + fi) * p.H : 0) + 2 * u0;
      ibeg = __ldg(p.row_ptr + fi);
      iend = __ldg(p.row_ptr + fi + 1);
      const int bb = bh / p.H, hh = bh % p.H + (gblk >> 1);
      grow0 = (gblk & 1) ? bb * p.rv.x + hh * p.rv.y : bb * p.rk.x + hh * p.rk.y;
      const int rq = __ldg(p.fine_rows + fi) & 0x7fffffff;
      const int hq = bh % p.H;
      qrow0 = (int)(bb * p.rq.x + hq * p.rq.y + (int64_t)rq * p.rq.z);
      qrow1 = (int)(qrow0 + p.rq.y);
    }
    is = 0;
  };
  uint32_t phase = 0;   // bit s: parity of the next completion of stage s
  auto issue_step = [&](uint32_t stg) {
    if (gi < nrows) {
      const int nb0 = ibeg + kS * is;
      if ((is & 1) == 0) icol = is > 0 ? icol_next : (nb0 + lane < iend ? __ldg(p.cols + nb0 + lane) : -1);
      const int off = (is & 1) * 16 + 4 * gq;
      int4 cols;
      cols.x = __shfl_sync(0xffffffffu, icol, off);
      cols.y = __shfl_sync(0xffffffffu, icol, off + 1);
      cols.z = __shfl_sync(0xffffffffu, icol, off + 2);
      cols.w = __shfl_sync(0xffffffffu, icol, off + 3);
      const uint32_t st = ring + stg * kStageBytesT, bar = bars + 8 * stg;
      // (the stage was last read by this warp's ldmatrix: order those generic reads before the
      // async-proxy writes)
      fence_proxy_async_smem();
      if (lane == 0) mbar_arrive_expect_tx(bar, 4 * kS * kRowBytes + (is == 0 ? 512u : 0u));
      __syncwarp();
      if (lane < 16) gather4(st + gblk * (kS * kRowBytes) + gq * 512, gmap, bar, row_coords(cols, grow0, rstep), pol);
      if (is == 0 && lane == 16) gather4(st + kQOffT, &tmq2, bar, make_int4(qrow0, qrow1, -1, -1), pol);
      if ((is & 1) == 1 && nb0 + kS < iend) icol_next = nb0 + kS + lane < iend ? __ldg(p.cols + nb0 + kS + lane) : -1;
      if (nb0 + kS < iend) {
        ++is;
      } else {
        gi += W;
        open_issue_row();
      }
    }
  };

  open_issue_row();
#pragma unroll
  for (int s0 = 0; s0 < kStages - 1; ++s0) issue_step(s0);
  uint32_t stage = 0, istage = kStages - 1;
  const uint32_t a_row = (lane & 7) * kRowBytes, b_row = a_row + 8 * kRowBytes;
  const uint32_t vr = (lane & 7) + 8 * (lane >> 4);

  for (int64_t gw = w0; gw < nrows; gw += W) {
    int u0, fi;
    split_row(gw, p.n_fine_rows, r32, u0, fi);
    const int bh = (p.fine_sample ? __ldg(p.fine_sample + fi) * p.H : 0) + 2 * u0;
    const int enc = __ldg(p.fine_rows + fi);
    const int r = enc & 0x7fffffff;
    const bool final_out = enc < 0;
    const int bb = bh / p.H, hh = bh % p.H;
    uint32_t qa[2][kJ], qb[2][kJ];
    const int beg = __ldg(p.row_ptr + fi), end = __ldg(p.row_ptr + fi + 1);
    const int nvalid = kPad ? max(__ldg(p.valid_len + bb), 0) : 0x7fffffff;
    const bool pad_row = kPad && r >= nvalid;

    float m[2] = {-INFINITY, -INFINITY}, l[2] = {0.f, 0.f};
    float acc[2][kJ][4];
#pragma unroll
    for (int hd = 0; hd < 2; ++hd)
#pragma unroll
      for (int j = 0; j < kJ; ++j)
#pragma unroll
        for (int e = 0; e < 4; ++e) acc[hd][j][e] = 0.f;

    for (int base_i = beg; base_i < end; base_i += kS) {
      issue_step(istage);
      istage = istage == kStages - 1 ? 0 : istage + 1;
      mbar_wait(bars + 8 * stage, (phase >> stage) & 1);
      phase ^= 1u << stage;
      const uint32_t st = ring + stage * kStageBytesT;
      stage = stage == kStages - 1 ? 0 : stage + 1;
      if (base_i == beg) {
#pragma unroll
        for (int hd = 0; hd < 2; ++hd)
#pragma unroll
          for (int j = 0; j < kJ; ++j) {
            // the q rows' 16-byte chunks are swizzled like every row of the stage (row 0 / 1)
            const uint32_t qrow = st + kQOffT + hd * 128;
            const uint32_t ch0 = (2 * j) ^ hd, ch1 = (2 * j + 1) ^ hd;
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(qa[hd][j]) : "r"(qrow + (ch0 << 4) + 4 * t));
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(qb[hd][j]) : "r"(qrow + (ch1 << 4) + 4 * t));
          }
      }
      const int rem = end - base_i - 2 * t;
      float s[2][4];
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
        const uint32_t sk = st + hd * kHB;
        float sa[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
        float sb[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          uint32_t ka[4], kb[4];
          const uint32_t sw = ((uint32_t)(((lane >> 3) + 4 * h) ^ (lane & 7))) << 4;
          ldsm_x4(ka, sk + a_row + sw);
          ldsm_x4(kb, sk + b_row + sw);
          mma16816<kBF16>(sa[h], qa[hd][2 * h], qa[hd][2 * h], qb[hd][2 * h], qb[hd][2 * h], ka[0], ka[1]);
          mma16816<kBF16>(sb[h], qa[hd][2 * h], qa[hd][2 * h], qb[hd][2 * h], qb[hd][2 * h], kb[0], kb[1]);
          mma16816<kBF16>(sa[h], qa[hd][2 * h + 1], qa[hd][2 * h + 1], qb[hd][2 * h + 1], qb[hd][2 * h + 1], ka[2], ka[3]);
          mma16816<kBF16>(sb[h], qa[hd][2 * h + 1], qa[hd][2 * h + 1], qb[hd][2 * h + 1], qb[hd][2 * h + 1], kb[2], kb[3]);
        }
        s[hd][0] = rem > 0 ? sa[0][0] + sa[1][0] : -INFINITY;
        s[hd][1] = rem > 1 ? sa[0][1] + sa[1][1] : -INFINITY;
        s[hd][2] = rem > 8 ? sb[0][0] + sb[1][0] : -INFINITY;
        s[hd][3] = rem > 9 ? sb[0][1] + sb[1][1] : -INFINITY;
      }
      if (kPad) {
        const int o4[4] = {0, 1, 8, 9};
#pragma unroll
        for (int i = 0; i < 4; ++i)
          if (rem > o4[i] && __ldg(p.cols + base_i + 2 * t + o4[i]) >= nvalid) s[0][i] = s[1][i] = -INFINITY;
      }
      float mx[2];
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) mx[hd] = fmaxf(fmaxf(s[hd][0], s[hd][1]), fmaxf(s[hd][2], s[hd][3]));
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) mx[hd] = fmaxf(mx[hd], __shfl_xor_sync(0xffffffffu, mx[hd], 1));
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) mx[hd] = fmaxf(mx[hd], __shfl_xor_sync(0xffffffffu, mx[hd], 2));
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
        if (mx[hd] > m[hd] + thresh) {
          const float alpha = ex2((m[hd] - mx[hd]) * c);
          l[hd] *= alpha;
#pragma unroll
          for (int j = 0; j < kJ; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[hd][j][e] *= alpha;
          m[hd] = mx[hd];
        }
      }
#pragma unroll
      for (int hd = 0; hd < 2; ++hd) {
        const float nbias = m[hd] == -INFINITY ? 0.f : -m[hd] * c;
        float pv[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          pv[i] = ex2(fmaf(s[hd][i], c, nbias));
          l[hd] += pv[i];
        }
        const uint32_t pb0 = pack2<kBF16>(pv[0], pv[1]), pb1 = pack2<kBF16>(pv[2], pv[3]);
        const uint32_t sv = st + hd * kHB + kS * kRowBytes;
#pragma unroll
        for (int j = 0; j < kJ; ++j) {
          uint32_t a[4];
          const uint32_t ch = 2 * j + ((lane >> 3) & 1);
          ldsm_x4_t(a, sv + vr * kRowBytes + ((ch ^ (vr & 7)) << 4));
          mma16816<kBF16>(acc[hd][j], a[0], a[1], a[2], a[3], pb0, pb1);
        }
      }
      __syncwarp();
    }
#pragma unroll
    for (int hd = 0; hd < 2; ++hd) {
      float lh = l[hd];
      lh += __shfl_xor_sync(0xffffffffu, lh, 1);
      lh += __shfl_xor_sync(0xffffffffu, lh, 2);
      float v0 = acc[hd][0][0], v1 = acc[hd][0][2];
#pragma unroll
      for (int j = 1; j < 4; ++j)
        if (t == j) {
          v0 = acc[hd][j][0];
          v1 = acc[hd][j][2];
        }
      const int d0 = 16 * t + g;
      float inv = lh > 0.f ? 1.f / lh : 0.f;
      bool write_o = final_out;
      if (!final_out) {
        const size_t idx = (size_t)(2 * u0 + hd) * p.n_fine_rows + fi;
        __stcg(p.part_acc + idx * kD + d0, v0);
        __stcg(p.part_acc + idx * kD + d0 + 8, v1);
        if (lane == 0) __stcg(p.part_ml + idx, make_float2(m[hd], lh));
        if (p.concurrent) {
          __threadfence();
          __syncwarp();
          int old = 0;
          if (lane == 0) old = atomicAdd(p.part_flags + idx, 1);
          old = __shfl_sync(0xffffffffu, old, 0);
          if (old & 1) {
            __threadfence();
            const float2 mlc = __ldcg(p.part_c_ml + idx);
            const float mt = fmaxf(m[hd], mlc.x);
            const float mu = mt == -INFINITY ? 0.f : mt;
            const float af = ex2((m[hd] - mu) * c), ac = ex2((mlc.x - mu) * c);
            const float den = lh * af + mlc.y * ac;
            inv = den > 0.f ? 1.f / den : 0.f;
            v0 = v0 * af + __ldcg(p.part_c_acc + idx * kD + d0) * ac;
            v1 = v1 * af + __ldcg(p.part_c_acc + idx * kD + d0 + 8) * ac;
            write_o = true;
          }
        }
      }
      if (pad_row) {
        write_o = final_out;
        v0 = v1 = 0.f;
      }
      if (write_o) {
        uint16_t* orow = p.o.data + bb * p.o.sb + (hh + hd) * p.o.sh + (int64_t)r * p.o.sl;
        const uint32_t pk = pack2<kBF16>(v0 * inv, v1 * inv);
        orow[d0] = (uint16_t)(pk & 0xffffu);
        orow[d0 + 8] = (uint16_t)(pk >> 16);
      }
    }
  }
}

cudaError_t launch_fine_tma2(const FineParams& p, const CUtensorMap& tmq2, const CUtensorMap& tmk2,
                             const CUtensorMap& tmv2, bool bf16, int sms, cudaStream_t stream) {
  const int64_t units = (int64_t)(p.BH / 2) * p.n_fine_rows;
  if (units == 0) return cudaSuccess;
  using K = void (*)(const CUtensorMap, const CUtensorMap, const CUtensorMap, const FineParams);
  static const K table[4] = {fine_tma2_kernel<false, false>, fine_tma2_kernel<false, true>,
                             fine_tma2_kernel<true, false>, fine_tma2_kernel<true, true>};
  const K kern = table[(bf16 ? 2 : 0) + (p.valid_len ? 1 : 0)];
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytesT);
  if (e != cudaSuccess) return e;
  static std::mutex mu;
  static std::map<std::pair<int, int>, int> per_sm;
  const int vi = (bf16 ? 2 : 0) + (p.valid_len ? 1 : 0);
  int dev = 0, n = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  {
    std::lock_guard<std::mutex> lk(mu);
    auto it = per_sm.find({dev, vi});
    if (it == per_sm.end()) {
      if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, kWarps * 32, kSmemBytesT)) != cudaSuccess)
        return e;
      it = per_sm.emplace(std::make_pair(dev, vi), std::max(n, 1)).first;
    }
    n = it->second;
  }
  const int64_t blocks = std::min<int64_t>((units + kWarps - 1) / kWarps, (int64_t)n * std::max(sms, 1));
  kern<<<(unsigned)blocks, kWarps * 32, kSmemBytesT, stream>>>(tmq2, tmk2, tmv2, p);
  return cudaGetLastError();
}

cudaError_t launch_fine_mma(const FineParams& p, bool bf16, int sms, cudaStream_t stream) {
  const int64_t warps = (int64_t)p.BH * p.n_fine_rows;
  if (warps == 0) return cudaSuccess;
  using K = void (*)(const FineParams);
  static const K table[8] = {fine_mma_kernel<false, false, 64>, fine_mma_kernel<false, true, 64>,
                             fine_mma_kernel<true, false, 64>,  fine_mma_kernel<true, true, 64>,
                             fine_mma_kernel<false, false, 128>, fine_mma_kernel<false, true, 128>,
                             fine_mma_kernel<true, false, 128>,  fine_mma_kernel<true, true, 128>};
  if (p.d != 64 && p.d != 128) return cudaErrorInvalidValue;
  // two heads per warp when the heads pair up within a batch element and the head strides fit the
  // kernel's 32-bit offsets (MG_FINE_HEADS2=0 in the environment selects one head per warp, A/B)
  static const bool no_hp2 = [] {
    const char* e = std::getenv("MG_FINE_HEADS2");
    return e && e[0] == '0';
  }();
  const bool hp2 = !no_hp2 && p.d == 64 && (p.H % 2) == 0 && p.k.sh < (int64_t(1) << 31) &&
                   p.v.sh < (int64_t(1) << 31) && p.q.sh < (int64_t(1) << 31);
  static const K table2[8] = {fine_mma2_kernel<false, false, false>, fine_mma2_kernel<false, true, false>,
                              fine_mma2_kernel<true, false, false>,  fine_mma2_kernel<true, true, false>,
                              fine_mma2_kernel<false, false, true>,  fine_mma2_kernel<false, true, true>,
                              fine_mma2_kernel<true, false, true>,   fine_mma2_kernel<true, true, true>};
  const int vi = hp2 ? 8 + (bf16 ? 2 : 0) + (p.valid_len ? 1 : 0) : (p.d == 128 ? 4 : 0) + (bf16 ? 2 : 0) + (p.valid_len ? 1 : 0);
  // dynamic rows (SM-split mode) exist in the two-head kernel only; the others keep the static order
  const K kern = hp2 ? table2[vi - 8 + (p.row_ctr ? 4 : 0)] : table[vi];
  const int kSmemBytes = hp2 ? kSmemBytes2 : (p.d == 128 ? FCfg<128>::kSmemBytes : FCfg<64>::kSmemBytes);
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytes);
  if (e != cudaSuccess) return e;
  // persistent grid: every resident block slot of `sms` SMs (the plan's SM count, or its num_sms
  // test override), or fewer if the rows are few. Resident blocks per SM of each variant, per
  // device, computed once under a lock (launches may come from several host threads).
  static std::mutex mu;
  static std::map<std::pair<int, int>, int> per_sm;
  int dev = 0, n = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  {
    std::lock_guard<std::mutex> lk(mu);
    const int key = vi + (hp2 && p.row_ctr ? 100 : 0);
    auto it = per_sm.find({dev, key});
    if (it == per_sm.end()) {
      if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, kWarps * 32, kSmemBytes)) != cudaSuccess)
        return e;
      it = per_sm.emplace(std::make_pair(dev, key), std::max(n, 1)).first;
    }
    n = it->second;
  }
  const int64_t units = hp2 ? warps / 2 : warps;
  const int64_t blocks = std::min<int64_t>((units + kWarps - 1) / kWarps, (int64_t)n * std::max(sms, 1));
  kern<<<(unsigned)blocks, kWarps * 32, kSmemBytes, stream>>>(p);
  return cudaGetLastError();
}

}  // namespace mg
