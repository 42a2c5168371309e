// Staged ("paper dataflow") forward: every step of the method as its own kernel, with the scores
// S and the probabilities P materialised in the plan's formats (SURVEY §8(a) staged mode, §8(f)
// f-4). This is the dataflow of the paper's Fig. 5 / §3: coarse and fine SDDMM,
// the compound SpSoftmax that sweeps the row's non-zero blocks and then its non-zero elements
// (three sweeps: max, sum, normalise), and coarse and fine SpMM, with the
// global rows as a separate dense part. The fused kernels (coarse_pp_sm100.cu,
// fine_mma.cu) compute the same result without writing S and P; this path exists so that each step
// can be checked against the oracle's intermediates (O-7) and as an ablation of the fused design.
//
// Formats (per batch*head unit bh, all row-major):
//   S_t [BH][n_tiles][128][128] fp32, -inf where the canonical tile bit is 0 (BSR order of the plan)
//   S_f [BH][nnz_csr] fp32 (canonical CSR order)          S_g [BH][n_global][Lpad] fp32, -inf at c >= L
//   P_t, P_f, P_g: the same shapes in the operand dtype (bf16 / fp16, RNE)
//   O_f [BH][L][64] fp32: the CSR SpMM's contribution (rows with CSR nnz only)
// Lpad = 128 * ceil(L / 128). The contractions run on the warp-level tensor cores (mma.sync
// m16n8k16, fp32 accumulation): these kernels are bounded by the HBM traffic of S and P, not by
// the MMA rate.
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "kernels.cuh"
#include "sm100_ptx.cuh"

namespace mg {

using namespace ptx;

namespace {

constexpr int kT = 128;   // tile edge

template <bool kBF16>
__device__ __forceinline__ void mma16816(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  if (kBF16)
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
  else
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
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
__device__ __forceinline__ void sts16(uint32_t a, int4 v) {
  asm volatile("st.shared.v4.s32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}

template <bool kBF16>
__device__ __forceinline__ uint16_t to16(float x) {
  if (kBF16) return __bfloat16_as_ushort(__float2bfloat16_rn(x));
  return __half_as_ushort(__float2half_rn(x));
}
template <bool kBF16>
__device__ __forceinline__ float from16(uint16_t x) {
  if (kBF16) return __uint_as_float((uint32_t)x << 16);
  return __half2float(__ushort_as_half(x));
}
template <bool kBF16>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  return kBF16 ? pack_bf16(lo, hi) : pack_f16(lo, hi);
}

// swizzled 16-byte chunk address in a tile of `cpr` chunks per row (cpr = 8 or 16)
__device__ __forceinline__ uint32_t swz(uint32_t base, int row, int chunk, int cpr) {
  return base + (uint32_t)(row * cpr + (chunk ^ (row & 7))) * 16u;
}

// Load 128 rows x 64 16-bit elements (row i from `src(i)`, nullptr -> zeros) into a swizzled
// 8-chunks-per-row tile; all 256 threads.
template <class F>
__device__ __forceinline__ void load_rows64(uint32_t dst, F src) {
  for (int e = threadIdx.x; e < kT * 8; e += blockDim.x) {
    const int row = e >> 3, ch = e & 7;
    const uint16_t* s = src(row);
    const int4 v = s ? ld_nc_v4(s + ch * 8) : make_int4(0, 0, 0, 0);
    sts16(swz(dst, row, ch, 8), v);
  }
}

}  // namespace

// ------------------------------------------------------------------------------------------------
// a-2 / a-4 (SDDMM part): one 128 x 128 score tile per block. blockIdx.x < n_tiles: BSR tile t
// (rows of its row block, columns of its column block, canonical bitmask); otherwise a
// (global-row chunk, column block) tile of the dense-row part. 8 warps x 16 rows.
template <bool kBF16>
__global__ void __launch_bounds__(256) staged_sddmm_tiles(const StagedParams p) {
  __shared__ __align__(128) uint8_t sm[2 * kT * 128];
  const uint32_t sQ = smem_u32(sm), sK = sQ + kT * 128;
  const int bh = blockIdx.y, bb = bh / p.H, hh = bh % p.H;
  const int x = blockIdx.x;
  int rowI = 0, J = 0, gchunk = -1, nrows = kT;
  const uint64_t* mask = nullptr;
  if (x < p.n_tiles) {
    rowI = __ldg(p.tile_row + x) * kT;
    J = __ldg(p.bsr_col + x);
    mask = p.tile_masks + (size_t)x * (kT * 2);
  } else {
    gchunk = (x - p.n_tiles) / p.nb;
    J = (x - p.n_tiles) % p.nb;
    nrows = min(kT, p.n_global - gchunk * kT);
  }
  const uint16_t* Qb = p.q.data + bb * p.q.sb + hh * p.q.sh;
  const uint16_t* Kb = p.k.data + bb * p.k.sb + hh * p.k.sh;
  load_rows64(sQ, [&](int i) -> const uint16_t* {
    if (gchunk < 0) {
      const int64_t r = rowI + i;
      return r < p.L ? Qb + r * p.q.sl : nullptr;
    }
    return i < nrows ? Qb + (int64_t)__ldg(p.global_rows + gchunk * kT + i) * p.q.sl : nullptr;
  });
  load_rows64(sK, [&](int j) -> const uint16_t* {
    const int64_t c = (int64_t)J * kT + j;
    return c < p.L ? Kb + c * p.k.sl : nullptr;
  });
  __syncthreads();

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int r0 = warp * 16;
  uint32_t a[4][4];   // Q fragments of the warp's 16 rows, 4 k16 steps
#pragma unroll
  for (int kk = 0; kk < 4; ++kk)
    ldsm_x4(a[kk], swz(sQ, r0 + (lane & 7) + 8 * ((lane >> 3) & 1), 2 * kk + (lane >> 4), 8));
  // validity of this lane's rows r0 + g and r0 + g + 8: tile bitmask words, or c < L (dense rows)
  uint64_t mw[2][2] = {{~0ull, ~0ull}, {~0ull, ~0ull}};
  if (mask) {
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      mw[h][0] = __ldg(mask + (r0 + g + 8 * h) * 2);
      mw[h][1] = __ldg(mask + (r0 + g + 8 * h) * 2 + 1);
    }
  }
  const float sf = p.sf;
  for (int n8 = 0; n8 < 16; ++n8) {
    float d[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      uint32_t b[4];
      ldsm_x4(b, swz(sK, n8 * 8 + (lane & 7), 4 * h + (lane >> 3), 8));
      mma16816<kBF16>(d, a[2 * h], b[0], b[1]);
      mma16816<kBF16>(d, a[2 * h + 1], b[2], b[3]);
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int i = r0 + g + 8 * h;
      const int j = n8 * 8 + 2 * t;
      const int64_t cg = (int64_t)J * kT + j;
      bool v0, v1;
      if (mask) {
        const uint64_t w = (j >> 6) ? mw[h][1] : mw[h][0];
        v0 = (w >> (j & 63)) & 1;
        v1 = (w >> ((j + 1) & 63)) & 1;
      } else {
        v0 = cg < p.L;
        v1 = cg + 1 < p.L;
      }
      const float2 o = make_float2(v0 ? d[2 * h] * sf : -INFINITY, v1 ? d[2 * h + 1] * sf : -INFINITY);
      float* dst;
      if (gchunk < 0) {
        dst = p.S_t + ((size_t)bh * p.n_tiles + x) * (kT * kT) + i * kT + j;
      } else {
        if (i >= nrows) continue;
        dst = p.S_g + ((size_t)bh * p.n_global + gchunk * kT + i) * p.Lpad + cg;
      }
      *reinterpret_cast<float2*>(dst) = o;
    }
  }
}

// a-3: the CSR SDDMM, warp per (row, bh); 4 groups of 8 lanes, one nnz per group and step.
__global__ void __launch_bounds__(256) staged_sddmm_csr(const StagedParams p, bool bf16) {
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= (int64_t)p.BH * p.L) return;
  const int bh = (int)(gw / p.L);
  const int r = (int)(gw % p.L);
  const int beg = __ldg(p.csr_row_ptr + r), end = __ldg(p.csr_row_ptr + r + 1);
  if (beg == end) return;
  const int lane = threadIdx.x & 31, grp = lane >> 3, q8 = lane & 7;
  const int bb = bh / p.H, hh = bh % p.H;
  const int4 qv = ld_nc_v4(p.q.data + bb * p.q.sb + hh * p.q.sh + (int64_t)r * p.q.sl + q8 * 8);
  const uint16_t* qh = reinterpret_cast<const uint16_t*>(&qv);
  float qf[8];
#pragma unroll
  for (int e = 0; e < 8; ++e) qf[e] = bf16 ? from16<true>(qh[e]) : from16<false>(qh[e]);
  const uint16_t* Kb = p.k.data + bb * p.k.sb + hh * p.k.sh + q8 * 8;
  for (int i0 = beg; i0 < end; i0 += 4) {
    const int i = i0 + grp;
    float dot = 0.f;
    if (i < end) {
      const int c = __ldg(p.csr_col + i);
      const int4 kv = ld_nc_v4(Kb + (int64_t)c * p.k.sl);
      const uint16_t* kh = reinterpret_cast<const uint16_t*>(&kv);
#pragma unroll
      for (int e = 0; e < 8; ++e) dot = fmaf(qf[e], bf16 ? from16<true>(kh[e]) : from16<false>(kh[e]), dot);
    }
    dot += __shfl_xor_sync(0xffffffffu, dot, 1);
    dot += __shfl_xor_sync(0xffffffffu, dot, 2);
    dot += __shfl_xor_sync(0xffffffffu, dot, 4);
    if (q8 == 0 && i < end) p.S_f[(size_t)bh * p.nnz_csr + i] = dot * p.sf;
  }
}

// a-5: compound SpSoftmax, warp per (row slot, bh). Slots [0, nb*128): the rows of every row block
// (its BSR tile rows, then its CSR elements; global and padding rows have only -inf there and get
// P = 0); slots [nb*128, nb*128 + G): the dense global rows. Three sweeps over the row's scores as
// in P:128-131: the maximum, the sum of exponentials, then the normalised probabilities.
template <bool kBF16>
__global__ void __launch_bounds__(256) staged_softmax(const StagedParams p) {
  const int64_t slots = (int64_t)p.nb * kT + p.n_global;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= (int64_t)p.BH * slots) return;
  const int bh = (int)(gw / slots);
  const int64_t slot = gw % slots;
  const int lane = threadIdx.x & 31;
  const float LOG2E = 1.4426950408889634f;
  // the row's segments: (pointer to S, pointer to P, length); BSR tiles: 128 each
  int t0 = 0, t1 = 0, c0 = 0, c1 = 0;
  const float* sg = nullptr;
  uint16_t* pg = nullptr;
  int64_t ti = 0;
  if (slot < (int64_t)p.nb * kT) {
    const int I = (int)(slot / kT);
    ti = slot % kT;
    t0 = __ldg(p.bsr_row_ptr + I);
    t1 = __ldg(p.bsr_row_ptr + I + 1);
    if (slot < p.L) {
      c0 = __ldg(p.csr_row_ptr + slot);
      c1 = __ldg(p.csr_row_ptr + slot + 1);
    }
  } else {
    const int gi = (int)(slot - (int64_t)p.nb * kT);
    sg = p.S_g + ((size_t)bh * p.n_global + gi) * p.Lpad;
    pg = p.P_g + ((size_t)bh * p.n_global + gi) * p.Lpad;
  }
  const float* St = p.S_t + (size_t)bh * p.n_tiles * (kT * kT) + ti * kT;
  uint16_t* Pt = p.P_t + (size_t)bh * p.n_tiles * (kT * kT) + ti * kT;
  const float* Sf = p.S_f + (size_t)bh * p.nnz_csr;
  uint16_t* Pf = p.P_f + (size_t)bh * p.nnz_csr;

  // sweep 1: row maximum over the non-zero blocks, then the non-zero elements
  float m = -INFINITY;
  if (sg) {
    for (int c = lane * 4; c < p.Lpad; c += 128) {
      const float4 s = *reinterpret_cast<const float4*>(sg + c);
      m = fmaxf(m, fmaxf(fmaxf(s.x, s.y), fmaxf(s.z, s.w)));
    }
  } else {
    for (int t = t0; t < t1; ++t) {
      const float4 s = *reinterpret_cast<const float4*>(St + (size_t)t * (kT * kT) + lane * 4);
      m = fmaxf(m, fmaxf(fmaxf(s.x, s.y), fmaxf(s.z, s.w)));
    }
    for (int i = c0 + lane; i < c1; i += 32) m = fmaxf(m, Sf[i]);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  const float mb = m == -INFINITY ? 0.f : m * LOG2E;   // empty row: every exp is 0
  // sweep 2: sum of exponentials
  auto e2 = [&](float s) { return ex2(fmaf(s, LOG2E, -mb)); };
  float l = 0.f;
  if (sg) {
    for (int c = lane * 4; c < p.Lpad; c += 128) {
      const float4 s = *reinterpret_cast<const float4*>(sg + c);
      l += e2(s.x) + e2(s.y) + e2(s.z) + e2(s.w);
    }
  } else {
    for (int t = t0; t < t1; ++t) {
      const float4 s = *reinterpret_cast<const float4*>(St + (size_t)t * (kT * kT) + lane * 4);
      l += e2(s.x) + e2(s.y) + e2(s.z) + e2(s.w);
    }
    for (int i = c0 + lane; i < c1; i += 32) l += e2(Sf[i]);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o);
  const float inv = l > 0.f ? 1.f / l : 0.f;
  // sweep 3: normalised probabilities in the operand dtype
  if (sg) {
    for (int c = lane * 4; c < p.Lpad; c += 128) {
      const float4 s = *reinterpret_cast<const float4*>(sg + c);
      *reinterpret_cast<uint2*>(pg + c) =
          make_uint2(pack2<kBF16>(e2(s.x) * inv, e2(s.y) * inv), pack2<kBF16>(e2(s.z) * inv, e2(s.w) * inv));
    }
  } else {
    for (int t = t0; t < t1; ++t) {
      const float4 s = *reinterpret_cast<const float4*>(St + (size_t)t * (kT * kT) + lane * 4);
      *reinterpret_cast<uint2*>(Pt + (size_t)t * (kT * kT) + lane * 4) =
          make_uint2(pack2<kBF16>(e2(s.x) * inv, e2(s.y) * inv), pack2<kBF16>(e2(s.z) * inv, e2(s.w) * inv));
    }
    for (int i = c0 + lane; i < c1; i += 32) Pf[i] = to16<kBF16>(e2(Sf[i]) * inv);
  }
}

// a-6: the CSR SpMM, warp per (row with CSR nnz, bh): O_f[r] = sum_c P_f(r, c) V[c] in fp32.
__global__ void __launch_bounds__(256) staged_spmm_csr(const StagedParams p, bool bf16) {
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= (int64_t)p.BH * p.L) return;
  const int bh = (int)(gw / p.L);
  const int r = (int)(gw % p.L);
  const int beg = __ldg(p.csr_row_ptr + r), end = __ldg(p.csr_row_ptr + r + 1);
  if (beg == end) return;
  const int lane = threadIdx.x & 31, grp = lane >> 3, q8 = lane & 7;
  const int bb = bh / p.H, hh = bh % p.H;
  const uint16_t* Vb = p.v.data + bb * p.v.sb + hh * p.v.sh + q8 * 8;
  const uint16_t* Pf = p.P_f + (size_t)bh * p.nnz_csr;
  float acc[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
  for (int i = beg + grp; i < end; i += 4) {
    const int c = __ldg(p.csr_col + i);
    const float pr = bf16 ? from16<true>(Pf[i]) : from16<false>(Pf[i]);
    const int4 vv = ld_nc_v4(Vb + (int64_t)c * p.v.sl);
    const uint16_t* vh = reinterpret_cast<const uint16_t*>(&vv);
#pragma unroll
    for (int e = 0; e < 8; ++e) acc[e] = fmaf(pr, bf16 ? from16<true>(vh[e]) : from16<false>(vh[e]), acc[e]);
  }
#pragma unroll
  for (int e = 0; e < 8; ++e) {
    acc[e] += __shfl_xor_sync(0xffffffffu, acc[e], 8);
    acc[e] += __shfl_xor_sync(0xffffffffu, acc[e], 16);
  }
  if (lane < 8) {
    float4* dst = reinterpret_cast<float4*>(p.O_f + ((size_t)bh * p.L + r) * 64 + q8 * 8);
    dst[0] = make_float4(acc[0], acc[1], acc[2], acc[3]);
    dst[1] = make_float4(acc[4], acc[5], acc[6], acc[7]);
  }
}

// a-7 / a-4 (SpMM part) / a-8: O = sum_J P_IJ V_J (+ O_f of the row's CSR part) per 128-row block
// (blockIdx.x < nb) or per global-row chunk (P from P_g, every column block); 8 warps x 16 rows,
// 16-bit output. Global rows inside a band row block are skipped there (their P is 0 in the tiles;
// the dense-row chunk writes them, A5).
template <bool kBF16>
__global__ void __launch_bounds__(256) staged_spmm_tiles(const StagedParams p) {
  __shared__ __align__(128) uint8_t sm[kT * 256 + kT * 128];
  const uint32_t sP = smem_u32(sm), sV = sP + kT * 256;
  const int bh = blockIdx.y, bb = bh / p.H, hh = bh % p.H;
  const int x = blockIdx.x + p.blk0;
  const bool dense = x >= p.nb;
  const int gchunk = dense ? x - p.nb : -1;
  const int nrows = dense ? min(kT, p.n_global - gchunk * kT) : kT;
  const int t0 = dense ? 0 : __ldg(p.bsr_row_ptr + x), t1 = dense ? p.nb : __ldg(p.bsr_row_ptr + x + 1);
  const uint16_t* Vb = p.v.data + bb * p.v.sb + hh * p.v.sh;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int r0 = warp * 16;
  float acc[8][4];
#pragma unroll
  for (int n = 0; n < 8; ++n)
#pragma unroll
    for (int e = 0; e < 4; ++e) acc[n][e] = 0.f;

  for (int tt = t0; tt < t1; ++tt) {
    const int J = dense ? tt : __ldg(p.bsr_col + tt);
    // P rows (128 keys = 16 chunks each) and V rows of column block J
    const uint16_t* Pbase = dense ? p.P_g + ((size_t)bh * p.n_global + gchunk * kT) * p.Lpad + (size_t)J * kT
                                  : p.P_t + ((size_t)bh * p.n_tiles + tt) * (kT * kT);
    const int64_t prs = dense ? p.Lpad : kT;
    for (int e = threadIdx.x; e < kT * 16; e += blockDim.x) {
      const int row = e >> 4, ch = e & 15;
      const int4 v = row < nrows ? *reinterpret_cast<const int4*>(Pbase + row * prs + ch * 8) : make_int4(0, 0, 0, 0);
      sts16(swz(sP, row, ch, 16), v);
    }
    load_rows64(sV, [&](int j) -> const uint16_t* {
      const int64_t c = (int64_t)J * kT + j;
      return c < p.L ? Vb + c * p.v.sl : nullptr;
    });
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < 8; ++kk) {   // 16 keys per step
      uint32_t a[4];
      ldsm_x4(a, swz(sP, r0 + (lane & 7) + 8 * ((lane >> 3) & 1), 2 * kk + (lane >> 4), 16));
#pragma unroll
      for (int np = 0; np < 4; ++np) {   // pairs of n8 tiles (16 dims)
        uint32_t b[4];
        ldsm_x4_t(b, swz(sV, 16 * kk + (lane & 7) + 8 * ((lane >> 3) & 1), 2 * np + (lane >> 4), 8));
        mma16816<kBF16>(acc[2 * np], a, b[0], b[1]);
        mma16816<kBF16>(acc[2 * np + 1], a, b[2], b[3]);
      }
    }
    __syncthreads();
  }
  // epilogue: rows r0 + g (+8); lane holds dims 8n + 2t, 8n + 2t + 1
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    const int i = r0 + g + 8 * h;
    int64_t r;
    if (dense) {
      if (i >= nrows) continue;
      r = __ldg(p.global_rows + gchunk * kT + i);
    } else {
      r = (int64_t)x * kT + i;
      if (r >= p.L || __ldg(p.row_is_global + r)) continue;
    }
    const float* of = nullptr;
    if (!dense && __ldg(p.csr_row_ptr + r + 1) > __ldg(p.csr_row_ptr + r)) of = p.O_f + ((size_t)bh * p.L + r) * 64;
    uint16_t* orow = p.o.data + bb * p.o.sb + hh * p.o.sh + r * p.o.sl;
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      float v0 = acc[n][2 * h], v1 = acc[n][2 * h + 1];
      if (of) {
        const float2 f = *reinterpret_cast<const float2*>(of + 8 * n + 2 * t);
        v0 += f.x;
        v1 += f.y;
      }
      *reinterpret_cast<uint32_t*>(orow + 8 * n + 2 * t) = pack2<kBF16>(v0, v1);
    }
  }
}

cudaError_t launch_staged_sddmm(const StagedParams& p, bool bf16, cudaStream_t stream, cudaStream_t side) {
  const int gtiles = ((p.n_global + kT - 1) / kT) * p.nb;
  if (p.nnz_csr > 0) {   // fine part (side stream when concurrent)
    const int64_t warps = (int64_t)p.BH * p.L;
    staged_sddmm_csr<<<(unsigned)((warps + 7) / 8), 256, 0, side>>>(p, bf16);
  }
  if (p.n_tiles + gtiles > 0) {   // coarse tiles and dense-row tiles
    dim3 grid(p.n_tiles + gtiles, p.BH);
    if (bf16)
      staged_sddmm_tiles<true><<<grid, 256, 0, stream>>>(p);
    else
      staged_sddmm_tiles<false><<<grid, 256, 0, stream>>>(p);
  }
  return cudaGetLastError();
}

cudaError_t launch_staged_softmax(const StagedParams& p, bool bf16, cudaStream_t stream) {
  const int64_t warps = (int64_t)p.BH * ((int64_t)p.nb * kT + p.n_global);
  if (warps == 0) return cudaSuccess;
  if (bf16)
    staged_softmax<true><<<(unsigned)((warps + 7) / 8), 256, 0, stream>>>(p);
  else
    staged_softmax<false><<<(unsigned)((warps + 7) / 8), 256, 0, stream>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_staged_spmm(const StagedParams& p, bool bf16, cudaStream_t stream, cudaStream_t side,
                               cudaEvent_t ev) {
  auto tiles = [&](int blk0, int nblk) {
    if (nblk <= 0) return;
    StagedParams q = p;
    q.blk0 = blk0;
    dim3 grid(nblk, p.BH);
    if (bf16)
      staged_spmm_tiles<true><<<grid, 256, 0, stream>>>(q);
    else
      staged_spmm_tiles<false><<<grid, 256, 0, stream>>>(q);
  };
  const int gchunks = (p.n_global + kT - 1) / kT;
  if (p.nnz_csr > 0) {
    const int64_t warps = (int64_t)p.BH * p.L;
    staged_spmm_csr<<<(unsigned)((warps + 7) / 8), 256, 0, side>>>(p, bf16);
  }
  if (side != stream && p.nnz_csr > 0) {
    // dense-row chunks need no O_csr: they run beside the CSR SpMM; the row blocks wait for it
    tiles(p.nb, gchunks);
    cudaError_t e = cudaEventRecord(ev, side);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(stream, ev, 0);
    if (e != cudaSuccess) return e;
    tiles(0, p.nb);
  } else {
    tiles(0, p.nb + gchunks);
  }
  return cudaGetLastError();
}

}  // namespace mg
