// Fine-grained CSR kernel on the warp-level tensor cores (mma.sync m16n8k16), the default for the
// CUDA-core CSR rows of the plan (the low-locality residual). Same contract as
// fine_rows.cu (one warp per (CSR row, batch*head); SDDMM -> online softmax -> SpMM fused; final
// row or fp32 partial for the coarse epilogue's merge), but the two dot-product phases
// run as small MMAs instead of per-element FMAs and shuffle reductions: the CUDA-core kernel is
// issue-bound (73% issue-active, 27 warp instructions per nnz, profiles/r01c_ncu_full_c4_fine.txt),
// while the gathers alone would run at ~22 TB/s from L2 (tools/microbench/gather_bw.cu).
//
// A step handles 16 nnz of the row, as two chunks A and B of 8. Lane = 4g + t.
//   SDDMM  s^T = q . K_c^T as mma(M=16 x N=8 x K=16) x 4 (64 dims): A = q broadcast to all 16
//          rows, B column n = gathered K row c_{chunk[n]}. The contraction order over d is free,
//          so lane t owns dims {8t..8t+7} and {32+8t..32+8t+7} of both q and the K row it loads
//          (two 16-byte loads, half-line contiguous per 4 lanes); mma j uses the lane's register
//          pairs 2j, 2j+1 for k {2t,2t+1} and {2t+8,2t+9}. D: lane (g,t) gets s of chunk nnz 2t, 2t+1.
//   SpMM   O^T = V_c^T . p as mma(M=16 dims x N=8 x K=16 nnz) x 4 (64 dims): k = nnz (chunk A
//          nnz 2t,2t+1 -> k 2t,2t+1; chunk B -> k 2t+8, 2t+9), which is exactly where the SDDMM
//          left each lane's p, so P never moves between lanes; the M (dim) order is free too: lane
//          g owns dims 8g..8g+7, i.e. one 16-byte load per gathered V row, and the A fragment is
//          built from the four rows with byte permutes.
// p is rounded to the operand dtype for the SpMM (as in the coarse kernel, A9); s, the
// running max/sum and O accumulate in fp32. Lazy rescaling: the exponent keeps a stale max until
// a step's max exceeds it by 8/c (p <= 256), warp-uniform because all lanes see the same max.
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

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
  uint32_t r;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
  return r;
}

template <bool kBF16>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  return kBF16 ? pack_bf16(lo, hi) : pack_f16(lo, hi);
}

// the gathered rows of one 16-nnz step
struct Step {
  int4 k[4];   // K rows of chunk A nnz g (k[0], k[1]) and chunk B nnz g (k[2], k[3])
  int4 v[4];   // V rows of nnz A 2t, A 2t+1, B 2t, B 2t+1 (dims 8g..8g+7)
};

}  // namespace

// The gathers of step i+1 are issued into registers before step i is computed (one step in flight
// per warp, 16 warps per SM). A shared-memory ring filled by cp.async measured 6x slower: cp.async
// of 16-byte pieces that cover only part of a 128-byte line per instruction is pathological on
// sm_100 (tools/microbench/gather_bw.cu: 2.4 TB/s vs 17.6 TB/s for the same loads into registers).
template <bool kBF16>
__global__ void __launch_bounds__(256, 2) fine_mma_kernel(const FineParams p) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= (int64_t)p.BH * p.n_fine_rows) return;
  const int bh = (int)(gw / p.n_fine_rows);
  const int fi = (int)(gw % p.n_fine_rows);
  const int enc = __ldg(p.fine_rows + fi);
  const int r = enc & 0x7fffffff;
  const bool final_out = enc < 0;
  const int bb = bh / p.H, hh = bh % p.H;
  const int g = lane >> 2, t = lane & 3;
  const float c = p.scale_log2;

  const uint16_t* Kb = p.k.data + bb * p.k.sb + hh * p.k.sh + t * 8;   // + 32 for the second half
  const uint16_t* Vb = p.v.data + bb * p.v.sb + hh * p.v.sh + g * 8;
  const uint16_t* qrow = p.q.data + bb * p.q.sb + hh * p.q.sh + (int64_t)r * p.q.sl + t * 8;
  const int4 q0 = ld_nc_v4(qrow), q1 = ld_nc_v4(qrow + 32);
  const uint32_t qr[8] = {(uint32_t)q0.x, (uint32_t)q0.y, (uint32_t)q0.z, (uint32_t)q0.w,
                          (uint32_t)q1.x, (uint32_t)q1.y, (uint32_t)q1.z, (uint32_t)q1.w};

  const int beg = __ldg(p.row_ptr + fi), end = __ldg(p.row_ptr + fi + 1);
  // row strides fit 32 bits (checked by the forward's validation: (L - 1) * stride_l < 2^32)
  const uint32_t ksl = (uint32_t)p.k.sl, vsl = (uint32_t)p.v.sl;

  // step loader: the 16 column indices of a step come from `col` (lane i holds index base0 + i of
  // a 32-index window; `off` = 0 or 16 selects the half). Indices past the row's end are -1 and
  // read row 0 (the values are masked / multiplied by p = 0).
  auto load_step = [&](Step& st, int col, int off) {
    const int ca = __shfl_sync(0xffffffffu, col, off + g), cb = __shfl_sync(0xffffffffu, col, off + 8 + g);
    const int va0 = __shfl_sync(0xffffffffu, col, off + 2 * t), va1 = __shfl_sync(0xffffffffu, col, off + 2 * t + 1);
    const int vb0 = __shfl_sync(0xffffffffu, col, off + 8 + 2 * t);
    const int vb1 = __shfl_sync(0xffffffffu, col, off + 9 + 2 * t);
    const uint16_t* ka = Kb + (uint32_t)max(ca, 0) * ksl;
    const uint16_t* kb = Kb + (uint32_t)max(cb, 0) * ksl;
    st.k[0] = ld_nc_v4(ka);
    st.k[1] = ld_nc_v4(ka + 32);
    st.k[2] = ld_nc_v4(kb);
    st.k[3] = ld_nc_v4(kb + 32);
    st.v[0] = ld_nc_v4(Vb + (uint32_t)max(va0, 0) * vsl);
    st.v[1] = ld_nc_v4(Vb + (uint32_t)max(va1, 0) * vsl);
    st.v[2] = ld_nc_v4(Vb + (uint32_t)max(vb0, 0) * vsl);
    st.v[3] = ld_nc_v4(Vb + (uint32_t)max(vb1, 0) * vsl);
  };
  auto load_cols = [&](int base) { return base + lane < end ? __ldg(p.cols + base + lane) : -1; };

  float m = -INFINITY, l = 0.f;
  float acc[4][4];
#pragma unroll
  for (int j = 0; j < 4; ++j)
#pragma unroll
    for (int e = 0; e < 4; ++e) acc[j][e] = 0.f;
  const float thresh = 8.f / c;

  Step cur;
  int col = load_cols(beg);
  if (beg < end) load_step(cur, col, 0);
  for (int base = beg; base < end; base += 16) {
    // prefetch the next step's rows (the 32-index window advances every other step)
    Step nxt;
    const int nb = base + 16;
    const int off_next = ((nb - beg) & 16);
    if (off_next == 0) col = load_cols(nb);
    load_step(nxt, col, off_next);

    // ---- SDDMM: chunk A -> sa, chunk B -> sb (lane holds nnz 2t, 2t+1 of each)
    float sa[4] = {0.f, 0.f, 0.f, 0.f}, sb[4] = {0.f, 0.f, 0.f, 0.f};
    const uint32_t ka[8] = {(uint32_t)cur.k[0].x, (uint32_t)cur.k[0].y, (uint32_t)cur.k[0].z, (uint32_t)cur.k[0].w,
                            (uint32_t)cur.k[1].x, (uint32_t)cur.k[1].y, (uint32_t)cur.k[1].z, (uint32_t)cur.k[1].w};
    const uint32_t kb[8] = {(uint32_t)cur.k[2].x, (uint32_t)cur.k[2].y, (uint32_t)cur.k[2].z, (uint32_t)cur.k[2].w,
                            (uint32_t)cur.k[3].x, (uint32_t)cur.k[3].y, (uint32_t)cur.k[3].z, (uint32_t)cur.k[3].w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      mma16816<kBF16>(sa, qr[2 * j], qr[2 * j], qr[2 * j + 1], qr[2 * j + 1], ka[2 * j], ka[2 * j + 1]);
      mma16816<kBF16>(sb, qr[2 * j], qr[2 * j], qr[2 * j + 1], qr[2 * j + 1], kb[2 * j], kb[2 * j + 1]);
    }
    // this lane's score positions: nnz base + 2t, + 2t+1 (chunk A), + 8 + 2t, + 9 + 2t (chunk B)
    const int rem = end - base - 2 * t;
    float s[4] = {rem > 0 ? sa[0] : -INFINITY, rem > 1 ? sa[1] : -INFINITY, rem > 8 ? sb[0] : -INFINITY,
                  rem > 9 ? sb[1] : -INFINITY};
    // ---- online softmax over the step (warp-uniform max: lanes with equal t hold equal values)
    float mx = fmaxf(fmaxf(s[0], s[1]), fmaxf(s[2], s[3]));
    mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 1));
    mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 2));
    if (mx > m + thresh) {   // also taken on the first step (m = -inf); mx is finite (>= 1 valid nnz)
      const float alpha = ex2((m - mx) * c);
      l *= alpha;
#pragma unroll
      for (int j = 0; j < 4; ++j)
#pragma unroll
        for (int e = 0; e < 4; ++e) acc[j][e] *= alpha;
      m = mx;
    }
    const float nbias = -m * c;
    float pr[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      pr[i] = ex2(fmaf(s[i], c, nbias));
      l += pr[i];
    }
    const uint32_t pb0 = pack2<kBF16>(pr[0], pr[1]), pb1 = pack2<kBF16>(pr[2], pr[3]);
    // ---- SpMM: O^T[dims 8g+2j, 8g+2j+1] += V^T . p
    const uint32_t v0[4] = {(uint32_t)cur.v[0].x, (uint32_t)cur.v[0].y, (uint32_t)cur.v[0].z, (uint32_t)cur.v[0].w};
    const uint32_t v1[4] = {(uint32_t)cur.v[1].x, (uint32_t)cur.v[1].y, (uint32_t)cur.v[1].z, (uint32_t)cur.v[1].w};
    const uint32_t v2[4] = {(uint32_t)cur.v[2].x, (uint32_t)cur.v[2].y, (uint32_t)cur.v[2].z, (uint32_t)cur.v[2].w};
    const uint32_t v3[4] = {(uint32_t)cur.v[3].x, (uint32_t)cur.v[3].y, (uint32_t)cur.v[3].z, (uint32_t)cur.v[3].w};
#pragma unroll
    for (int j = 0; j < 4; ++j)
      mma16816<kBF16>(acc[j], prmt(v0[j], v1[j], 0x5410), prmt(v0[j], v1[j], 0x7632), prmt(v2[j], v3[j], 0x5410),
                      prmt(v2[j], v3[j], 0x7632), pb0, pb1);
    cur = nxt;
  }
  // row sum: lanes with the same g hold disjoint nnz subsets (t); every g holds the same sums
  l += __shfl_xor_sync(0xffffffffu, l, 1);
  l += __shfl_xor_sync(0xffffffffu, l, 2);
  // lane (g, 0): O dims 8g .. 8g+7 = acc[j][0] (dim 8g+2j), acc[j][2] (dim 8g+2j+1)
  float o8[8] = {acc[0][0], acc[0][2], acc[1][0], acc[1][2], acc[2][0], acc[2][2], acc[3][0], acc[3][2]};
  float inv = l > 0.f ? 1.f / l : 0.f;
  bool write_o = final_out;
  if (!final_out) {
    const size_t idx = (size_t)bh * p.n_fine_rows + fi;
    if (t == 0) {
      float4* dst = reinterpret_cast<float4*>(p.part_acc + idx * 64 + g * 8);
      __stcg(dst, make_float4(o8[0], o8[1], o8[2], o8[3]));
      __stcg(dst + 1, make_float4(o8[4], o8[5], o8[6], o8[7]));
      if (lane == 0) __stcg(p.part_ml + idx, make_float2(m, l));
    }
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
        const float4* src = reinterpret_cast<const float4*>(p.part_c_acc + idx * 64 + g * 8);
        const float4 c0 = __ldcg(src), c1 = __ldcg(src + 1);
        const float cc[8] = {c0.x, c0.y, c0.z, c0.w, c1.x, c1.y, c1.z, c1.w};
#pragma unroll
        for (int e = 0; e < 8; ++e) o8[e] = o8[e] * af + cc[e] * ac;
        write_o = true;
      }
    }
  }
  if (t != 0 || !write_o) return;
  uint4 o4;
  o4.x = pack2<kBF16>(o8[0] * inv, o8[1] * inv);
  o4.y = pack2<kBF16>(o8[2] * inv, o8[3] * inv);
  o4.z = pack2<kBF16>(o8[4] * inv, o8[5] * inv);
  o4.w = pack2<kBF16>(o8[6] * inv, o8[7] * inv);
  *reinterpret_cast<uint4*>(p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)r * p.o.sl + g * 8) = o4;
}

cudaError_t launch_fine_mma(const FineParams& p, bool bf16, cudaStream_t stream) {
  const int64_t warps = (int64_t)p.BH * p.n_fine_rows;
  if (warps == 0) return cudaSuccess;
  const int64_t blocks = (warps + 7) / 8;
  if (bf16)
    fine_mma_kernel<true><<<(unsigned)blocks, 256, 0, stream>>>(p);
  else
    fine_mma_kernel<false><<<(unsigned)blocks, 256, 0, stream>>>(p);
  return cudaGetLastError();
}

}  // namespace mg
