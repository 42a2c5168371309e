// Fine-grained CSR kernel (CUDA cores): the CSR residual rows that are not carried by a
// tensor-core strip tile. "We execute the sparse patterns with low spatial locality on the
// fine-grained kernels to reduce unnecessary computation and memory accesses" (P:12, P:81,
// P:101). The paper adapts Sputnik (row-splitting SDDMM, 1-D tiled SpMM); here SDDMM ->
// online softmax -> SpMM are fused per row, one warp per (row, batch*head):
//   * the warp is 4 groups x 8 lanes; a group reads one 128-byte K (or V) row with
//     8 x 16-byte vector loads (coalesced, L1-bypassing .nc path);
//   * 32 column indices are loaded per step (one per lane) and broadcast with shuffles;
//   * each group keeps its own running (max, sum, acc[8]); the 4 groups are merged with a
//     log-sum-exp shuffle reduction at the end.
// Output: the final O row (16-bit) when the row has no coarse part, otherwise fp32 partial
// (max, sum, acc[64]) merged by the coarse kernel's epilogue (compound SpSoftmax).
#include <cuda_bf16.h>
#include <cuda_fp16.h>

#include "kernels.cuh"
#include "sm100_ptx.cuh"

namespace mg {

using namespace ptx;

namespace {

template <bool kBF16>
__device__ __forceinline__ void unpack8(const int4 v, float (&f)[8]) {
  const uint32_t w[4] = {(uint32_t)v.x, (uint32_t)v.y, (uint32_t)v.z, (uint32_t)v.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    if (kBF16) {
      f[2 * i] = __uint_as_float(w[i] << 16);
      f[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
    } else {
      const __half2 h = *reinterpret_cast<const __half2*>(&w[i]);
      const float2 ff = __half22float2(h);
      f[2 * i] = ff.x;
      f[2 * i + 1] = ff.y;
    }
  }
}

template <bool kBF16>
__device__ __forceinline__ uint32_t pack2(float lo, float hi) {
  return kBF16 ? pack_bf16(lo, hi) : pack_f16(lo, hi);
}

}  // namespace

template <bool kBF16>
__global__ void __launch_bounds__(256, 2) fine_rows_kernel(const FineParams p) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= (int64_t)p.BH * p.n_fine_rows) return;
  const int u0 = (int)(gw / p.n_fine_rows);
  const int fi = (int)(gw % p.n_fine_rows);
  const int bh = p.fine_sample ? __ldg(p.fine_sample + fi) * p.H + u0 : u0;   // (batched plans)
  const int enc = __ldg(p.fine_rows + fi);
  const int r = enc & 0x7fffffff;
  const bool final_out = enc < 0;
  const int bb = bh / p.H, hh = bh % p.H;
  const int grp = lane >> 3, q8 = lane & 7;
  const float c = p.scale_log2;

  const uint16_t* Kb = p.k.data + bb * p.k.sb + hh * p.k.sh + q8 * 8;
  const uint16_t* Vb = p.v.data + bb * p.v.sb + hh * p.v.sh + q8 * 8;
  float qf[8];
  unpack8<kBF16>(ld_nc_v4(p.q.data + bb * p.q.sb + hh * p.q.sh + (int64_t)r * p.q.sl + q8 * 8), qf);

  const int beg = __ldg(p.row_ptr + fi), end = __ldg(p.row_ptr + fi + 1);
  float m = -INFINITY, l = 0.f;
  float acc[8];
#pragma unroll
  for (int e = 0; e < 8; ++e) acc[e] = 0.f;

  for (int base = beg; base < end; base += 32) {
    const int col = (base + lane < end) ? __ldg(p.cols + base + lane) : -1;
    int4 kv[8], vv[8];
    int cc[8];
#pragma unroll
    for (int s = 0; s < 8; ++s) {
      cc[s] = __shfl_sync(0xffffffffu, col, s * 4 + grp);
      if (cc[s] >= 0) {
        kv[s] = ld_nc_v4(Kb + (int64_t)cc[s] * p.k.sl);
        vv[s] = ld_nc_v4(Vb + (int64_t)cc[s] * p.v.sl);
      } else {
        kv[s] = make_int4(0, 0, 0, 0);
        vv[s] = make_int4(0, 0, 0, 0);
      }
    }
    float sc[8];
#pragma unroll
    for (int s = 0; s < 8; ++s) {
      float kf[8];
      unpack8<kBF16>(kv[s], kf);
      float d = 0.f;
#pragma unroll
      for (int e = 0; e < 8; ++e) d = fmaf(qf[e], kf[e], d);
      d += __shfl_xor_sync(0xffffffffu, d, 1);
      d += __shfl_xor_sync(0xffffffffu, d, 2);
      d += __shfl_xor_sync(0xffffffffu, d, 4);
      sc[s] = cc[s] >= 0 ? d : -INFINITY;
    }
    float cmax = sc[0];
#pragma unroll
    for (int s = 1; s < 8; ++s) cmax = fmaxf(cmax, sc[s]);
    const float m_new = fmaxf(m, cmax);
    const float mu = (m_new == -INFINITY) ? 0.f : m_new;
    const float alpha = ex2((m - mu) * c);
    const float nb = -mu * c;
    l *= alpha;
#pragma unroll
    for (int e = 0; e < 8; ++e) acc[e] *= alpha;
#pragma unroll
    for (int s = 0; s < 8; ++s) {
      const float pv = ex2(fmaf(sc[s], c, nb));
      l += pv;
      float vf[8];
      unpack8<kBF16>(vv[s], vf);
#pragma unroll
      for (int e = 0; e < 8; ++e) acc[e] = fmaf(pv, vf[e], acc[e]);
    }
    m = m_new;
  }
  // merge the 4 groups (lanes q8, q8+8, q8+16, q8+24 hold the same output columns)
#pragma unroll
  for (int off = 8; off <= 16; off <<= 1) {
    const float mo = __shfl_xor_sync(0xffffffffu, m, off);
    const float lo = __shfl_xor_sync(0xffffffffu, l, off);
    const float mn = fmaxf(m, mo);
    const float mu = (mn == -INFINITY) ? 0.f : mn;
    const float a = ex2((m - mu) * c), bsc = ex2((mo - mu) * c);
    l = l * a + lo * bsc;
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      const float ao = __shfl_xor_sync(0xffffffffu, acc[e], off);
      acc[e] = acc[e] * a + ao * bsc;
    }
    m = mn;
  }
  if (lane >= 8) return;
  if (final_out) {
    const float inv = l > 0.f ? 1.f / l : 0.f;
    uint4 o4;
    o4.x = pack2<kBF16>(acc[0] * inv, acc[1] * inv);
    o4.y = pack2<kBF16>(acc[2] * inv, acc[3] * inv);
    o4.z = pack2<kBF16>(acc[4] * inv, acc[5] * inv);
    o4.w = pack2<kBF16>(acc[6] * inv, acc[7] * inv);
    *reinterpret_cast<uint4*>(p.o.data + bb * p.o.sb + hh * p.o.sh + (int64_t)r * p.o.sl + q8 * 8) = o4;
  } else {
    const size_t idx = (size_t)u0 * p.n_fine_rows + fi;
    float4* dst = reinterpret_cast<float4*>(p.part_acc + idx * 64 + q8 * 8);
    dst[0] = make_float4(acc[0], acc[1], acc[2], acc[3]);
    dst[1] = make_float4(acc[4], acc[5], acc[6], acc[7]);
    if (lane == 0) p.part_ml[idx] = make_float2(m, l);
  }
}

cudaError_t launch_fine(const FineParams& p, bool bf16, cudaStream_t stream) {
  const int64_t warps = (int64_t)p.BH * p.n_fine_rows;
  if (warps == 0) return cudaSuccess;
  const int64_t blocks = (warps + 7) / 8;
  if (bf16)
    fine_rows_kernel<true><<<(unsigned)blocks, 256, 0, stream>>>(p);
  else
    fine_rows_kernel<false><<<(unsigned)blocks, 256, 0, stream>>>(p);
  return cudaGetLastError();
}

}  // namespace mg
