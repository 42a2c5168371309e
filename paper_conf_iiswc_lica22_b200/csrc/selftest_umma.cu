// One-shot tcgen05 MMA checks (diagnostics only; used by tests/test_gpu_umma.py).
// They pin the exact operand layouts the attention kernel relies on:
//   mode 0: SS form, A and B both K-major SWIZZLE_128B (Q.K^T of the coarse SDDMM)
//   mode 1: TS form, A (P) in TMEM written with tcgen05.st as packed 16-bit pairs, B (V)
//           MN-major SWIZZLE_128B as a TMA box of V would land (coarse SpMM).
#include <cuda_bf16.h>

#include "kernels.cuh"
#include "sm100_ptx.cuh"

namespace mg {

using namespace ptx;

__global__ void __launch_bounds__(128, 1)
selftest_umma_kernel(int mode, const uint16_t* __restrict__ A, const uint16_t* __restrict__ Bm, float* __restrict__ D) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* As = smem;              // 16 KB
  uint8_t* Bs = smem + 16384;      // 16 KB
  __shared__ uint64_t bar;
  __shared__ uint32_t tmem_base;
  const int t = threadIdx.x;
  const int warp = t >> 5;

  if (mode == 0) {
    // A[128][64], B[128][64] row-major -> K-major SW128: row m at m*128B, 16B chunk c at (c ^ (m&7))*16
    for (int m = t; m < 128; m += 128) {
      for (int c = 0; c < 8; ++c) {
        *reinterpret_cast<int4*>(As + m * 128 + ((c ^ (m & 7)) * 16)) = *reinterpret_cast<const int4*>(A + m * 64 + c * 8);
        *reinterpret_cast<int4*>(Bs + m * 128 + ((c ^ (m & 7)) * 16)) = *reinterpret_cast<const int4*>(Bm + m * 64 + c * 8);
      }
    }
  } else {
    // B[128 k][64 n] row-major (n contiguous) -> MN-major SW128: row k at k*128B, chunk swizzled
    for (int k = t; k < 128; k += 128)
      for (int c = 0; c < 8; ++c)
        *reinterpret_cast<int4*>(Bs + k * 128 + ((c ^ (k & 7)) * 16)) = *reinterpret_cast<const int4*>(Bm + k * 64 + c * 8);
  }
  fence_proxy_async_smem();
  if (t == 0) { mbar_init(smem_u32(&bar), 1); fence_barrier_init(); }
  if (warp == 0) { tmem_alloc(smem_u32(&tmem_base), 256); tmem_relinquish(); }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = tmem_base;
  const uint32_t lane_off = (uint32_t)((warp & 3) * 32) << 16;

  if (mode == 1) {
    // thread t owns row t of A[128][128]: 64 packed columns at TMEM columns [128, 192)
    for (int cb = 0; cb < 4; ++cb) {
      uint32_t r[16];
      for (int i = 0; i < 16; ++i) r[i] = *reinterpret_cast<const uint32_t*>(A + t * 128 + cb * 32 + 2 * i);
      tmem_st16(tbase + lane_off + 128 + cb * 16, r);
    }
    tmem_wait_st();
    tc_fence_before();
  }
  __syncthreads();
  tc_fence_after();
  if (t == 0) {
    if (mode == 0) {
      const uint32_t id = idesc_f16(true, 128, 128, false, false);
      for (int kk = 0; kk < 4; ++kk) {
        uint64_t ad = smem_desc_sw128(smem_u32(As) + kk * 32, 16, 1024);
        uint64_t bd = smem_desc_sw128(smem_u32(Bs) + kk * 32, 16, 1024);
        mma_ss(tbase, ad, bd, id, kk > 0);
      }
    } else {
      const uint32_t id = idesc_f16(true, 128, 64, false, true);
      for (int kk = 0; kk < 8; ++kk) {
        uint64_t bd = smem_desc_sw128(smem_u32(Bs) + kk * 2048, 8192, 1024);
        mma_ts(tbase, tbase + 128 + kk * 8, bd, id, kk > 0);
      }
    }
    mma_commit(smem_u32(&bar));
  }
  mbar_wait(smem_u32(&bar), 0);
  tc_fence_after();
  const int ncols = mode == 0 ? 128 : 64;
  for (int c = 0; c < ncols; c += 32) {
    uint32_t r[32];
    tmem_ld32(tbase + lane_off + c, r);
    tmem_wait_ld();
    for (int i = 0; i < 32; ++i) D[t * ncols + c + i] = __uint_as_float(r[i]);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tbase, 256);
}

cudaError_t launch_selftest_umma(int mode, const void* A, const void* B, float* D, cudaStream_t stream) {
  const int smem = 32768 + 1024;
  cudaError_t e = cudaFuncSetAttribute(selftest_umma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  selftest_umma_kernel<<<1, 128, smem, stream>>>(mode, static_cast<const uint16_t*>(A), static_cast<const uint16_t*>(B), D);
  return cudaGetLastError();
}

}  // namespace mg
