// Microbenchmark: throughput of the softmax inner-loop instruction mix on one SM.
//   mode 0: ex2.approx only            mode 1: FFMA2 + 2 ex2 + FADD2 + F2FP (the exp chunk)
//   mode 2: FMNMX3 only (max pass)
// Launch: 1 CTA of W warps; reports cycles per warp-instruction-group.
#include <cstdio>
#include <cuda_bf16.h>
#include <cstdint>
__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ uint32_t pk(float a, float b) { uint32_t r; asm("cvt.rn.bf16x2.f32 %0, %2, %1;" : "=r"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ float fmax3(float a, float b, float c) { float d; asm("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c)); return d; }
template <int MODE>
__global__ void k(float* out, long long* cyc, int iters) {
  float v[32];
  for (int i = 0; i < 32; ++i) v[i] = -0.001f * (threadIdx.x + i);
  float2 acc = make_float2(0, 0); uint32_t x = 0; float mx = -1e30f;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 32; i += 2) {
      if (MODE == 0) { v[i] = ex2(v[i]); v[i+1] = ex2(v[i+1]); }
      if (MODE == 1) {
        float2 y = __ffma2_rn(make_float2(v[i], v[i+1]), make_float2(0.18f, 0.18f), make_float2(-1.f, -1.f));
        float p0 = ex2(y.x), p1 = ex2(y.y);
        acc = __fadd2_rn(acc, make_float2(p0, p1));
        x ^= pk(p0, p1);
        v[i] = p0 - 1.0f; v[i+1] = p1 - 1.0f;
      }
      if (MODE == 2) { mx = fmax3(mx, v[i], v[i+1]); v[i] += 1e-7f; }
    }
  }
  long long t1 = clock64();
  float s = acc.x + acc.y + mx + (float)x;
  for (int i = 0; i < 32; ++i) s += v[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
int main() {
  float* out; long long* cyc; cudaMalloc(&out, 1 << 20); cudaMalloc(&cyc, 1024 * 8);
  const int iters = 2000;
  for (int mode = 0; mode < 3; ++mode)
    for (int warps : {4, 8, 12, 16}) {
      for (int rep = 0; rep < 2; ++rep) {
        if (mode == 0) k<0><<<148, warps * 32>>>(out, cyc, iters);
        if (mode == 1) k<1><<<148, warps * 32>>>(out, cyc, iters);
        if (mode == 2) k<2><<<148, warps * 32>>>(out, cyc, iters);
      }
      cudaDeviceSynchronize();
      long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
      // elements per SM processed = warps * 32 lanes * 32 elems * iters
      double elems = (double)warps * 32 * 32 * iters;
      printf("mode %d warps/SM %2d: %.3f elements/clk/SM (%.2f cycles per warp-elem-instr per SMSP)\n", mode, warps,
             elems / c, (double)c / ((double)warps / 4 * 32 * iters));
    }
  return 0;
}
