// Microbenchmark: throughput of the softmax chunk's non-MUFU instructions on one SM.
//   mode 0: cvt.rn.bf16x2.f32 (F2FP pack) only
//   mode 1: FFMA2 + FADD2 + F2FP per pair (the chunk without ex2)
//   mode 2: FFMA2 + FADD2 + PRMT pack (truncating pack on the integer pipe)
//   mode 3: ex2 only (reference)
//   mode 4: FFMA2 + 2 ex2 + FADD2 + F2FP (the full chunk)
// Launch: 148 CTAs of W warps; reports elements (fp32 values) per clk per SM.
#include <cstdio>
#include <cstdint>
#include <cuda_bf16.h>
__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ uint32_t pk(float a, float b) { uint32_t r; asm volatile("cvt.rn.bf16x2.f32 %0, %2, %1;" : "=r"(r) : "f"(a), "f"(b)); return r; }
__device__ __forceinline__ uint32_t pk_t(float a, float b) { uint32_t r; asm volatile("prmt.b32 %0, %1, %2, 0x7632;" : "=r"(r) : "r"(__float_as_uint(a)), "r"(__float_as_uint(b))); return r; }
template <int MODE>
__global__ void k(float* out, long long* cyc, int iters) {
  float v[32];
  for (int i = 0; i < 32; ++i) v[i] = -0.001f * (threadIdx.x + i);
  float2 acc = make_float2(0, 0); uint32_t x = 0;
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 32; i += 2) {
      if (MODE == 0) { x ^= pk(v[i], v[i + 1]); v[i] += 1e-7f; }
      if (MODE == 1 || MODE == 2 || MODE == 4) {
        float2 y = __ffma2_rn(make_float2(v[i], v[i+1]), make_float2(0.18f, 0.18f), make_float2(-1.f, -1.f));
        float p0 = y.x, p1 = y.y;
        if (MODE == 4) { p0 = ex2(y.x); p1 = ex2(y.y); }
        acc = __fadd2_rn(acc, make_float2(p0, p1));
        x ^= (MODE == 2) ? pk_t(p0, p1) : pk(p0, p1);
        v[i] = p0 - 1.0f; v[i+1] = p1 - 1.0f;
      }
      if (MODE == 3) { v[i] = ex2(v[i]); v[i+1] = ex2(v[i+1]); }
    }
  }
  long long t1 = clock64();
  float s = acc.x + acc.y + (float)x;
  for (int i = 0; i < 32; ++i) s += v[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
template <int M> void run(float* out, long long* cyc, int warps, int iters) {
  for (int rep = 0; rep < 2; ++rep) k<M><<<148, warps * 32>>>(out, cyc, iters);
  cudaDeviceSynchronize();
  long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  double elems = (double)warps * 32 * 32 * iters;
  printf("mode %d warps/SM %2d: %.2f elements/clk/SM\n", M, warps, elems / c);
}
int main() {
  float* out; long long* cyc; cudaMalloc(&out, 1 << 20); cudaMalloc(&cyc, 1024 * 8);
  for (int w : {4, 8, 16}) { run<0>(out, cyc, w, 2000); run<1>(out, cyc, w, 2000); run<2>(out, cyc, w, 2000); run<3>(out, cyc, w, 2000); run<4>(out, cyc, w, 2000); }
  return 0;
}
