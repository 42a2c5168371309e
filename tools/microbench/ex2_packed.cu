#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t ex2bf2(uint32_t x) { uint32_t y; asm volatile("ex2.approx.ftz.bf16x2 %0, %1;" : "=r"(y) : "r"(x)); return y; }
__device__ __forceinline__ uint32_t ex2h2(uint32_t x) { uint32_t y; asm volatile("ex2.approx.f16x2 %0, %1;" : "=r"(y) : "r"(x)); return y; }
__device__ __forceinline__ float ex2f(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
template <int MODE>
__global__ void k(uint32_t* out, long long* cyc, int iters) {
  uint32_t v[32];
  for (int i = 0; i < 32; ++i) v[i] = 0xbf80bf80u ^ (threadIdx.x + i);
  __syncthreads();
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      if (MODE == 0) v[i] = __float_as_uint(ex2f(__uint_as_float(v[i])));
      if (MODE == 1) v[i] = ex2bf2(v[i]);
      if (MODE == 2) v[i] = ex2h2(v[i]);
    }
  }
  long long t1 = clock64();
  uint32_t s = 0;
  for (int i = 0; i < 32; ++i) s ^= v[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
template <int M> void run(uint32_t* out, long long* cyc, int warps) {
  for (int r = 0; r < 2; ++r) k<M><<<148, warps * 32>>>(out, cyc, 1000);
  cudaDeviceSynchronize();
  long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  double ops = (double)warps * 32 * 32 * 1000;   // instructions x lanes
  printf("mode %d warps %2d: %.2f lane-ops/clk/SM (%s)\n", M, warps, ops / c, M == 0 ? "f32: 1 value" : "x2: 2 values");
}
int main() { uint32_t* o; long long* c; cudaMalloc(&o, 1 << 20); cudaMalloc(&c, 8 * 1024);
  for (int w : {4, 8, 16}) { run<0>(o, c, w); run<1>(o, c, w); run<2>(o, c, w); } return 0; }
