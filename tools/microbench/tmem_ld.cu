// Microbenchmark: latency of tcgen05.ld (4 x 32x32b.x16 in flight + wait) per warp, with 1..3
// warps per SMSP doing the same, and of a single x16 load + wait.
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ void ld16(uint32_t a, uint32_t (&r)[16]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
    : "=r"(r[0]),"=r"(r[1]),"=r"(r[2]),"=r"(r[3]),"=r"(r[4]),"=r"(r[5]),"=r"(r[6]),"=r"(r[7]),"=r"(r[8]),"=r"(r[9]),"=r"(r[10]),"=r"(r[11]),"=r"(r[12]),"=r"(r[13]),"=r"(r[14]),"=r"(r[15]) : "r"(a));
}
__global__ void k(int nld, int iters, long long* cyc, uint32_t* sink) {
  __shared__ uint32_t base;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"((uint32_t)__cvta_generic_to_shared(&base)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;"); __syncthreads(); asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t t = base + ((uint32_t)((warp & 3) * 32) << 16) + (warp >> 2) * 128;
  uint32_t acc = 0;
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    uint32_t r0[16], r1[16], r2[16], r3[16];
    ld16(t, r0);
    if (nld > 1) ld16(t + 16, r1);
    if (nld > 2) ld16(t + 32, r2);
    if (nld > 3) ld16(t + 48, r3);
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    acc += r0[i & 15] + (nld > 1 ? r1[3] : 0) + (nld > 2 ? r2[5] : 0) + (nld > 3 ? r3[7] : 0);
  }
  long long t1 = clock64();
  sink[threadIdx.x] = acc;
  if (threadIdx.x == 0) cyc[0] = t1 - t0;
  asm volatile("tcgen05.fence::before_thread_sync;"); __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(base));
}
int main() {
  long long* cyc; uint32_t* sink; cudaMalloc(&cyc, 8); cudaMalloc(&sink, 4096);
  for (int warps : {4, 8, 12})
    for (int nld : {1, 4}) {
      k<<<1, warps * 32>>>(nld, 1000, cyc, sink);
      k<<<1, warps * 32>>>(nld, 1000, cyc, sink);
      cudaDeviceSynchronize();
      long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
      printf("warps %2d  x16 loads in flight %d: %.1f cycles per (loads + wait) per warp iteration  err=%s\n", warps, nld,
             (double)c / 1000, cudaGetErrorString(cudaGetLastError()));
    }
  return 0;
}
