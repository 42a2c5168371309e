// Microbenchmark: round-trip latencies of the synchronisation primitives the attention kernel uses.
//   A: mbarrier ping-pong between two warps (arrive -> try_wait wake-up), per handoff
//   B: tcgen05.commit (no MMA outstanding) -> mbarrier, observed by another warp
//   C: tcgen05.st x8 + tcgen05.wait::st
//   D: tcgen05.mma 128x128x16 (4 issued) + commit -> wait (same thread)
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void arrive(uint32_t b) { asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" :: "r"(b) : "memory"); }
__device__ __forceinline__ void wait(uint32_t b, uint32_t ph) {
  uint32_t ok = 0;
  while (!ok) asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(ok) : "r"(b), "r"(ph) : "memory");
}
__global__ void k(long long* out, int iters) {
  __shared__ uint64_t b0, b1, b2;
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&b0)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&b1)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&b2)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(su(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;"); __syncthreads(); asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tbase;
  // A: ping-pong warp 0 <-> warp 1 via b0 (0->1) and b1 (1->0)
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    if (warp == 0) { if (lane == 0) arrive(su(&b0)); wait(su(&b1), i & 1); }
    if (warp == 1) { wait(su(&b0), i & 1); if (lane == 0) arrive(su(&b1)); }
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (t1 - t0) / (2 * iters);
  __syncthreads();
  // B: warp 0 lane 0 commits (nothing outstanding) -> b2; warp 1 waits, then signals back via b0
  t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    if (warp == 0) {
      if (lane == 0) asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(&b2)) : "memory");
      wait(su(&b1), (iters + i) & 1);
    }
    if (warp == 1) { wait(su(&b2), i & 1); if (lane == 0) arrive(su(&b1)); }
  }
  t1 = clock64();
  if (threadIdx.x == 0) out[1] = (t1 - t0) / iters;
  __syncthreads();
  // C: tcgen05.st x8 + wait::st (warp 0)
  t0 = clock64();
  if (warp == 0)
    for (int i = 0; i < iters; ++i) {
      asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1};" :: "r"(tb + 256), "r"(i) : "memory");
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    }
  t1 = clock64();
  if (threadIdx.x == 0) out[2] = (t1 - t0) / iters;
  __syncthreads();
  // D: 4 x tcgen05.mma 128x128x16 (zero smem descriptors -> garbage values, timing only) + commit + wait
  __shared__ __align__(1024) uint8_t sm[32768];
  const uint32_t a = su(sm);
  const uint64_t desc = ((uint64_t)((a >> 4) & 0x3FFF)) | ((uint64_t)1 << 16) | ((uint64_t)64 << 32) | ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((128u >> 3) << 17) | ((128u >> 4) << 24);
  t0 = clock64();
  if (warp == 0 && lane == 0)
    for (int i = 0; i < iters; ++i) {
      for (int kk = 0; kk < 4; ++kk)
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}" :: "r"(tb), "l"(desc + kk * 2), "l"(desc + kk * 2), "r"(idesc), "r"(kk) : "memory");
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(&b2)) : "memory");
      wait(su(&b2), (iters + i) & 1);
    }
  t1 = clock64();
  if (threadIdx.x == 0) out[3] = (t1 - t0) / iters;
  asm volatile("tcgen05.fence::before_thread_sync;"); __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tb));
}
int main() {
  long long* o; cudaMalloc(&o, 64);
  k<<<1, 64>>>(o, 2000); k<<<1, 64>>>(o, 2000);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[4]; cudaMemcpy(h, o, 32, cudaMemcpyDeviceToHost);
  printf("err=%s\nA mbarrier handoff warp->warp: %lld cycles\nB commit(no mma)->mbarrier->other warp->back: %lld cycles per round trip\nC tcgen05.st x8 + wait::st: %lld cycles\nD 4x mma 128x128x16 + commit + wait: %lld cycles\n",
         cudaGetErrorString(e), h[0], h[1], h[2], h[3]);
  return 0;
}
