// Microbenchmark: issue cost of single synchronisation operations on an uncontended path
// (barrier phase already complete), one warp per SMSP, as used per tile by the softmax warps.
//   E try_wait.parity.acquire (complete)   F test_wait.parity.acquire (complete)
//   G try_wait.parity.relaxed (complete)   H mbarrier.arrive.release
//   I tcgen05.fence::before + __syncwarp   J 4 x tcgen05.ld 32x32b.x16 + wait::ld
//   K ld.shared.v4                          L empty loop
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int MODE>
__device__ __forceinline__ uint32_t op(uint32_t b, uint32_t tb, uint32_t& acc) {
  uint32_t ok = 0;
  if (MODE == 0) asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(ok) : "r"(b), "r"(1) : "memory");
  if (MODE == 1) asm volatile("{\n.reg .pred P;\nmbarrier.test_wait.parity.acquire.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(ok) : "r"(b), "r"(1) : "memory");
  if (MODE == 2) asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.relaxed.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(ok) : "r"(b), "r"(1) : "memory");
  if (MODE == 3) { if ((threadIdx.x & 31) == 0) asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" :: "r"(b + 8) : "memory"); ok = 1; }
  if (MODE == 4) { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); __syncwarp(); ok = 1; }
  if (MODE == 5) {
    uint32_t r[16];
    for (int q = 0; q < 4; ++q) {
      asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                   : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                     "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                   : "r"(tb + q * 16));
      acc += r[0] + r[15];
    }
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    ok = 1;
  }
  if (MODE == 6) { uint32_t x, y, z, w; asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(x), "=r"(y), "=r"(z), "=r"(w) : "r"(b + 16)); acc += x + w; ok = 1; }
  if (MODE == 7) ok = 1;
  return ok;
}
template <int MODE>
__global__ void k(long long* out, int iters) {
  __shared__ __align__(16) uint64_t bars[4 * 16];
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x >> 5;
  uint64_t* mine = bars + 4 * warp;
  if ((threadIdx.x & 31) == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(mine)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1000000;" :: "r"(su(mine + 1)));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" :: "r"(su(mine)) : "memory");  // phase 0 done
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(su(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;"); __syncthreads(); asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tbase + ((uint32_t)((warp & 3) * 32) << 16);
  uint32_t acc = 0, okc = 0;
  __syncwarp();
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) okc += op<MODE>(su(mine), tb, acc);
  long long t1 = clock64();
  if ((threadIdx.x & 31) == 0) out[warp] = (t1 - t0) / iters + (acc == 12345 && okc == 7 ? 1 : 0);
  asm volatile("tcgen05.fence::before_thread_sync;"); __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tbase));
}
template <int MODE>
void run(const char* name, long long* o) {
  long long h[16];
  for (int nw : {1, 4, 8}) {
    k<MODE><<<1, 32 * nw>>>(o, 4000);
    cudaError_t e = cudaDeviceSynchronize();
    cudaMemcpy(h, o, 8 * nw, cudaMemcpyDeviceToHost);
    printf("%-40s warps=%d  %lld cycles/op  (%s)\n", name, nw, h[0], cudaGetErrorString(e));
  }
}
int main() {
  long long* o; cudaMalloc(&o, 256);
  run<0>("E try_wait.acquire (complete)", o);
  run<1>("F test_wait.acquire (complete)", o);
  run<2>("G try_wait.relaxed (complete)", o);
  run<3>("H arrive.release", o);
  run<4>("I tcgen05.fence::before + syncwarp", o);
  run<5>("J 4x tcgen05.ld x16 + wait::ld", o);
  run<6>("K ld.shared.v4", o);
  run<7>("L empty loop", o);
  return 0;
}
