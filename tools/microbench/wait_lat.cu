// Microbenchmark: LATENCY of a dependent chain of mbarrier waits on already-completed phases
// (each wait's result feeds the next wait's parity), try_wait vs test_wait, vs ld.shared.
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int MODE>
__global__ void k(long long* out, int iters) {
  __shared__ __align__(16) uint64_t bars[2];
  __shared__ uint32_t word[2];
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&bars[0])));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" :: "r"(su(&bars[0])) : "memory");  // phase 0 done
    word[0] = 0;
    word[1] = 0;
  }
  __syncthreads();
  uint32_t ok = 1, acc = 0;
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    const uint32_t par = ok ^ 1;  // 0: the completed phase; data-dependent on the previous result
    if (MODE == 0)
      asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(ok) : "r"(su(&bars[0])), "r"(par) : "memory");
    if (MODE == 1)
      asm volatile("{\n.reg .pred P;\nmbarrier.test_wait.parity.acquire.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(ok) : "r"(su(&bars[0])), "r"(par) : "memory");
    if (MODE == 2)
      asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.relaxed.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(ok) : "r"(su(&bars[0])), "r"(par) : "memory");
    if (MODE == 3) { uint32_t v; asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(su(&word[0]) + par * 4)); ok = v + 1; }
    if (MODE == 4) {  // the kernel's pattern: wait loop, then branch
      uint32_t r = 0;
      while (!r) asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(r) : "r"(su(&bars[0])), "r"(par) : "memory");
      ok = r;
    }
    acc += ok;
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) out[0] = (t1 - t0) / iters + (acc == 7 ? 1 : 0);
}
template <int MODE>
void run(const char* name, long long* o) {
  k<MODE><<<1, 32>>>(o, 2000);
  cudaError_t e = cudaDeviceSynchronize();
  long long h; cudaMemcpy(&h, o, 8, cudaMemcpyDeviceToHost);
  printf("%-34s %lld cycles per dependent op (%s)\n", name, h, cudaGetErrorString(e));
}
int main() {
  long long* o; cudaMalloc(&o, 64);
  run<0>("try_wait.acquire (complete)", o);
  run<1>("test_wait.acquire (complete)", o);
  run<2>("try_wait.relaxed (complete)", o);
  run<3>("ld.shared (dependent)", o);
  run<4>("try_wait loop + branch (complete)", o);
  return 0;
}
