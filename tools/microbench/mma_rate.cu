// Microbenchmark: tcgen05.mma issue-to-completion throughput for the shapes the attention kernel
// issues (kind::f16, bf16 -> fp32, cta_group::1), one thread issuing R back-to-back MMAs into
// one accumulator then commit + wait. Reports cycles per MMA instruction.
//   SS 128x128x16 (S = Q K^T), SS 128x64x16, TS 128x64x16 (O += P V, P from TMEM), TS 128x128x16
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void wait(uint32_t b, uint32_t ph) {
  uint32_t ok = 0;
  while (!ok) asm volatile("{\n.reg .pred P;\nmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P, [%1], %2;\nselp.u32 %0,1,0,P;\n}" : "=r"(ok) : "r"(b), "r"(ph) : "memory");
}
template <int TS, int N>
__global__ void k(long long* out, int reps) {
  __shared__ uint64_t b0;
  __shared__ uint32_t tbase;
  __shared__ __align__(1024) uint8_t sm[32768];
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(&b0)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" :: "r"(su(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;"); __syncthreads(); asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tb = tbase;
  const uint32_t a = su(sm);
  const uint64_t desc = ((uint64_t)((a >> 4) & 0x3FFF)) | ((uint64_t)1 << 16) | ((uint64_t)64 << 32) | ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((128u >> 4) << 24) | (TS ? (1u << 16) : 0u);
  long long best = 1LL << 60;
  for (int trial = 0; trial < 3; ++trial) {
    long long t0 = clock64();
    if (threadIdx.x == 0) {
      for (int i = 0; i < reps; ++i) {
        if (TS)
          asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %3, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %4, p;\n}"
                       :: "r"(tb + 256), "r"(tb + 128 + (i & 7) * 8), "l"(desc + (i & 3) * 128), "r"(i), "r"(idesc) : "memory");
        else
          asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                       :: "r"(tb + (i & 1) * 128), "l"(desc + (i & 3) * 2), "l"(desc + (i & 3) * 2), "r"(idesc), "r"(i) : "memory");
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su(&b0)) : "memory");
      wait(su(&b0), trial & 1);
    }
    long long t1 = clock64();
    if (t1 - t0 < best) best = t1 - t0;
  }
  if (threadIdx.x == 0) out[0] = best;
  asm volatile("tcgen05.fence::before_thread_sync;"); __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" :: "r"(tb));
}
template <int TS, int N>
void run(const char* name, long long* o) {
  for (int reps : {4, 8, 64, 512}) {
    k<TS, N><<<1, 128>>>(o, reps);
    cudaError_t e = cudaDeviceSynchronize();
    long long h;
    cudaMemcpy(&h, o, 8, cudaMemcpyDeviceToHost);
    const double flops = 2.0 * 128 * N * 16 * reps;
    printf("%-18s reps=%4d  %7lld cycles  %6.1f cyc/MMA  %6.0f flop/clk (%s)\n", name, reps, h, (double)h / reps,
           flops / h, cudaGetErrorString(e));
  }
}
int main() {
  long long* o; cudaMalloc(&o, 64);
  run<0, 128>("SS 128x128x16", o);
  run<0, 64>("SS 128x64x16", o);
  run<0, 256>("SS 128x256x16", o);
  run<1, 64>("TS 128x64x16", o);
  run<1, 128>("TS 128x128x16", o);
  return 0;
}
