// Microbenchmark for the fine (CSR) kernel's ceiling on B200:
//   (1) gather bandwidth of random 128-byte K and V rows within a head (the C4 pattern:
//       32 heads x 16384 rows, 164 random columns per row, K+V = 4 MB per head, L2-resident),
//       for several lane-to-row mappings; no arithmetic beyond an XOR to keep the loads live;
//   (2) legacy mma.sync m16n8k16 bf16 throughput per SM (the fine kernel's tensor-core option).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_bw gather_bw.cu
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

constexpr int L = 16384, BH = 32, NNZ = 164, D = 64;

__device__ __forceinline__ int4 ldv4(const void* p) {
  int4 r;
  asm volatile("ld.global.nc.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// LPR lanes per row: each lane loads 128/LPR bytes of the K row and of the V row
template <int LPR>
__global__ void __launch_bounds__(256) gather(const uint16_t* K, const uint16_t* V, const int* cols, int* out) {
  const int lane = threadIdx.x & 31;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= BH * L) return;
  const int bh = gw / L, r = gw % L;
  const uint16_t* Kb = K + (size_t)bh * L * D;
  const uint16_t* Vb = V + (size_t)bh * L * D;
  const int* c = cols + (size_t)r * NNZ;
  constexpr int RPI = 32 / LPR;       // rows per warp instruction
  constexpr int V4 = 8 / LPR;         // 16-byte loads per lane per row
  const int sub = lane / LPR, part = lane % LPR;
  int acc = 0;
  for (int base = 0; base < NNZ; base += 32) {
    const int col = base + lane < NNZ ? __ldg(c + base + lane) : -1;
#pragma unroll
    for (int s = 0; s < 32 / RPI; ++s) {
      const int cc = __shfl_sync(0xffffffffu, col, s * RPI + sub);
      if (cc >= 0) {
#pragma unroll
        for (int u = 0; u < V4; ++u) {
          const int4 a = ldv4(Kb + (size_t)cc * D + part * (8 * V4) + u * 8);
          const int4 b = ldv4(Vb + (size_t)cc * D + part * (8 * V4) + u * 8);
          acc ^= a.x ^ a.y ^ a.z ^ a.w ^ b.x ^ b.y ^ b.z ^ b.w;
        }
      }
    }
  }
  if (acc == 0x12345678) out[gw] = acc;
}

// same gathers through cp.async.cg into a warp-private shared-memory ring (NS stages), lane-private
// chunks read back with ld.shared after cp.async.wait_group
template <int LPR, int NS>
__global__ void __launch_bounds__(128) gather_cpasync(const uint16_t* K, const uint16_t* V, const int* cols, int* out) {
  extern __shared__ __align__(16) uint8_t sm[];
  const int lane = threadIdx.x & 31;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (gw >= BH * L) return;
  const int bh = gw / L, r = gw % L;
  const uint16_t* Kb = K + (size_t)bh * L * D;
  const uint16_t* Vb = V + (size_t)bh * L * D;
  const int* c = cols + (size_t)r * NNZ;
  constexpr int RPI = 32 / LPR, V4 = 8 / LPR;
  constexpr int CH = 2 * V4 * (32 / RPI) / 4;   // 16-byte chunks per lane per quarter-window (8 rows)
  const int sub = lane / LPR, part = lane % LPR;
  const uint32_t ring = (uint32_t)__cvta_generic_to_shared(sm) + (threadIdx.x >> 5) * NS * CH * 512 + lane * 16;
  int acc = 0;
  // a "step" = 8 rows of the 32-index window
  const int nsteps = (NNZ + 7) / 8;
  auto issue = [&](int s) {
    if (s < nsteps) {
      const int idx = s * 8 + (lane & 7);
      const int col = idx < NNZ ? __ldg(c + idx) : 0;
      const uint32_t dst = ring + (s % NS) * CH * 512;
      int k = 0;
#pragma unroll
      for (int q = 0; q < 8 / RPI; ++q) {
        const int cc = __shfl_sync(0xffffffffu, col, q * RPI + sub);
#pragma unroll
        for (int u = 0; u < V4; ++u) {
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst + (k++) * 512), "l"(Kb + (size_t)cc * D + part * (8 * V4) + u * 8) : "memory");
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst + (k++) * 512), "l"(Vb + (size_t)cc * D + part * (8 * V4) + u * 8) : "memory");
        }
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  for (int s = 0; s < NS - 1; ++s) issue(s);
  for (int s = 0; s < nsteps; ++s) {
    issue(s + NS - 1);
    asm volatile("cp.async.wait_group %0;" ::"n"(NS - 1) : "memory");
    const uint32_t src = ring + (s % NS) * CH * 512;
#pragma unroll
    for (int k = 0; k < CH; ++k) {
      int4 v;
      asm volatile("ld.shared.v4.s32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(src + k * 512));
      acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
  }
  if (acc == 0x12345678) out[gw] = acc;
}

__global__ void mma_rate(float* out, int iters) {
  uint32_t a0 = threadIdx.x, a1 = a0 * 3, a2 = a0 * 5, a3 = a0 * 7, b0 = a0 ^ 9, b1 = a0 ^ 11;
  float c[8][4] = {};
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j)
      asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                   : "+f"(c[j][0]), "+f"(c[j][1]), "+f"(c[j][2]), "+f"(c[j][3])
                   : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
  }
  float s = 0;
  for (int j = 0; j < 8; ++j) s += c[j][0] + c[j][1] + c[j][2] + c[j][3];
  if (s == 1.2345f) out[0] = s;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  size_t n = (size_t)BH * L * D;
  uint16_t *K, *V;
  int *cols, *out;
  cudaMalloc(&K, n * 2);
  cudaMalloc(&V, n * 2);
  cudaMemset(K, 1, n * 2);
  cudaMemset(V, 2, n * 2);
  std::vector<int> hc((size_t)L * NNZ);
  srand(1);
  for (auto& x : hc) x = rand() % L;
  cudaMalloc(&cols, hc.size() * 4);
  cudaMemcpy(cols, hc.data(), hc.size() * 4, cudaMemcpyHostToDevice);
  cudaMalloc(&out, (size_t)BH * L * 4);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const double bytes = (double)BH * L * NNZ * 256;
  auto run = [&](auto kern, const char* name) {
    const int blocks = BH * L / 8;
    for (int i = 0; i < 3; ++i) kern<<<blocks, 256>>>(K, V, cols, out);
    cudaEventRecord(e0);
    for (int i = 0; i < 10; ++i) kern<<<blocks, 256>>>(K, V, cols, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    ms /= 10;
    printf("%-28s %.3f ms  %.0f GB/s gathered (%s)\n", name, ms, bytes / ms / 1e6,
           cudaGetErrorString(cudaGetLastError()));
  };
  run(gather<8>, "8 lanes/row (16 B each)");
  run(gather<4>, "4 lanes/row (32 B each)");
  run(gather<2>, "2 lanes/row (64 B each)");
  run(gather<1>, "1 lane/row (128 B each)");
  auto runc = [&](auto kern, int ns, int lpr, const char* name) {
    const int CH = 2 * (8 / lpr) * (lpr * 8 / 32 > 0 ? lpr * 8 / 32 : 1) ;
    const int smem = 4 * ns * 4 * 512;   // 4 warps x NS stages x 4 chunks x 512 B
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const int blocks = BH * L / 4;
    for (int i = 0; i < 3; ++i) kern<<<blocks, 128, smem>>>(K, V, cols, out);
    cudaEventRecord(e0);
    for (int i = 0; i < 10; ++i) kern<<<blocks, 128, smem>>>(K, V, cols, out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    ms /= 10;
    (void)CH;
    printf("%-28s %.3f ms  %.0f GB/s gathered (%s, smem %d)\n", name, ms, bytes / ms / 1e6,
           cudaGetErrorString(cudaGetLastError()), smem);
  };
  runc(gather_cpasync<8, 2>, 2, 8, "cp.async 8 lanes/row NS=2");
  runc(gather_cpasync<8, 4>, 4, 8, "cp.async 8 lanes/row NS=4");
  runc(gather_cpasync<4, 4>, 4, 4, "cp.async 4 lanes/row NS=4");
  runc(gather_cpasync<8, 8>, 8, 8, "cp.async 8 lanes/row NS=8");
  float* f;
  cudaMalloc(&f, 64);
  for (int warps = 4; warps <= 32; warps *= 2) {
    const int iters = 4096;
    mma_rate<<<sms, warps * 32>>>(f, 16);
    cudaEventRecord(e0);
    mma_rate<<<sms, warps * 32>>>(f, iters);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double flops = (double)sms * warps * iters * 8 * 4096;
    printf("mma.sync m16n8k16 bf16, %2d warps/SM: %.1f TFLOP/s (%.2f SM-clk per mma per SM at 1.965 GHz)\n", warps,
           flops / ms / 1e9, (ms * 1e-3 * 1.965e9) / ((double)warps * iters * 8));
  }
  return 0;
}
