// dsmem_ubench.cu -- random-address DSMEM throughput on sm_100a, for a cluster-distributed
// C4 design (y and the partial w of n = 1e5 spread over the shared memory of a cluster):
//   0: ld.shared::cluster.u32 random gather, uniform over the cluster's CTAs (incl. own)
//   1: red.shared::cluster.add.u32 random (no return)
//   2: atom.shared::cluster.add.u32 random (with return)
//   3: local ld.shared.u32 random (reference)
//   4: local atom.shared.add.u32 (reference, no return)
// Template CS = cluster size; 1 CTA of 512 threads per SM, 160 KB smem window per CTA.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/dsm dsmem_ubench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int BS = 512;
constexpr int ITERS = 2048;
constexpr int WORDS = 40960;  // 160 KB per CTA

template <int CS, int MODE>
__global__ void __launch_bounds__(BS) k(unsigned* gout) {
  extern __shared__ __align__(16) uint32_t sm[];
  for (int j = threadIdx.x; j < WORDS; j += BS) sm[j] = j;
  asm volatile("barrier.cluster.arrive.release; barrier.cluster.wait.acquire;" ::: "memory");
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
  uint32_t rbase[CS];
#pragma unroll
  for (int r = 0; r < CS; ++r) asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(rbase[r]) : "r"(base), "r"(r));
  uint32_t st = (blockIdx.x * BS + threadIdx.x) * 2654435761u + 12345u;
  uint32_t acc = 0;
#pragma unroll 8
  for (int it = 0; it < ITERS; ++it) {
    st = st * 1664525u + 1013904223u;
    const uint32_t w = (uint32_t)(((uint64_t)(st >> 8) * (WORDS * CS)) >> 24);
    const uint32_t r = w / WORDS, o = w - r * WORDS;
    uint32_t ra = 0;
#pragma unroll
    for (int q = 0; q < CS; ++q) ra = (r == q) ? rbase[q] : ra;
    ra += o * 4;
    if constexpr (MODE == 0) {
      uint32_t v;
      asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(ra));
      acc += v;
    } else if constexpr (MODE == 1) {
      asm volatile("red.shared::cluster.add.u32 [%0], %1;" ::"r"(ra), "r"(st & 0xffu) : "memory");
    } else if constexpr (MODE == 2) {
      uint32_t v;
      asm volatile("atom.shared::cluster.add.u32 %0, [%1], %2;" : "=r"(v) : "r"(ra), "r"(st & 0xffu) : "memory");
      acc += v;
    } else if constexpr (MODE == 3) {
      acc += sm[o];
    } else {
      atomicAdd(sm + o, st & 0xffu);
    }
  }
  asm volatile("barrier.cluster.arrive.release; barrier.cluster.wait.acquire;" ::: "memory");
  if (acc == 0x12345678u) gout[0] = acc;
}

template <int CS, int MODE>
void run(int sms, int clk, unsigned* g, const char* name) {
  auto f = k<CS, MODE>;
  const int smem = WORDS * 4;
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (CS > 8) cudaFuncSetAttribute(f, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = CS;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cfg.blockDim = dim3(BS);
  cfg.dynamicSmemBytes = smem;
  int ncl = 0;
  cfg.gridDim = dim3(CS);
  cudaOccupancyMaxActiveClusters(&ncl, f, &cfg);
  cfg.gridDim = dim3(ncl * CS);
  cudaLaunchKernelEx(&cfg, f, g);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  cudaLaunchKernelEx(&cfg, f, g);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  cudaError_t e = cudaGetLastError();
  const double ops = (double)ncl * CS * BS * ITERS / (ms * 1e-3);
  printf("CS %2d %-36s clusters %3d  %8.3f ms  %8.1f G ops/s  %6.2f ops/clk/SM(active)  %s\n", CS, name, ncl, ms,
         ops / 1e9, ops / ((double)ncl * CS * clk * 1e3), cudaGetErrorString(e));
}

int main() {
  int sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  unsigned* g;
  cudaMalloc(&g, 64);
  run<1, 3>(sms, clk, g, "local LDS random");
  run<1, 4>(sms, clk, g, "local ATOMS.ADD random");
  run<2, 0>(sms, clk, g, "DSMEM ld random");
  run<2, 1>(sms, clk, g, "DSMEM red.add.u32 random");
  run<2, 2>(sms, clk, g, "DSMEM atom.add.u32 random (ret)");
  run<4, 0>(sms, clk, g, "DSMEM ld random");
  run<4, 1>(sms, clk, g, "DSMEM red.add.u32 random");
  run<4, 2>(sms, clk, g, "DSMEM atom.add.u32 random (ret)");
  run<8, 0>(sms, clk, g, "DSMEM ld random");
  run<8, 1>(sms, clk, g, "DSMEM red.add.u32 random");
  return 0;
}
