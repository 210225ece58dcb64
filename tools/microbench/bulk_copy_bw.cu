// bulk_copy_bw.cu -- microbenchmark: HBM->SMEM streaming bandwidth of cp.async.bulk (one
// elected thread issues copies of S bytes into a D-deep ring, completion on mbarriers) versus
// plain 16/32-byte LDG, as a function of copy size, ring depth and CTAs per SM.  Used to size
// the wide-row cluster kernel's ring.  nvcc -arch=sm_100a -O3.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned su32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

__global__ void k_bulk(const char* src, size_t total, int S, int D, float* sink) {
  extern __shared__ __align__(128) char buf[];
  __shared__ uint64_t bar[16];
  const size_t nchunk = total / S;
  if (threadIdx.x == 0) {
    for (int i = 0; i < D; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[i])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  auto issue = [&](size_t c, int b) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[b])), "r"(S) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     su32(buf + (size_t)b * S)),
                 "l"(src + c * S), "r"(S), "r"(su32(&bar[b]))
                 : "memory");
  };
  size_t c0 = blockIdx.x;
  const size_t step = gridDim.x;
  if (threadIdx.x == 0)
    for (int i = 0; i < D; ++i)
      if (c0 + i * step < nchunk) issue(c0 + i * step, i);
  float acc = 0.f;
  unsigned ph[16] = {0};
  int b = 0;
  for (size_t c = c0; c < nchunk; c += step) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}" ::"r"(
            su32(&bar[b])),
        "r"(ph[b])
        : "memory");
    ph[b] ^= 1;
    const float4* f = (const float4*)(buf + (size_t)b * S);
    for (int i = threadIdx.x; i < S / 16; i += blockDim.x) {
      float4 t = f[i];
      acc += t.x + t.y + t.z + t.w;
    }
    __syncthreads();
    if (threadIdx.x == 0 && c + D * step < nchunk) issue(c + D * step, b);
    b = (b + 1 == D) ? 0 : b + 1;
  }
  if (acc == 12345.f) sink[0] = acc;
}

__global__ void k_ldg(const float4* src, size_t n4, float* sink) {
  float acc = 0.f;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
    float4 t;
    asm("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(t.x), "=f"(t.y), "=f"(t.z), "=f"(t.w) : "l"(src + i));
    acc += t.x + t.y + t.z + t.w;
  }
  if (acc == 12345.f) sink[0] = acc;
}

int main() {
  const size_t total = (size_t)4 << 30;
  char* d;
  float* sink;
  cudaMalloc(&d, total);
  cudaMalloc(&sink, 4);
  cudaMemset(d, 0, total);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaFuncSetAttribute(k_bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  float ms;
  for (int bps : {1, 2, 4}) {
    k_ldg<<<sms * bps * 4, 256>>>((const float4*)d, total / 16, sink);
    cudaEventRecord(e0);
    k_ldg<<<sms * bps * 4, 256>>>((const float4*)d, total / 16, sink);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("ldg16 grid=%d: %.0f GB/s\n", sms * bps * 4, total / ms / 1e6);
  }
  for (int S : {4096, 8192, 16384, 32768, 65536})
    for (int D : {2, 3, 4, 6})
      for (int bps : {1, 2}) {
        size_t smem = (size_t)S * D;
        if (smem * bps > 220 * 1024) continue;
        k_bulk<<<sms * bps, 256, smem>>>(d, total, S, D, sink);
        cudaEventRecord(e0);
        k_bulk<<<sms * bps, 256, smem>>>(d, total, S, D, sink);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        cudaError_t err = cudaGetLastError();
        cudaEventElapsedTime(&ms, e0, e1);
        printf("bulk S=%6d D=%d ctas/sm=%d: %.0f GB/s %s\n", S, D, bps, total / ms / 1e6,
               err ? cudaGetErrorString(err) : "");
      }
  return 0;
}
