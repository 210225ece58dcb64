// read_bw.cu -- ceiling of a pure HBM read stream on this GPU (what C2's dense kernel, which
// reads X once, can at most reach).  256-bit L1::no_allocate / L2::evict_first loads, grid-stride,
// one add per element so the loads cannot be elided.  nvcc -gencode arch=compute_100a,code=sm_100a
//   -O3 -o read_bw read_bw.cu && ./read_bw
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ void ld32(const float* p, float (&r)[8]) {
  asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]), "=f"(r[6]), "=f"(r[7])
               : "l"(p));
}

template <int U>
__global__ void k_read(const float* __restrict__ x, size_t n8, float* out) {
  float acc = 0.f;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + (U - 1) * stride < n8; i += U * stride) {
    float r[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) ld32(x + (i + u * stride) * 8, r[u]);
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int e = 0; e < 8; ++e) acc += r[u][e];
  }
  for (; i < n8; i += stride) {
    float r[8];
    ld32(x + i * 8, r);
#pragma unroll
    for (int e = 0; e < 8; ++e) acc += r[e];
  }
  if (acc == 12345.f) out[0] = acc;
}

template <int U>
void run(const float* x, size_t n8, float* out, int grid, int bs) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int w = 0; w < 3; ++w) k_read<U><<<grid, bs>>>(x, n8, out);
  float best = 1e9f;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(a);
    k_read<U><<<grid, bs>>>(x, n8, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    best = ms < best ? ms : best;
  }
  printf("U=%d grid=%d bs=%d: %.3f ms  %.1f GB/s\n", U, grid, bs, best, n8 * 32.0 / best / 1e6);
}

int main() {
  const size_t bytes = 5120000000ull;  // C2's X
  const size_t n8 = bytes / 32;
  float *x, *out;
  cudaMalloc(&x, bytes);
  cudaMalloc(&out, 4);
  cudaMemset(x, 0, bytes);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int per : {2, 4, 8}) {
    run<4>(x, n8, out, sms * per, 256);
    run<8>(x, n8, out, sms * per, 256);
  }
  run<4>(x, n8, out, sms * 2, 1024);
  run<8>(x, n8, out, sms * 1, 1024);
  return 0;
}
