// smem_scatter2.cu -- throughput ceilings of the on-chip scatter/gather primitives that bound
// the CSR small-n path (C3: n = 1000 fp64 partial w and y in shared memory), at full occupancy
// (48 warps/SM), addresses from a 1-multiply LCG so that address math is not the bound.
//   0: LDS.64 random gather (y[col])
//   1: fp64 shared atomicAdd (ATOMS.CAST.SPIN.64 CAS loop)
//   2: u32 shared atomicAdd (native ATOMS.ADD), one word per update
//   3: 64-bit fixed point as two u32 ATOMS.ADD (lo with return for the carry, then hi)
//   4: fp32 shared atomicAdd (CAS)
//   5: plain LDS.64+STS.64 RMW (collisions ignored; ceiling only)
//   6: u32 ATOMS.ADD x2 without return (lo, hi; carry-free limb form)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ss2 smem_scatter2.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int N = 1000;
constexpr int BS = 512;
constexpr int ITERS = 4096;

template <int MODE>
__global__ void __launch_bounds__(BS) k(double* gout) {
  __shared__ __align__(16) unsigned char raw[N * 8 * 2];
  double* s = reinterpret_cast<double*>(raw);
  uint32_t* lo = reinterpret_cast<uint32_t*>(raw);
  uint32_t* hi = lo + N;
  const int tid = threadIdx.x;
  for (int j = tid; j < 2 * N; j += BS) s[j] = 0.0;
  __syncthreads();
  uint32_t st = (blockIdx.x * BS + tid) * 2654435761u + 12345u;
  double acc = 0;
#pragma unroll 4
  for (int it = 0; it < ITERS; ++it) {
    st = st * 1664525u + 1013904223u;
    const int c = (int)(((st >> 16) * N) >> 16);
    const double v = (double)(int)(st & 15) - 7.5;
    if constexpr (MODE == 0) {
      acc += s[c];
    } else if constexpr (MODE == 1) {
      atomicAdd(s + c, v);
    } else if constexpr (MODE == 2) {
      atomicAdd(lo + c, st & 0xffffu);
    } else if constexpr (MODE == 3) {
      const long long T = (long long)(v * 0x1p40);
      const uint32_t l = (uint32_t)T;
      const uint32_t h = (uint32_t)(T >> 32);
      const uint32_t old = atomicAdd(lo + c, l);
      atomicAdd(hi + c, h + (old + l < old ? 1u : 0u));
    } else if constexpr (MODE == 4) {
      atomicAdd(reinterpret_cast<float*>(raw) + c, (float)v);
    } else if constexpr (MODE == 5) {
      s[c] += v;
    } else if constexpr (MODE == 6) {
      const long long T = (long long)(v * 0x1p40);
      atomicAdd(lo + c, (uint32_t)T & 0x3fffffu);
      atomicAdd(hi + c, (uint32_t)(T >> 22));
    }
  }
  __syncthreads();
  double t = acc;
  for (int j = tid; j < N; j += BS) t += s[j];
  if (t == -1.2345) gout[0] = t;
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk = 0;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double* gout;
  cudaMalloc(&gout, 64);
  const char* names[] = {"LDS.64 random gather", "fp64 smem atomicAdd (CAS)", "u32 ATOMS.ADD",
                         "fixed64 = 2x u32 ATOMS (carry)", "fp32 smem atomicAdd (CAS)", "plain fp64 RMW (ceiling)",
                         "2x u32 ATOMS no return"};
  void (*fs[])(double*) = {k<0>, k<1>, k<2>, k<3>, k<4>, k<5>, k<6>};
  for (int mode = 0; mode < 7; ++mode) {
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fs[mode], BS, 0);
    const int grid = sms * occ * 4;
    fs[mode]<<<grid, BS>>>(gout);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    fs[mode]<<<grid, BS>>>(gout);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    cudaError_t e = cudaGetLastError();
    double ups = (double)grid * BS * ITERS / (ms * 1e-3);
    printf("mode %d %-34s occ %d  %8.3f ms  %8.1f G ops/s  %6.2f ops/clk/SM (at %d MHz)  %s\n", mode, names[mode], occ,
           ms, ups / 1e9, ups / (sms * clk * 1e3), clk / 1000, cudaGetErrorString(e));
  }
  return 0;
}
