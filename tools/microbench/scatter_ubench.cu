// scatter_ubench.cu -- microbenchmark of the scatter primitives available to the CSR
// small-n aggregation (SURVEY 7 hard parts 1 and 3): random fp64 updates into an n-element
// partial w, per SM, on sm_100a.
//   mode 0: local shared atomicAdd (ATOMS.CAST.SPIN.64 CAS loop)
//   mode 1: remote DSMEM red.shared::cluster.add.f64 into the peer CTA of a 2-CTA cluster
//   mode 2: plain shared load-add-store into a per-warp private copy (no atomics)
//   mode 3: global red.add.f64 into a per-CTA slice (L2-resident)
//   mode 4: global red.add.f64 into one shared n-vector (all CTAs, L2 contention)
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/sub scatter_ubench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int N = 1000;
constexpr int BS = 256;
constexpr int ITERS = 2000;

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16; return x;
}

template <int MODE>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(BS) k(double* gout, double* gshared) {
  extern __shared__ double s[];  // MODE 2: 8 warps x N, else N
  const int tid = threadIdx.x, warp = tid >> 5;
  for (int j = tid; j < ((MODE == 2 || MODE >= 5) ? 8 * N : N); j += BS) s[j] = 0.0;
  asm volatile("barrier.cluster.arrive; barrier.cluster.wait;");
  uint32_t rank;
  asm("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  uint32_t st = hsh(blockIdx.x * BS + tid + 1);
  double* wp = s + ((MODE == 2 || MODE >= 5) ? warp * N : 0);
  for (int it = 0; it < ITERS; ++it) {
    st = hsh(st);
    const int c = st % N;
    const double v = 1.0 + (st & 7);
    if constexpr (MODE == 0) {
      atomicAdd(s + c, v);
    } else if constexpr (MODE == 1) {
      uint32_t a = (uint32_t)__cvta_generic_to_shared(s + c), ra;
      asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(a), "r"(rank ^ 1));
      asm volatile("red.shared::cluster.add.f64 [%0], %1;" ::"r"(ra), "d"(v) : "memory");
    } else if constexpr (MODE == 2) {
      // lanes of one warp may collide: serialise by lane quarter (8 lanes per round, like VS = 8)
      const int lane = tid & 31;
      for (int r = 0; r < 4; ++r) {
        if ((lane >> 3) == r) wp[c] += v;
        __syncwarp();
      }
    } else if constexpr (MODE == 5) {
      wp[c] += v;  // single round, collisions ignored (throughput ceiling only)
      __syncwarp();
    } else if constexpr (MODE == 6) {
      // tag check: winners (tag == lane) update, losers retry next round
      int* tag = reinterpret_cast<int*>(s + 8 * N) + warp * N;
      const int lane = tid & 31;
      bool pending = true;
      while (__any_sync(0xffffffffu, pending)) {
        if (pending) tag[c] = lane;
        __syncwarp();
        const bool win = pending && tag[c] == lane;
        if (win) { wp[c] += v; pending = false; }
        __syncwarp();
      }
    } else if constexpr (MODE == 3) {
      atomicAdd(gout + (size_t)blockIdx.x * N + c, v);
    } else {
      atomicAdd(gshared + c, v);
    }
  }
  asm volatile("barrier.cluster.arrive; barrier.cluster.wait;");
  double t = 0;
  for (int j = tid; j < N; j += BS) t += s[j];
  if (t == -1.0) gout[0] = t;
}

int main() {
  int sms = 148;
  const int grid = sms * 2 * 2;  // 2 clusters-worth of CTAs per SM pair ...
  double *gout, *gsh;
  cudaMalloc(&gout, (size_t)grid * N * sizeof(double));
  cudaMalloc(&gsh, N * sizeof(double));
  cudaMemset(gout, 0, (size_t)grid * N * sizeof(double));
  cudaMemset(gsh, 0, N * sizeof(double));
  const char* names[] = {"smem CAS atomicAdd f64", "DSMEM remote red f64", "private smem RMW (4 rounds)",
                         "global red f64 per-CTA slice", "global red f64 shared vector", "private RMW 1 round (ceiling)",
                         "private RMW + tag dedup"};
  for (int mode = 0; mode < 7; ++mode) {
    size_t smem = (mode == 2 || mode == 5 ? 8 * N * 8 : mode == 6 ? 8 * N * 12 : N * 8);
    void (*f)(double*, double*) = mode == 0 ? k<0> : mode == 1 ? k<1> : mode == 2 ? k<2> : mode == 3 ? k<3> : mode == 4 ? k<4> : mode == 5 ? k<5> : k<6>;
    cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    f<<<grid, BS, smem>>>(gout, gsh);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    f<<<grid, BS, smem>>>(gout, gsh);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    cudaError_t e = cudaGetLastError();
    double ups = (double)grid * BS * ITERS / (ms * 1e-3);
    printf("mode %d %-32s %8.3f ms  %7.1f G updates/s  %6.2f updates/clk/SM  %s\n", mode, names[mode], ms, ups / 1e9,
           ups / (148 * 1.9e9), cudaGetErrorString(e));
  }
  return 0;
}
