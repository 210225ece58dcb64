// probe.cu -- fp_probe_rates: live throughput of the random on-chip accesses that bound the
// CSR paths (SURVEY 8(d) C4 "second ceiling": y gathers and w updates hitting L1/L2 instead
// of streaming from HBM).  Measurement support for bench.py's roofline report; the same
// access patterns as tools/microbench/{l2_scatter,smem_scatter2}.cu, timed with CUDA events.
//   rate[0]  random 4-byte gathers from an n-element fp32 vector in global memory (L1/L2)
//   rate[1]  random fp32 red.global.add into an n-element vector (the per-nonzero scatter of
//            variants 4/7/16)
//   rate[2]  random native 32-bit shared-memory atomic adds (variant 17's consumer)
//   rate[3]  random fp64 shared-memory atomicAdd (a CAS loop on sm_100a; variant 3's partial)
//   rate[4]  random 8-byte shared-memory gathers (fp64 y staged in smem, variant 3)
// Each in operations per second over the whole device at full occupancy.
#include "common.cuh"

namespace {

constexpr int kPBS = 512;
constexpr int kPIters = 1024;

template <int MODE>
__global__ void __launch_bounds__(kPBS) k_probe(const float* __restrict__ y, float* w, int n, int nsm,
                                               float* sink) {
  extern __shared__ __align__(16) unsigned char sm[];
  uint32_t* su = reinterpret_cast<uint32_t*>(sm);
  double* sd = reinterpret_cast<double*>(sm);
  if constexpr (MODE >= 2) {
    for (int j = threadIdx.x; j < nsm; j += kPBS) {
      if constexpr (MODE == 2) su[j] = 0;
      else sd[j] = 0.0;
    }
    __syncthreads();
  }
  uint32_t st = (blockIdx.x * kPBS + threadIdx.x) * 2654435761u + 12345u;
  float acc = 0.f;
  double accd = 0.0;
  const int range = MODE >= 2 ? nsm : n;
#pragma unroll 8
  for (int it = 0; it < kPIters; ++it) {
    st = st * 1664525u + 1013904223u;
    const int c = (int)(((uint64_t)(st >> 8) * (uint64_t)range) >> 24);
    if constexpr (MODE == 0) acc += __ldg(y + c);
    else if constexpr (MODE == 1) atomicAdd(w + c, (float)(st & 7));
    else if constexpr (MODE == 2) atomicAdd(su + c, st & 0xffu);
    else if constexpr (MODE == 3) atomicAdd(sd + c, (double)(st & 7));
    else accd += sd[c];
  }
  if constexpr (MODE >= 2) {
    __syncthreads();
    acc += (float)su[threadIdx.x] + (float)accd;
  }
  if (acc == -1.2345f) sink[0] = acc;
}

template <int MODE>
double run_probe(const float* y, float* w, int n, int nsm, float* sink, cudaStream_t s) {
  const size_t smem = MODE >= 2 ? (size_t)nsm * (MODE == 2 ? 4 : 8) : 0;
  fp::set_max_dynamic_smem((const void*)k_probe<MODE>);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_probe<MODE>, kPBS, smem);
  const int sms = fp::device_info(fp::current_device()).sm_count;
  const int grid = sms * (occ > 0 ? occ : 1) * 2;
  k_probe<MODE><<<grid, kPBS, smem, s>>>(y, w, n, nsm, sink);  // warm-up
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a, s);
  k_probe<MODE><<<grid, kPBS, smem, s>>>(y, w, n, nsm, sink);
  cudaEventRecord(b, s);
  cudaEventSynchronize(b);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, a, b);
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  return ms > 0.f ? (double)grid * kPBS * kPIters / (ms * 1e-3) : 0.0;
}

}  // namespace

extern "C" fp_status fp_probe_rates(int64_t n, int64_t smem_elems, double* rates, fp_stream stream) {
  FP_REQUIRE(rates && n > 0 && n <= (1 << 30) && smem_elems > 0 && smem_elems * 8 <= 200 * 1024, FP_ERR_INVALID_ARG,
             "fp_probe_rates: bad arguments (0 < n <= 2^30, 0 < smem_elems <= 25600)");
  cudaStream_t s = (cudaStream_t)stream;
  float* buf = nullptr;
  FP_CUDA(cudaMallocAsync((void**)&buf, (size_t)(2 * n + 16) * sizeof(float), s));
  FP_CUDA(cudaMemsetAsync(buf, 0, (size_t)(2 * n + 16) * sizeof(float), s));
  const float* y = buf;
  float* w = buf + n;
  float* sink = buf + 2 * n;
  const int N = (int)n, S = (int)smem_elems;
  rates[0] = run_probe<0>(y, w, N, S, sink, s);
  rates[1] = run_probe<1>(y, w, N, S, sink, s);
  rates[2] = run_probe<2>(y, w, N, S, sink, s);
  rates[3] = run_probe<3>(y, w, N, S, sink, s);
  rates[4] = run_probe<4>(y, w, N, S, sink, s);
  FP_CUDA(cudaFreeAsync(buf, s));
  FP_CUDA(cudaStreamSynchronize(s));
  return FP_OK;
}
