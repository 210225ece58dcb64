// cluster_xchg.cu -- microbenchmark: latency of one all-to-all exchange of a scalar among the CTAs
// of a thread-block cluster, per round: (a) barrier.cluster arrive.release/wait.acquire only;
// (b) DSMEM store to every peer + that barrier; (c) st.async to every peer with mbarrier
// complete_tx (one-way signal, 4-deep slots, no cluster barrier).  Sizes the exchange of the
// wide-row dense kernel.  nvcc -arch=sm_100a -O3.
#include <cooperative_groups.h>
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
namespace cg = cooperative_groups;

__device__ __forceinline__ unsigned su32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

template <int MODE>
__global__ void k_xchg(int rounds, float* out) {
  cg::cluster_group cl = cg::this_cluster();
  const int cs = (int)cl.num_blocks(), rank = (int)cl.block_rank(), tid = threadIdx.x;
  __shared__ float slot[4][16];
  __shared__ uint64_t bar[4];
  if (tid == 0)
    for (int b = 0; b < 4; ++b) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[b])));
  asm volatile("fence.mbarrier_init.release.cluster;");
  cl.sync();
  if (MODE == 2 && tid == 0)
    for (int b = 0; b < 4; ++b)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[b])), "r"(cs * 4));
  float acc = 0.f;
  unsigned ph = 0;
  for (int i = 0; i < rounds; ++i) {
    const int s = i & 3;
    const float val = (float)(i + rank);
    if (MODE == 0) {
      asm volatile("barrier.cluster.arrive.release.aligned;\n" ::: "memory");
      asm volatile("barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
    } else if (MODE == 1) {
      if (tid < cs) *cl.map_shared_rank(&slot[s][rank], tid) = val;
      asm volatile("barrier.cluster.arrive.release.aligned;\n" ::: "memory");
      asm volatile("barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
      acc += slot[s][0];
    } else {
      if (tid < cs) {
        unsigned la = su32(&slot[s][rank]), lb = su32(&bar[s]), ra, rb;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(la), "r"(tid));
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(rb) : "r"(lb), "r"(tid));
        asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b32 [%0], %1, [%2];" ::"r"(ra),
                     "r"(__float_as_uint(val)), "r"(rb)
                     : "memory");
      }
      asm volatile(
          "{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n\t@!p bra "
          "W_%=;\n\t}" ::"r"(su32(&bar[s])),
          "r"((ph >> s) & 1u)
          : "memory");
      ph ^= 1u << s;
      acc += slot[s][0];
      __syncthreads();  // everyone read slot s before re-arming it
      if (tid == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(cs * 4));
    }
  }
  cl.sync();
  if (acc == -1.f) out[0] = acc;
}

template <int MODE>
float run(int cs, int sms, float* out) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((sms / cs) * cs);
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = 150 * 1024;  // one CTA per SM
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = cs;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cudaFuncSetAttribute(k_xchg<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, 150 * 1024);
  const int rounds = 20000;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaLaunchKernelEx(&cfg, k_xchg<MODE>, rounds, out);
  cudaEventRecord(e0);
  cudaLaunchKernelEx(&cfg, k_xchg<MODE>, rounds, out);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaError_t err = cudaGetLastError();
  if (err) printf("error %s\n", cudaGetErrorString(err));
  return ms * 1e6f / rounds;
}

int main() {
  float* out;
  cudaMalloc(&out, 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int cs : {2, 4, 8})
    printf("cs=%d  barrier: %.0f ns  dsmem+barrier: %.0f ns  st.async+mbarrier: %.0f ns\n", cs, run<0>(cs, sms, out),
           run<1>(cs, sms, out), run<2>(cs, sms, out));
  return 0;
}
