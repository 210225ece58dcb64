// dense_cluster.cuh -- wide-row dense kernel on a thread-block CLUSTER (included by
// dense_kernels.cuh).
//
// The paper gives up on fusion when a dense row no longer fits the registers of one vector
// (n > ~6K on Kepler: "launch two separate cuBLAS Level 2 kernels").  On sm_100a a
// cluster of CS CTAs (CS <= 8, portable) shares distributed shared memory, so the vector of
// Table 3 can span CS SMs: VS = CS * BS threads per row, each CTA owning a contiguous column
// slice of y and of the partial w in registers and streaming its slice of the row once.  Per
// row, every CTA reduces its slice's dot (warp shuffles + smem), writes the partial into a
// slot of EVERY CTA of the cluster (DSMEM stores, st.shared::cluster), and one cluster
// barrier (arrive.release / wait.acquire) later each CTA sums the CS partials in rank order
// -- all CTAs see the same p[r], scale by v[r] and scatter their slice from the same
// registers.  Slots are double-buffered by row parity, so one cluster barrier per row suffices.
// Limit: CS * BS * TL elements per row (TL <= 64 fp32 / 32 fp64): 128K fp32 / 64K fp64 at CS=8.
#pragma once
#include <cooperative_groups.h>

namespace fp {

template <typename T, int NCH, int E, int CS, int YM, int BS>
__global__ void __launch_bounds__(BS) k_dense_cluster(const DenseKArgs a) {
  namespace cg = cooperative_groups;
  cg::cluster_group cluster = cg::this_cluster();
  constexpr int NW = BS / 32;
  const T* __restrict__ X = (const T*)a.X;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int rank = (int)cluster.block_rank();
  const int64_t m = a.m, n = a.n, ld = a.ld;
  // column slice of this CTA: chunks [rank*SC, (rank+1)*SC), SC = chunks per slice
  const int64_t nchunks = (n + E - 1) / E;
  const int64_t SC = (nchunks + CS - 1) / CS;
  const int64_t c_lo = rank * SC;
  const int64_t nfull = n / E;

  __shared__ T red[NW];
  __shared__ T slot[2][CS];  // partial dots of the cluster's CTAs, by row parity

  T ly[NCH][E], lw[NCH][E];
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t c = c_lo + k * BS + tid;
      const int64_t col = c * E + e;
      ly[k][e] = (YM != 0 && c < c_lo + SC && col < n) ? y[col] : T(0);
      lw[k][e] = T(0);
    }
  cluster.sync();  // all CTAs resident before the first DSMEM store
  const int64_t nclusters = gridDim.x / CS;
  const int64_t cid = blockIdx.x / CS;
  double loss_acc = 0.0;
  int buf = 0;
  for (int64_t row = cid; row < m; row += nclusters) {
    T x[NCH][E];
    const T* xr = X + row * ld;
#pragma unroll
    for (int k = 0; k < NCH; ++k) {
      const int64_t c = c_lo + k * BS + tid;
      const bool in = c < c_lo + SC;
      if (in && c < nfull) {
        fpd::ld_chunk<E * (int)sizeof(T)>(xr + c * E, x[k]);
      } else {
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const int64_t col = c * E + e;
          x[k][e] = (in && col < n) ? xr[col] : T(0);
        }
      }
    }
    const T vr = v ? v[row] : T(1);
    T q;
    if constexpr (YM != 0) {
      T p = T(0);
#pragma unroll
      for (int k = 0; k < NCH; ++k)
#pragma unroll
        for (int e = 0; e < E; ++e) p = fma(x[k][e], ly[k][e], p);
      p = fpd::vector_allreduce<32>(p);
      if (lane == 0) red[warp] = p;
      __syncthreads();
      if (tid < CS) {  // thread t stores this CTA's partial into slot[buf][rank] of CTA t
        T s = T(0);
#pragma unroll
        for (int i = 0; i < NW; ++i) s += red[i];
        T* remote = cluster.map_shared_rank(&slot[buf][rank], tid);
        *remote = s;
      }
      // release our DSMEM stores / acquire everyone's: one cluster barrier per row
      asm volatile("barrier.cluster.arrive.release.aligned;\n" ::: "memory");
      asm volatile("barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
      p = T(0);
#pragma unroll
      for (int i = 0; i < CS; ++i) p += slot[buf][i];  // rank order: identical in every CTA
      buf ^= 1;
      if constexpr (YM == 2) q = fpd::row_epilogue<T>(p, vr, true, row, rank == 0 && tid == 0, a.epi, loss_acc);
      else q = p * vr;
    } else {
      q = vr;
    }
#pragma unroll
    for (int k = 0; k < NCH; ++k)
#pragma unroll
      for (int e = 0; e < E; ++e) lw[k][e] = fma(x[k][e], q, lw[k][e]);
  }
  if constexpr (YM == 2) fpd::flush_loss(a.epi, loss_acc);
  cluster.sync();  // no CTA exits while a peer may still store into its slots

  // this CTA's slice of the partial w -> fp64 accumulator; last CTA of the grid finalises
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t c = c_lo + k * BS + tid;
      const int64_t col = c * E + e;
      if (c < c_lo + SC && col < n) atomicAdd(a.acc + col, (double)lw[k][e]);
    }
  __threadfence();
  __syncthreads();
  __shared__ int s_last;
  if (tid == 0) s_last = (atomicAdd(a.counter, 1ull) == (unsigned long long)gridDim.x - 1ull);
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  const T* z = (const T*)a.z;
  T* w = (T*)a.w;
  for (int64_t j = tid; j < n; j += BS) {
    double s = __ldcg(a.acc + j);
    a.acc[j] = 0.0;
    double r = a.alpha * s;
    if (a.add_beta_z && a.beta != 0.0) r += a.beta * (double)z[j];
    if (a.accumulate) r += (double)w[j];
    w[j] = (T)r;
  }
  if (tid == 0) *a.counter = 0ull;
}

}  // namespace fp
