// dense_cluster.cuh -- wide-row dense kernel on a thread-block CLUSTER (included by
// dense_kernels.cuh).
//
// The paper gives up on fusion when a dense row no longer fits the registers of one vector
// (n > ~6K on Kepler: "launch two separate cuBLAS Level 2 kernels").  On sm_100a a
// cluster of CS CTAs (CS <= 8, portable) shares distributed shared memory, so the vector of
// Table 3 can span CS SMs: VS = CS * BS threads per row, each CTA owning a contiguous column
// slice of y and of the partial w in registers and streaming its slice of the row once.  Per
// row, every CTA reduces its slice's dot (warp shuffles + smem) and writes the partial into a
// slot of EVERY CTA of the cluster with st.async, which credits the bytes to that CTA's
// mbarrier for the slot; once all CS partials landed each CTA sums them in rank order -- all
// CTAs see the same p[r], scale by v[r] and scatter their slice from the same registers.  No
// barrier.cluster (its release half is a MEMBAR.ALL.GPU per row).  Slots are 4-deep: a CTA
// sends row j only after receiving row j-1, by which time every peer has finished row j-2.
// Limit: CS * BS * TL elements per row (TL <= 64 fp32 / 32 fp64): 128K fp32 / 64K fp64 at CS=8.
#pragma once
#include <cooperative_groups.h>

namespace fp {

// 128-byte thread slices are meant to run two CTAs per SM (one's exchange overlaps the other's
// loads): cap them at 128 registers.
template <typename T, int NCH, int E, int CS, int YM, int BS>
__global__ void __launch_bounds__(BS, (NCH * E * sizeof(T) <= 128) ? 2 : 1) k_dense_cluster(const DenseKArgs a) {
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

  constexpr int NSLOT = 4;
  __shared__ T red[NW];
  __shared__ T slot[NSLOT][CS];  // partial dots of the cluster's CTAs, by row % 4
  __shared__ uint64_t xbar[NSLOT];

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
  if (tid == 0) {
    for (int b = 0; b < NSLOT; ++b) fpd::mbar_init(&xbar[b], 1);
    fpd::fence_mbar_init();
    if constexpr (YM != 0)
      for (int b = 0; b < NSLOT; ++b) fpd::mbar_arrive_expect_tx(&xbar[b], CS * (unsigned)sizeof(T));
  }
  cluster.sync();  // all CTAs resident, exchange barriers armed, before the first st.async
  unsigned r_slot = 0, r_bar = 0;
  if (warp == 0 && lane < CS) {
    r_slot = fpd::mapa_u32(fpd::smem_u32(&slot[0][rank]), (unsigned)lane);
    r_bar = fpd::mapa_u32(fpd::smem_u32(&xbar[0]), (unsigned)lane);
  }
  const int64_t nclusters = gridDim.x / CS;
  const int64_t cid = blockIdx.x / CS;
  double loss_acc = 0.0;
  int64_t it = 0;
  for (int64_t row = cid; row < m; row += nclusters, ++it) {
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
      const int sl = (int)(it & (NSLOT - 1));
      if (warp == 0) {  // this CTA's partial -> slot[row % 4][rank] of every CTA (st.async)
        T s = T(0);
#pragma unroll
        for (int i = 0; i < NW; ++i) s += red[i];
        if (lane < CS) fpd::st_async(r_slot + sl * CS * (unsigned)sizeof(T), s, r_bar + sl * (unsigned)sizeof(uint64_t));
        if (lane == 0) {  // every partial of this row landed (cluster-scope acquire), re-arm
          fpd::mbar_wait_cluster(&xbar[sl], (unsigned)((it / NSLOT) & 1));
          fpd::mbar_arrive_expect_tx(&xbar[sl], CS * (unsigned)sizeof(T));
        }
      }
      __syncthreads();  // publishes the slots; red[] is free again
      p = T(0);
#pragma unroll
      for (int i = 0; i < CS; ++i) p += slot[sl][i];  // rank order: identical in every CTA
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

namespace fp {

// Same cluster-wide vector, fed by bulk asynchronous copies (cp.async.bulk global->shared,
// completion on mbarriers; SASS UBLKCP) so that HBM keeps streaming while the CTA waits for
// the row's exchange:
//  * each CTA's slice of a row (NCH*BS*E elements, 32 KB at BS=256 x 128 B) lands in a
//    D-deep shared-memory ring (D = dynamic smem / slice, 3 -> two CTAs per SM), one bulk copy
//    per row issued by thread 0, D-1 rows ahead;
//  * a row is moved smem -> registers at once (16-byte LDS) and its buffer is refilled right
//    after the CTA barrier of the dot reduction, so copies of the next rows are in flight
//    during the exchange; the scale-back uses the registers;
//  * the exchange is the register kernel's st.async + per-slot mbarrier protocol.
// Chunk-to-thread map and reduction trees are those of k_dense_cluster: same bits.
template <typename T, int NCH, int E, int CS, int YM, int BS>
__global__ void __launch_bounds__(BS, 2) k_dense_cluster_tma(const DenseKArgs a) {
  namespace cg = cooperative_groups;
  static_assert(E * sizeof(T) >= 16, "bulk copies need 16-byte granules");
  cg::cluster_group cluster = cg::this_cluster();
  constexpr int NW = BS / 32;
  constexpr int NSLOT = 4;
  constexpr int CAP = NCH * BS * E;  // slice capacity (elements)
  const T* __restrict__ X = (const T*)a.X;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int rank = (int)cluster.block_rank();
  const int64_t m = a.m, n = a.n, ld = a.ld;
  const int64_t nchunks = (n + E - 1) / E;
  const int64_t SC = (nchunks + CS - 1) / CS;
  const int64_t c_lo = rank * SC;
  const int64_t e_lo = c_lo * E;
  const int64_t e_hi = (c_lo + SC) * E < n ? (c_lo + SC) * E : n;
  const int64_t slice = e_hi > e_lo ? e_hi - e_lo : 0;
  const unsigned bulk_bytes = (unsigned)((slice * (int64_t)sizeof(T)) & ~(int64_t)15);
  const int bulk_el = (int)(bulk_bytes / sizeof(T));
  unsigned dyn;
  asm("mov.u32 %0, %%dynamic_smem_size;" : "=r"(dyn));
  const int D = (int)(dyn / (unsigned)(CAP * sizeof(T)));  // ring depth (host guarantees 2..8)

  extern __shared__ __align__(128) unsigned char smem_raw[];
  T* xbuf = reinterpret_cast<T*>(smem_raw);  // [D][CAP]
  __shared__ uint64_t mbar[8];               // ring: bulk copy landed
  __shared__ uint64_t xbar[NSLOT];           // exchange: all CS partials of a row landed
  __shared__ T red[NW];
  __shared__ T slot[NSLOT][CS];

  // row-invariant: bit k of `fast` = chunk k lies wholly inside the bulk copy (16-byte LDS);
  // other chunks: per-element global loads of the sub-16-byte tail, or zeros past the slice
  unsigned fast = 0u;
  T ly[NCH][E], lw[NCH][E];
#pragma unroll
  for (int k = 0; k < NCH; ++k) {
    const int64_t c = c_lo + k * BS + tid;
    if (c < c_lo + SC && (k * BS + tid) * E + E <= bulk_el) fast |= 1u << k;
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t col = c * E + e;
      ly[k][e] = (YM != 0 && c < c_lo + SC && col < n) ? y[col] : T(0);
      lw[k][e] = T(0);
    }
  }
  if (tid == 0) {
    for (int b = 0; b < D; ++b) fpd::mbar_init(&mbar[b], 1);
    for (int b = 0; b < NSLOT; ++b) fpd::mbar_init(&xbar[b], 1);
    fpd::fence_mbar_init();
    if constexpr (YM != 0)
      for (int b = 0; b < NSLOT; ++b) fpd::mbar_arrive_expect_tx(&xbar[b], CS * (unsigned)sizeof(T));
  }
  cluster.sync();  // barriers initialised and armed in every CTA before the first st.async
  unsigned r_slot = 0, r_bar = 0;
  if (warp == 0 && lane < CS) {
    r_slot = fpd::mapa_u32(fpd::smem_u32(&slot[0][rank]), (unsigned)lane);
    r_bar = fpd::mapa_u32(fpd::smem_u32(&xbar[0]), (unsigned)lane);
  }
  const int64_t nclusters = gridDim.x / CS;
  const int64_t cid = blockIdx.x / CS;
  const int64_t cnt = cid < m ? (m - 1 - cid) / nclusters + 1 : 0;  // rows of this cluster
  auto issue = [&](int64_t i, int b) {  // thread 0: row i of this cluster -> ring buffer b
    if (bulk_bytes == 0 || i >= cnt) return;
    fpd::mbar_arrive_expect_tx(&mbar[b], bulk_bytes);
    fpd::bulk_g2s(xbuf + b * CAP, X + (cid + i * nclusters) * ld + e_lo, bulk_bytes, &mbar[b]);
  };
  if (tid == 0)
    for (int i = 0; i < D; ++i) issue(i, i);
  unsigned phase = 0u;  // bit b: parity of the next completion of mbar[b]
  double loss_acc = 0.0;
  int b = 0;
  for (int64_t i = 0; i < cnt; ++i) {
    const int64_t row = cid + i * nclusters;
    if (bulk_bytes) {
      fpd::mbar_wait(&mbar[b], (phase >> b) & 1u);
      phase ^= 1u << b;
    }
    T x[NCH][E];
#pragma unroll
    for (int k = 0; k < NCH; ++k) {
      if (fast >> k & 1u) {
        using V = typename fpd::Vec16<T>::type;
        constexpr int PER = 16 / (int)sizeof(T);
        const V* xs = reinterpret_cast<const V*>(xbuf + b * CAP + (k * BS + tid) * E);
#pragma unroll
        for (int h = 0; h < E / PER; ++h) fpd::Vec16<T>::unpack(xs[h], x[k] + h * PER);
      } else {
        const int64_t c = c_lo + k * BS + tid;
        const T* xr = X + row * ld;
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const int64_t col = c * E + e;
          x[k][e] = (c < c_lo + SC && col < n) ? xr[col] : T(0);
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
      __syncthreads();  // row's partials in red[]; every thread holds its chunks: buffer b free
      const int sl = (int)(i & (NSLOT - 1));
      if (warp == 0) {
        if (lane == 0) {
          fpd::fence_proxy_async_smem();
          issue(i + D, b);
        }
        T s = T(0);
#pragma unroll
        for (int w = 0; w < NW; ++w) s += red[w];
        if (lane < CS) fpd::st_async(r_slot + sl * CS * (unsigned)sizeof(T), s, r_bar + sl * (unsigned)sizeof(uint64_t));
        if (lane == 0) {  // all CS partials landed (cluster-scope acquire); re-arm for row i + 4
          fpd::mbar_wait_cluster(&xbar[sl], (unsigned)((i / NSLOT) & 1));
          fpd::mbar_arrive_expect_tx(&xbar[sl], CS * (unsigned)sizeof(T));
        }
      }
      __syncthreads();  // publishes the slots; red[] free again
      p = T(0);
#pragma unroll
      for (int r = 0; r < CS; ++r) p += slot[sl][r];  // rank order: identical in every CTA
      if constexpr (YM == 2) q = fpd::row_epilogue<T>(p, vr, true, row, rank == 0 && tid == 0, a.epi, loss_acc);
      else q = p * vr;
    } else {
      __syncthreads();  // every thread holds its chunks: buffer b free
      if (tid == 0) {
        fpd::fence_proxy_async_smem();
        issue(i + D, b);
      }
      q = vr;
    }
#pragma unroll
    for (int k = 0; k < NCH; ++k)
#pragma unroll
      for (int e = 0; e < E; ++e) lw[k][e] = fma(x[k][e], q, lw[k][e]);
    b = b + 1 == D ? 0 : b + 1;
  }
  if constexpr (YM == 2) fpd::flush_loss(a.epi, loss_acc);
  cluster.sync();  // no CTA exits while a peer may still st.async into it

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
