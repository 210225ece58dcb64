// dense_kernels.cuh -- fused dense kernels for Eq. (1), re-designing Algorithm 3
// and its generated form, Listing 2, for sm_100a.
//
// What is kept from the paper: a "vector" of VS threads per row, TL elements of the row per
// thread held in registers (l_X), y held in registers (l_y), the row's partial dot
// reduced inside the vector and scaled by v[row] (Alg. 3 l.10-22), the row immediately
// streamed back from the same registers into the thread's register partial of w (l_w,
// l.23-24), coarsening over rows (l.25), and full unrolling of every TL loop, which the
// paper obtains by code generation and we obtain by C++ template instantiation.
// What changed for B200:
//   - rows are fetched with 256-bit LDG.E.256 streaming loads (L1 no-allocate, L2
//     evict-first); RPV rows per vector are loaded before any is reduced, so each lane keeps
//     RPV*32 bytes in flight (memory-level parallelism instead of occupancy alone);
//   - the vector reduction is an xor-shuffle all-reduce, so every lane gets p[r]*v[r]
//     without the warp-synchronous volatile smem broadcast of Listing 2, which
//     is a race on Volta+ independent thread scheduling;
//   - no zero padding of X or y: predicated tails;
//   - aggregation: warp xor-shuffle across vectors -> CTA smem (fixed warp order) ->
//     fp64 grid accumulator + last-CTA finalize (aggregate.cuh) instead of per-thread
//     atomicAdd into a w pre-initialised with beta*z (Alg. 3 l.6-7, l.26-27).
//   - VS > 32 (Alg. 3 l.16-22) is the CTA variant: warp shuffle + smem across warps.
#pragma once
#include "aggregate.cuh"
#include "kernels.cuh"

namespace fp {

struct DenseKArgs {
  int64_t m, n, ld;
  const void* X;
  const void* y;
  const void* v;
  const void* z;
  double alpha, beta;
  void* w;
  double* acc;
  unsigned long long* counter;
  int add_beta_z;
  int accumulate;
  fpd::RowEpi epi;
};

// Warp-granular vector kernel: VS in {1,2,4,8,16,32} lanes per row, NCH chunks of E
// elements per lane (thread load TL = NCH*E), RPV rows per vector per iteration.
#ifndef FP_DENSE_PF
#define FP_DENSE_PF 0
#endif
#ifndef FP_DENSE_MINB
#define FP_DENSE_MINB 1
#endif
#ifndef FP_DENSE_RPV32
#define FP_DENSE_RPV32 4
#endif
template <typename T, int VS, int NCH, int E, int RPV, int YM, int BS>
__global__ void __launch_bounds__(BS, FP_DENSE_MINB) k_dense_vector(const DenseKArgs a) {
  constexpr int VPW = 32 / VS;       // vectors per warp
  constexpr int NW = BS / 32;        // warps per CTA
  constexpr int RPW = VPW * RPV;     // rows per warp iteration
  const T* __restrict__ X = (const T*)a.X;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int lid = lane & (VS - 1), vid = lane / VS;
  const int64_t m = a.m, n = a.n, ld = a.ld;
  const int64_t nfull = n / E;  // chunks lying completely inside the row

  T ly[NCH][E], lw[NCH][E];
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t col = (int64_t)(k * VS + lid) * E + e;
      ly[k][e] = (YM != 0 && col < n) ? y[col] : T(0);
      lw[k][e] = T(0);
    }

  const int64_t nwarps = (int64_t)gridDim.x * NW;
  double loss_acc = 0.0;  // logistic epilogue only
  // rows [base + vid*RPV, +RPV) of this vector: x into registers (first and only HBM touch)
  auto LOAD = [&](int64_t base, T (&x)[RPV][NCH][E], T (&vr)[RPV], bool (&okr)[RPV]) {
#pragma unroll
    for (int i = 0; i < RPV; ++i) {
      const int64_t row = base + vid * RPV + i;
      const bool ok = row < m;
      okr[i] = ok;
      vr[i] = ok ? (v ? v[row] : T(1)) : T(0);
      const T* xr = X + (ok ? row : 0) * ld;
#pragma unroll
      for (int k = 0; k < NCH; ++k) {
        const int64_t c = k * VS + lid;
        if (ok && c < nfull) {
          fpd::ld_chunk<E * (int)sizeof(T)>(xr + c * E, x[i][k]);
        } else {
#pragma unroll
          for (int e = 0; e < E; ++e) {
            const int64_t col = c * E + e;
            x[i][k][e] = (ok && col < n) ? xr[col] : T(0);
          }
        }
      }
    }
  };
  // PF: the next iteration's rows are loaded before this iteration's are reduced (the loads
  // stay in flight through the shuffles).  Build switch for measurement only: on C2 it is
  // slower at every occupancy tried (RPV 2 + PF: 0.726 ms at 3 CTAs/SM, 0.794 ms at 2, 0.96 ms
  // at 4 with spills; RPV 4 + PF: 0.872 ms at 1) than the default (RPV 4, no PF: 0.717 ms).
  // FP_DENSE_MINB / FP_DENSE_RPV32 are the matching occupancy / rows-in-flight switches.
  constexpr bool PF = FP_DENSE_PF != 0;
  T x[RPV][NCH][E], xn[PF ? RPV : 1][NCH][E];
  T vr[RPV], vrn[PF ? RPV : 1];
  bool okr[RPV], okrn[PF ? RPV : 1];
  (void)xn;
  (void)vrn;
  (void)okrn;
  const int64_t base0 = ((int64_t)blockIdx.x * NW + warp) * RPW;
  if constexpr (PF) {
    if (base0 < m) LOAD(base0, x, vr, okr);
  }
  for (int64_t base = base0; base < m; base += nwarps * RPW) {
    if constexpr (PF) {
      if (base + nwarps * RPW < m) LOAD(base + nwarps * RPW, xn, vrn, okrn);
    } else {
      LOAD(base, x, vr, okr);
    }
#pragma unroll
    for (int i = 0; i < RPV; ++i) {
      T q;
      if constexpr (YM != 0) {
        T p = T(0);  // Eq. (2): X[r,:] . y, TL products per lane
#pragma unroll
        for (int k = 0; k < NCH; ++k)
#pragma unroll
          for (int e = 0; e < E; ++e) p = fma(x[i][k][e], ly[k][e], p);
        p = fpd::vector_allreduce<VS>(p);  // intra-vector reduce, every lane gets p[r]
        // q = v[r] p (rows past m contribute nothing, even if y has Inf), or the row epilogue
        if constexpr (YM == 2) q = fpd::row_epilogue<T>(p, vr[i], okr[i], base + vid * RPV + i, lid == 0, a.epi, loss_acc);
        else q = okr[i] ? p * vr[i] : T(0);
      } else {
        q = vr[i];  // Table 1 row 1: alpha X^T v
      }
#pragma unroll
      for (int k = 0; k < NCH; ++k)  // Eq. (3): l_w += X[r,:]^T q, same registers
#pragma unroll
        for (int e = 0; e < E; ++e) lw[k][e] = fma(x[i][k][e], q, lw[k][e]);
    }
    if constexpr (PF) {
#pragma unroll
      for (int i = 0; i < RPV; ++i) {
        vr[i] = vrn[i];
        okr[i] = okrn[i];
#pragma unroll
        for (int k = 0; k < NCH; ++k)
#pragma unroll
          for (int e = 0; e < E; ++e) x[i][k][e] = xn[i][k][e];
      }
    }
  }

  // ---- aggregation: vectors of a warp (xor over the vector-id lane bits) -> CTA -> grid
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e)
#pragma unroll
      for (int off = VS; off < 32; off <<= 1) lw[k][e] += __shfl_xor_sync(0xffffffffu, lw[k][e], off);

  if constexpr (YM == 2) fpd::flush_loss(a.epi, loss_acc);
  extern __shared__ double sw[];  // n doubles
  for (int64_t j = threadIdx.x; j < n; j += BS) sw[j] = 0.0;
  __syncthreads();
  for (int ww = 0; ww < NW; ++ww) {  // fixed warp order: deterministic within the CTA
    if (warp == ww && vid == 0) {
#pragma unroll
      for (int k = 0; k < NCH; ++k)
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const int64_t col = (int64_t)(k * VS + lid) * E + e;
          if (col < n) sw[col] += (double)lw[k][e];
        }
    }
    __syncthreads();
  }
  fpd::grid_finalize<T, double>(sw, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z, a.accumulate);
}

// CTA-wide vector (VS = BS > 32; Alg. 3 l.16-22): all BS threads share one row at a time;
// intra-warp shuffle reduce, then the NW warp sums through double-buffered smem (one
// barrier per row).  Thread t owns chunks t, t+BS, ... (NCH of them).
template <typename T, int NCH, int E, int YM, int BS>
__global__ void __launch_bounds__(BS) k_dense_cta(const DenseKArgs a) {
  constexpr int NW = BS / 32;
  const T* __restrict__ X = (const T*)a.X;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t m = a.m, n = a.n, ld = a.ld;
  const int64_t nfull = n / E;
  __shared__ T red[2][NW];

  T ly[NCH][E], lw[NCH][E];
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t col = (int64_t)(k * BS + tid) * E + e;
      ly[k][e] = (YM != 0 && col < n) ? y[col] : T(0);
      lw[k][e] = T(0);
    }
  int buf = 0;
  double loss_acc = 0.0;
  for (int64_t row = blockIdx.x; row < m; row += gridDim.x) {
    T x[NCH][E];
    const T* xr = X + row * ld;
    const T vr = v ? v[row] : T(1);
#pragma unroll
    for (int k = 0; k < NCH; ++k) {
      const int64_t c = k * BS + tid;
      if (c < nfull) {
        fpd::ld_chunk<E * (int)sizeof(T)>(xr + c * E, x[k]);
      } else {
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const int64_t col = c * E + e;
          x[k][e] = col < n ? xr[col] : T(0);
        }
      }
    }
    T q;
    if constexpr (YM != 0) {
      T p = T(0);
#pragma unroll
      for (int k = 0; k < NCH; ++k)
#pragma unroll
        for (int e = 0; e < E; ++e) p = fma(x[k][e], ly[k][e], p);
      p = fpd::vector_allreduce<32>(p);  // intra-warp (Alg. 3 l.17)
      if (lane == 0) red[buf][warp] = p;
      __syncthreads();                   // l.18-19
      p = T(0);
#pragma unroll
      for (int i = 0; i < NW; ++i) p += red[buf][i];  // inter-warp (l.20), same order everywhere
      buf ^= 1;
      if constexpr (YM == 2) q = fpd::row_epilogue<T>(p, vr, true, row, tid == 0, a.epi, loss_acc);
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
  extern __shared__ double sw[];
  __syncthreads();
  // every column has exactly one owner thread in the CTA: no intra-CTA reduction needed
  for (int64_t j = tid; j < n; j += BS) sw[j] = 0.0;
  __syncthreads();
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t col = (int64_t)(k * BS + tid) * E + e;
      if (col < n) sw[col] = (double)lw[k][e];
    }
  __syncthreads();
  fpd::grid_finalize<T, double>(sw, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z, a.accumulate);
}

// ------------------------------------------------------------------------------ dispatch
// Instantiation sets.  Thread load TL = NCH * E elements is capped at 256 bytes per thread
// (x, y and w partial all live in registers: 3 x 256 B = 192 registers).  E is the elements
// of one load: 32 bytes (LDG.256) when X and ld*sizeof(T) are 32-byte aligned, 16 bytes
// (LDG.128) when 16-byte aligned, else 1 element.
constexpr int kBS = 256;     // vector-kernel block size
constexpr int kBSCta = 256;  // CTA-kernel block size
using DenseKFn = void (*)(const DenseKArgs);

constexpr int rpv_for(int nch, int eb) { return nch * eb <= 32 ? FP_DENSE_RPV32 : (nch * eb <= 64 ? 2 : 1); }

template <typename T, int VS, int NCH, int E, int YM>
DenseKFn vec_k() {
  constexpr int EB = E * (int)sizeof(T);
  if constexpr (NCH * EB <= 256) return k_dense_vector<T, VS, NCH, E, rpv_for(NCH, EB), YM, kBS>;
  else return nullptr;
}

template <typename T, int NCH, int E, int YM>
DenseKFn cta_k() {
  if constexpr (NCH * E * (int)sizeof(T) <= 256) return k_dense_cta<T, NCH, E, YM, kBSCta>;
  else return nullptr;
}

template <typename T, int E, int YM>
DenseKFn pick_vector(int vs, int nch) {
  if (vs < 32 && nch != 1) return nullptr;
  switch (vs) {
    case 1: return vec_k<T, 1, 1, E, YM>();
    case 2: return vec_k<T, 2, 1, E, YM>();
    case 4: return vec_k<T, 4, 1, E, YM>();
    case 8: return vec_k<T, 8, 1, E, YM>();
    case 16: return vec_k<T, 16, 1, E, YM>();
    case 32: break;
    default: return nullptr;
  }
  switch (nch) {
    case 1: return vec_k<T, 32, 1, E, YM>();
    case 2: return vec_k<T, 32, 2, E, YM>();
    case 3: return vec_k<T, 32, 3, E, YM>();
    case 4: return vec_k<T, 32, 4, E, YM>();
    case 6: return vec_k<T, 32, 6, E, YM>();
    case 8: return vec_k<T, 32, 8, E, YM>();
    case 12: return vec_k<T, 32, 12, E, YM>();
    case 16: return vec_k<T, 32, 16, E, YM>();
    case 32: return vec_k<T, 32, 32, E, YM>();
    case 64: return vec_k<T, 32, 64, E, YM>();
    default: return nullptr;
  }
}

template <typename T, int E, int YM>
DenseKFn pick_cta(int nch) {
  switch (nch) {
    case 1: return cta_k<T, 1, E, YM>();
    case 2: return cta_k<T, 2, E, YM>();
    case 4: return cta_k<T, 4, E, YM>();
    case 8: return cta_k<T, 8, E, YM>();
    case 16: return cta_k<T, 16, E, YM>();
    case 32: return cta_k<T, 32, E, YM>();
    case 64: return cta_k<T, 64, E, YM>();
    default: return nullptr;
  }
}

}  // namespace fp
#include "dense_cluster.cuh"
namespace fp {

// cluster kernel: 256-byte thread load (NCH = 256 / (E * sizeof(T))) or 128-byte (NCH / 2,
// fewer registers -> two clusters' CTAs resident per SM, hiding the per-row cluster barrier)

template <typename T, int NCH, int E, int YM>
DenseKFn cluster_reg_k(int cs) {
  switch (cs) {
    case 2: return k_dense_cluster<T, NCH, E, 2, YM, kBSCta>;
    case 4: return k_dense_cluster<T, NCH, E, 4, YM, kBSCta>;
    case 8: return k_dense_cluster<T, NCH, E, 8, YM, kBSCta>;
    default: return nullptr;
  }
}

template <typename T, int NCH, int E, int YM>
DenseKFn cluster_tma_k(int cs) {
  if constexpr (E * sizeof(T) >= 16) {
    switch (cs) {
      case 2: return k_dense_cluster_tma<T, NCH, E, 2, YM, kBSCta>;
      case 4: return k_dense_cluster_tma<T, NCH, E, 4, YM, kBSCta>;
      case 8: return k_dense_cluster_tma<T, NCH, E, 8, YM, kBSCta>;
      default: return nullptr;
    }
  }
  return nullptr;
}

// cluster kernels.  Register kernel (BS = 256): 256- or 128-byte thread slices.  Bulk-copy
// ring kernel (BS = 256, 16/32-byte chunks only): 128- or 64-byte thread slices.
template <typename T, int E, int YM>
DenseKFn pick_cluster(int cs, int nch, int tma) {
  if (tma) {
    constexpr int NF = 128 / (E * (int)sizeof(T)), NHf = 64 / (E * (int)sizeof(T));
    if constexpr (NHf >= 1) {
      if (nch == NF) return cluster_tma_k<T, NF, E, YM>(cs);
      if (nch == NHf) return cluster_tma_k<T, NHf, E, YM>(cs);
    }
    return nullptr;
  }
  constexpr int NCH = 256 / (E * (int)sizeof(T));
  constexpr int NH = NCH / 2 > 0 ? NCH / 2 : 1;
  if (nch == NCH) return cluster_reg_k<T, NCH, E, YM>(cs);
  if (nch == NH) return cluster_reg_k<T, NH, E, YM>(cs);
  return nullptr;
}

template <typename T, int YM>
DenseKFn pick_t(int variant, int chunk_bytes, int vs, int nch, int tma) {
  constexpr int E32 = 32 / (int)sizeof(T), E16 = 16 / (int)sizeof(T);
  if (variant == FP_VAR_DENSE_CLUSTER) {
    const int cs = vs / kBSCta;
    if (chunk_bytes == 32) return pick_cluster<T, E32, YM>(cs, nch, tma);
    if (chunk_bytes == 16) return pick_cluster<T, E16, YM>(cs, nch, tma);
    if (chunk_bytes == (int)sizeof(T)) return pick_cluster<T, 1, YM>(cs, nch, 0);
    return nullptr;
  }
  const bool cta = variant == FP_VAR_DENSE_CTA;
  if (variant != FP_VAR_DENSE_VECTOR && !cta) return nullptr;
  if (chunk_bytes == 32) return cta ? pick_cta<T, E32, YM>(nch) : pick_vector<T, E32, YM>(vs, nch);
  if (chunk_bytes == 16) return cta ? pick_cta<T, E16, YM>(nch) : pick_vector<T, E16, YM>(vs, nch);
  if (chunk_bytes == (int)sizeof(T)) return cta ? pick_cta<T, 1, YM>(nch) : pick_vector<T, 1, YM>(vs, nch);
  return nullptr;
}

// defined in dense_f32.cu / dense_f64.cu (separate translation units: parallel build)
DenseKFn dense_pick_f32(int ym, int variant, int chunk_bytes, int vs, int nch, int tma);
DenseKFn dense_pick_f64(int ym, int variant, int chunk_bytes, int vs, int nch, int tma);

}  // namespace fp
