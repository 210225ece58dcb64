// aggregate.cuh -- grid-level aggregation of per-CTA partial w (rows a9-a10 of SURVEY 8).
//
// The paper aggregates per-block partials with one global atomicAdd per element
// (Alg. 1 l.15-16 P:195-196, Alg. 2 l.17-18 P:224-225, Alg. 3 l.26-27 P:286-287) into a w
// that must first hold beta*z -- which needs either grid-stride atomics in every block or
// a second kernel, because CUDA had no inter-block barrier.  On sm_100a we
// instead: (1) every CTA adds its fp64 partial into an fp64 workspace accumulator with
// fire-and-forget REDG.E.ADD.F64 (L2-resident, n*8 bytes), (2) takes a ticket on a
// device counter, and (3) the LAST CTA (ticket == gridDim-1) applies alpha and beta*z once
// and writes w -- one launch, no pre-zeroed w, no race on beta*z, and the workspace is
// re-zeroed for the next call.
#pragma once
#include "common.cuh"

namespace fpd {

template <typename T, typename S>
__device__ __forceinline__ void grid_finalize(const S* __restrict__ sw, int64_t n, double* acc,
                                              unsigned long long* counter, double alpha, double beta,
                                              const T* z, T* w, bool add_beta_z, bool accumulate) {
  for (int64_t j = threadIdx.x; j < n; j += blockDim.x) atomicAdd(acc + j, (double)sw[j]);
  __threadfence();
  __syncthreads();
  __shared__ int s_last;
  if (threadIdx.x == 0) s_last = (atomicAdd(counter, 1ull) == (unsigned long long)gridDim.x - 1ull);
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  for (int64_t j = threadIdx.x; j < n; j += blockDim.x) {
    double s = __ldcg(acc + j);
    acc[j] = 0.0;
    double r = alpha * s;
    if (add_beta_z && beta != 0.0) r += beta * (double)z[j];
    if (accumulate) r += (double)w[j];
    w[j] = (T)r;
  }
  if (threadIdx.x == 0) *counter = 0ull;
}

// Same, for a CTA whose partial covers only columns [off, off + len) of w (column-split
// cluster kernel): the last CTA of the grid still finalises all n columns.
template <typename T, typename S>
__device__ __forceinline__ void grid_finalize_window(const S* __restrict__ sw, int64_t off, int64_t len, int64_t n,
                                                     double* acc, unsigned long long* counter, double alpha,
                                                     double beta, const T* z, T* w, bool add_beta_z,
                                                     bool accumulate) {
  for (int64_t j = threadIdx.x; j < len; j += blockDim.x) atomicAdd(acc + off + j, (double)sw[j]);
  __threadfence();
  __syncthreads();
  __shared__ int s_last_w;
  if (threadIdx.x == 0) s_last_w = (atomicAdd(counter, 1ull) == (unsigned long long)gridDim.x - 1ull);
  __syncthreads();
  if (!s_last_w) return;
  __threadfence();
  for (int64_t j = threadIdx.x; j < n; j += blockDim.x) {
    double s = __ldcg(acc + j);
    acc[j] = 0.0;
    double r = alpha * s;
    if (add_beta_z && beta != 0.0) r += beta * (double)z[j];
    if (accumulate) r += (double)w[j];
    w[j] = (T)r;
  }
  if (threadIdx.x == 0) *counter = 0ull;
}

}  // namespace fpd

namespace fpd {

// Row epilogue: what the fused kernels do with a row's dot p = X[r,:] . y before the scale-
// back (Eq. 2).  kind 0: q = v[r] p (Eq. 1), optionally writing p (X y, the margins)
// to row_out.  kind 1 (logistic-regression gradient, reading R20): v[r] = label in {-1,+1},
// t = v[r] p, sigma = 1/(1+e^-t); q = C (sigma - 1) v[r]; row_out <- C sigma (1 - sigma) (the
// Hessian weights D); loss += log(1 + e^-t).  One pass over X gives gradient, D and loss.
struct RowEpi {
  int kind;
  double c;
  void* row_out;
  double* loss;
};

template <typename T>
__device__ __forceinline__ T row_epilogue(T p, T vr, bool ok, int64_t row, bool writer, const RowEpi& e,
                                          double& loss_acc) {
  if (e.kind == 0) {
    if (writer && ok && e.row_out) ((T*)e.row_out)[row] = p;
    return ok ? p * vr : T(0);
  }
  if (!ok) return T(0);
  const double t = (double)vr * (double)p;
  const double sg = 1.0 / (1.0 + exp(-t));
  if (writer) {
    if (e.row_out) ((T*)e.row_out)[row] = (T)(e.c * sg * (1.0 - sg));
    loss_acc += t > 0.0 ? log1p(exp(-t)) : (-t + log1p(exp(t)));
  }
  return (T)(e.c * (sg - 1.0) * (double)vr);
}

// warp-sum the per-thread loss and add it to the global scalar (fp64 atomic)
__device__ __forceinline__ void flush_loss(const RowEpi& e, double loss_acc) {
  if (e.kind != 1 || !e.loss) return;
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) loss_acc += __shfl_xor_sync(0xffffffffu, loss_acc, off);
  if ((threadIdx.x & 31) == 0 && loss_acc != 0.0) atomicAdd(e.loss, loss_acc);
}

}  // namespace fpd
