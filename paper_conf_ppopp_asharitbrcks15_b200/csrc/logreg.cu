// logreg.cu -- L2-regularised logistic regression by trust-region Newton (TRON), the
// algorithm the paper cites for LogReg (reference [24] Lin, Weng & Keerthi 2008);
// reading R20 of DESIGN.md.  Objective (labels y_i in {-1,+1}):
//
//   f(w) = 1/2 w.w + C sum_i log(1 + exp(-y_i x_i.w))
//   g(w) = w + X^T (C (sigma(y.*Xw) - 1) .* y)            <- ONE fused pass, logistic epilogue,
//                                                            also writes D and the loss
//   H(w) s = s + X^T (D .* (X s)),  D_i = C sigma_i (1 - sigma_i)   <- ONE fused pass, Eq. (1)
//
// Table 1 lists LogReg under X^T y (gradient), X^T(v (.) X y) and + beta z (Hessian-
// vector product): both become single launches of the fused kernel here.  The trust-region
// logic (step acceptance eta0, radius update eta1/eta2/sigma1..3, CG-Steihaug inner solver with
// tolerance 0.1 ||g||) follows [24]; vectors stay on the device, the handful of scalars per
// inner iteration are read back to drive the branches.
#include <math.h>
#include <string.h>

#include <vector>

#include "kernels.cuh"

namespace fp {
fp_status run_dense(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
fp_status run_csr(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
}  // namespace fp

extern "C" fp_status fp_allreduce(fp_comm* comm, void* buf, int64_t n, fp_dtype dtype, fp_stream stream);
extern "C" int fp_comm_rank(const fp_comm* comm);

namespace {

constexpr int kT = 1024;

template <typename T>
__global__ void __launch_bounds__(kT) k_dot2(int64_t n, const T* a, const T* b, const T* c, const T* d, double* out) {
  // out[0] = a.b, out[1] = c.d (c may be NULL): deterministic single-CTA reduction
  __shared__ double red[2][32];
  double s0 = 0.0, s1 = 0.0;
  for (int64_t j = threadIdx.x; j < n; j += kT) {
    s0 += (double)a[j] * (double)b[j];
    if (c) s1 += (double)c[j] * (double)d[j];
  }
  for (int off = 16; off > 0; off >>= 1) {
    s0 += __shfl_xor_sync(0xffffffffu, s0, off);
    s1 += __shfl_xor_sync(0xffffffffu, s1, off);
  }
  if ((threadIdx.x & 31) == 0) {
    red[0][threadIdx.x >> 5] = s0;
    red[1][threadIdx.x >> 5] = s1;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double t0 = 0.0, t1 = 0.0;
    for (int i = 0; i < kT / 32; ++i) {
      t0 += red[0][i];
      t1 += red[1][i];
    }
    out[0] = t0;
    out[1] = t1;
  }
}

// y = a*x + b*y
template <typename T>
__global__ void k_axpby(int64_t n, double a, const T* x, double b, T* y) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
    y[j] = (T)(a * (double)x[j] + b * (double)y[j]);
}

template <typename T>
struct Tron {
  fp::PatternArgs base;  // matrix part (dense or csr) + dtype
  bool csr;
  const void* labels;
  double C;
  fp_comm* comm;
  cudaStream_t s;
  int64_t n, m;
  double* scal = nullptr;  // device scratch: [0..1] dots, [2] loss
  // vectors are carved from the per-stream library workspace (allocated once and reused; no
  // per-solve cudaMallocAsync / cudaFreeAsync -- see drivers.cu cg_typed)
  char* cursor = nullptr;
  size_t left = 0;
  static size_t bytes_for(int64_t len) { return ((size_t)(len > 0 ? len : 1) * sizeof(T) + 255) / 256 * 256; }

  T* alloc(int64_t len, fp_status* st) {
    const size_t b = bytes_for(len);
    if (b > left) {
      *st = FP_ERR_NOMEM;
      return nullptr;
    }
    T* p = (T*)cursor;
    cursor += b;
    left -= b;
    return p;
  }
  ~Tron() { cudaStreamSynchronize(s); }
  fp_status fused(fp::PatternArgs a) {
    if (comm) a.add_beta_z = fp_comm_rank(comm) == 0;
    fp_status st = csr ? fp::run_csr(a, nullptr, s) : fp::run_dense(a, nullptr, s);
    if (st == FP_OK && comm) st = fp_allreduce(comm, a.w, n, base.dtype, s);
    return st;
  }
  fp_status dot2(const T* a, const T* b, const T* c, const T* d, double* out) {
    k_dot2<T><<<1, kT, 0, s>>>(n, a, b, c, d, scal);
    FP_CUDA(cudaGetLastError());
    FP_CUDA(cudaMemcpyAsync(out, scal, 2 * sizeof(double), cudaMemcpyDeviceToHost, s));
    FP_CUDA(cudaStreamSynchronize(s));
    return FP_OK;
  }
  fp_status axpby(double a, const T* x, double b, T* y) {
    int grid = (int)((n + 255) / 256);
    if (grid > 1184) grid = 1184;
    if (grid < 1) grid = 1;
    k_axpby<T><<<grid, 256, 0, s>>>(n, a, x, b, y);
    FP_CUDA(cudaGetLastError());
    return FP_OK;
  }
  // f, g, D at w: g = w + X^T(C (sigma - 1) y) in one fused pass (logistic epilogue)
  fp_status fun_grad(const T* w, T* g, T* D, double* f) {
    fp::PatternArgs a = base;
    a.y = w; a.v = labels; a.z = w; a.alpha = 1.0; a.beta = 1.0; a.w = g;
    a.epi_kind = 1; a.epi_c = C; a.row_out = D; a.scalar_out = scal + 2;
    fp_status st = fused(a);
    if (st != FP_OK) return st;
    if (comm) {
      st = fp_allreduce(comm, scal + 2, 1, FP_F64, s);
      if (st != FP_OK) return st;
    }
    double loss = 0.0, d2[2];
    FP_CUDA(cudaMemcpyAsync(&loss, scal + 2, sizeof(double), cudaMemcpyDeviceToHost, s));
    st = dot2(w, w, nullptr, nullptr, d2);
    *f = 0.5 * d2[0] + C * loss;
    return st;
  }
  // Hd = d + X^T (D (.) (X d)): Eq. (1) with v = D, beta = 1, z = d
  fp_status hess(const T* D, const T* d, T* Hd) {
    fp::PatternArgs a = base;
    a.y = d; a.v = D; a.z = d; a.alpha = 1.0; a.beta = 1.0; a.w = Hd;
    return fused(a);
  }
};

template <typename T>
fp_status tron_typed(fp::PatternArgs base, bool csr, const void* labels, double C, double eps, int max_iter,
                     int max_cg, void* w_out, int* iters_out, double* f_hist, fp_comm* comm, cudaStream_t s) {
  const double eta0 = 1e-4, eta1 = 0.25, eta2 = 0.75, sigma1 = 0.25, sigma2 = 0.5, sigma3 = 4.0;
  Tron<T> t{base, csr, labels, C, comm, s, base.n, base.m};
  fp_status st = FP_OK;
  {
    const size_t need = 256 + 7 * Tron<T>::bytes_for(base.n) + 2 * Tron<T>::bytes_for(base.m);
    fp::Workspace* ws = fp::workspace(s, 0, need);
    if (!ws) return FP_ERR_NOMEM;
    t.scal = (double*)ws->scratch;
    t.cursor = (char*)ws->scratch + 256;
    t.left = need - 256;
  }
  const int64_t n = base.n, m = base.m;
  T* w = (T*)w_out;
  T *g = t.alloc(n, &st), *sv = t.alloc(n, &st), *r = t.alloc(n, &st), *d = t.alloc(n, &st), *Hd = t.alloc(n, &st);
  T *wn = t.alloc(n, &st), *gn = t.alloc(n, &st), *D = t.alloc(m, &st), *Dn = t.alloc(m, &st);
  if (st != FP_OK) return st;
  FP_CUDA(cudaMemsetAsync(w, 0, (size_t)n * sizeof(T), s));
  double f = 0.0, dd[2];
  if ((st = t.fun_grad(w, g, D, &f)) != FP_OK) return st;
  if ((st = t.dot2(g, g, nullptr, nullptr, dd)) != FP_OK) return st;
  const double gnorm0 = sqrt(dd[0]);
  double gnorm = gnorm0, delta = gnorm0;
  int iter = 1, hist_i = 0;
  if (f_hist) f_hist[hist_i++] = f;
  while (iter <= max_iter && gnorm > eps * gnorm0) {
    // ---- CG-Steihaug on the trust region ||s|| <= delta: s = 0, r = -g, d = r
    FP_CUDA(cudaMemsetAsync(sv, 0, (size_t)n * sizeof(T), s));
    if ((st = t.axpby(-1.0, g, 0.0, r)) != FP_OK) return st;
    if ((st = t.axpby(1.0, r, 0.0, d)) != FP_OK) return st;
    double rTr = gnorm * gnorm;
    const double cgtol = 0.1 * gnorm;
    for (int cg = 0; cg < max_cg && sqrt(rTr) > cgtol; ++cg) {
      if ((st = t.hess(D, d, Hd)) != FP_OK) return st;
      if ((st = t.dot2(d, Hd, nullptr, nullptr, dd)) != FP_OK) return st;
      double alpha = rTr / dd[0];
      if ((st = t.axpby(alpha, d, 1.0, sv)) != FP_OK) return st;
      if ((st = t.dot2(sv, sv, nullptr, nullptr, dd)) != FP_OK) return st;
      if (sqrt(dd[0]) > delta) {  // left the region: back to the boundary along d
        if ((st = t.axpby(-alpha, d, 1.0, sv)) != FP_OK) return st;
        double sd[2], ss[2];
        if ((st = t.dot2(sv, d, sv, sv, sd)) != FP_OK) return st;
        if ((st = t.dot2(d, d, nullptr, nullptr, ss)) != FP_OK) return st;
        const double std_ = sd[0], sts = sd[1], dtd = ss[0], dsq = delta * delta;
        const double rad = sqrt(std_ * std_ + dtd * (dsq - sts));
        alpha = std_ >= 0.0 ? (dsq - sts) / (std_ + rad) : (rad - std_) / dtd;
        if ((st = t.axpby(alpha, d, 1.0, sv)) != FP_OK) return st;
        if ((st = t.axpby(-alpha, Hd, 1.0, r)) != FP_OK) return st;
        break;
      }
      if ((st = t.axpby(-alpha, Hd, 1.0, r)) != FP_OK) return st;
      if ((st = t.dot2(r, r, nullptr, nullptr, dd)) != FP_OK) return st;
      const double beta = dd[0] / rTr;
      rTr = dd[0];
      if ((st = t.axpby(1.0, r, beta, d)) != FP_OK) return st;
    }
    // ---- trial point, actual vs predicted reduction, radius update ([24] Section 2)
    if ((st = t.axpby(1.0, w, 0.0, wn)) != FP_OK) return st;
    if ((st = t.axpby(1.0, sv, 1.0, wn)) != FP_OK) return st;
    double gs_sr[2], sn[2];
    if ((st = t.dot2(g, sv, sv, r, gs_sr)) != FP_OK) return st;
    if ((st = t.dot2(sv, sv, nullptr, nullptr, sn)) != FP_OK) return st;
    const double gs = gs_sr[0], prered = -0.5 * (gs - gs_sr[1]);
    double fnew = 0.0;
    if ((st = t.fun_grad(wn, gn, Dn, &fnew)) != FP_OK) return st;
    const double actred = f - fnew, snorm = sqrt(sn[0]);
    if (iter == 1) delta = fmin(delta, snorm);
    double alpha;
    if (fnew - f - gs <= 0.0) alpha = sigma3;
    else alpha = fmax(sigma1, -0.5 * (gs / (fnew - f - gs)));
    if (actred < eta0 * prered) delta = fmin(fmax(alpha, sigma1) * snorm, sigma2 * delta);
    else if (actred < eta1 * prered) delta = fmax(sigma1 * delta, fmin(alpha * snorm, sigma2 * delta));
    else if (actred < eta2 * prered) delta = fmax(sigma1 * delta, fmin(alpha * snorm, sigma3 * delta));
    else delta = fmax(delta, fmin(alpha * snorm, sigma3 * delta));
    if (actred > eta0 * prered) {  // accept
      ++iter;
      if ((st = t.axpby(1.0, wn, 0.0, w)) != FP_OK) return st;
      std::swap(g, gn);
      std::swap(D, Dn);
      f = fnew;
      if ((st = t.dot2(g, g, nullptr, nullptr, dd)) != FP_OK) return st;
      gnorm = sqrt(dd[0]);
      if (f_hist && hist_i <= max_iter) f_hist[hist_i++] = f;
    }
    if (fabs(actred) <= 0.0 && prered <= 0.0) break;
    if (fabs(actred) <= 1e-12 * fabs(f) && fabs(prered) <= 1e-12 * fabs(f)) break;
  }
  if (iters_out) *iters_out = iter - 1;
  FP_CUDA(cudaStreamSynchronize(s));
  return FP_OK;
}

fp_status tron_entry(fp::PatternArgs base, bool csr, const void* labels, double C, double eps, int max_iter,
                     int max_cg, void* w, int* iters, double* f_hist, fp_comm* comm, cudaStream_t s) {
  FP_REQUIRE(fp::valid_dtype(base.dtype), FP_ERR_INVALID_ARG, "logreg: bad dtype");
  FP_REQUIRE(base.m >= 0 && base.n >= 1 && max_iter >= 0 && max_cg >= 1, FP_ERR_INVALID_ARG, "logreg: bad sizes");
  FP_REQUIRE(w && (base.m == 0 || labels) && C > 0.0, FP_ERR_INVALID_ARG, "logreg: w / labels NULL or C <= 0");
  if (base.dtype == FP_F64) return tron_typed<double>(base, csr, labels, C, eps, max_iter, max_cg, w, iters, f_hist, comm, s);
  return tron_typed<float>(base, csr, labels, C, eps, max_iter, max_cg, w, iters, f_hist, comm, s);
}

}  // namespace

extern "C" {

fp_status fp_logreg_tron_dense(int64_t m, int64_t n, const void* X, int64_t ld, const void* labels, double C,
                               double eps, int max_iter, int max_cg, void* w, int* iters, double* f_hist,
                               fp_dtype dtype, fp_comm* comm, fp_stream stream) {
  fp::PatternArgs a;
  a.m = m; a.n = n; a.X = X; a.ld = ld; a.dtype = dtype;
  FP_REQUIRE(X || m == 0, FP_ERR_INVALID_ARG, "fp_logreg_tron_dense: X is NULL");
  if (!X) a.X = (const void*)(uintptr_t)256;
  return tron_entry(a, false, labels, C, eps, max_iter, max_cg, w, iters, f_hist, comm, (cudaStream_t)stream);
}

fp_status fp_logreg_tron_csr(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                             const void* val, const void* labels, double C, double eps, int max_iter, int max_cg,
                             void* w, int* iters, double* f_hist, fp_dtype dtype, fp_comm* comm, fp_stream stream) {
  fp::PatternArgs a;
  a.m = m; a.n = n; a.nnz = nnz; a.rowptr = rowptr; a.colidx = colidx; a.val = val; a.dtype = dtype;
  return tron_entry(a, true, labels, C, eps, max_iter, max_cg, w, iters, f_hist, comm, (cudaStream_t)stream);
}

}  // extern "C"
