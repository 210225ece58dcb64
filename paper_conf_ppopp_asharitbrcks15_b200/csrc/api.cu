// api.cu -- the C ABI entry points of fusedpat.h for the single-GPU pattern: argument checks
// on every call (pointers, sizes, dtype, aliasing -- NOT the CSR structure, which
// fp_csr_validate / fp_csr_plan_create check once per matrix), the alpha == 0 / m == 0 path,
// plan + launch.
#include <string.h>

#include <array>
#include <map>
#include <mutex>

#include "kernels.cuh"

namespace fp {

static fp_status check_vec_alias(const void* w, size_t wb, const void* p, size_t pb, const char* what) {
  FP_REQUIRE(!overlaps(w, wb, p, pb), FP_ERR_ALIAS, "w overlaps %s", what);
  return FP_OK;
}

// Shared validation of the vector / scalar part (R2-R4 of DESIGN.md).
static fp_status check_common(const PatternArgs& a) {
  FP_REQUIRE(valid_dtype(a.dtype), FP_ERR_INVALID_ARG, "dtype must be FP_F32 or FP_F64");
  FP_REQUIRE(a.m >= 0 && a.n >= 0, FP_ERR_INVALID_ARG, "negative size (m=%lld n=%lld)", (long long)a.m,
             (long long)a.n);
  if (a.n == 0) return FP_OK;
  FP_REQUIRE(a.w != nullptr, FP_ERR_INVALID_ARG, "w is NULL");
  FP_REQUIRE(a.beta == 0.0 || a.z != nullptr, FP_ERR_INVALID_ARG, "beta != 0 requires z");
  const size_t s = dtype_size(a.dtype), wb = (size_t)a.n * s;
  if (a.z && a.z != a.w) {
    fp_status st = check_vec_alias(a.w, wb, a.z, wb, "z (only exact aliasing w == z is allowed)");
    if (st != FP_OK) return st;
  }
  if (a.alpha != 0.0 && a.m > 0) {
    fp_status st = check_vec_alias(a.w, wb, a.y, a.y ? wb : 0, "y");
    if (st == FP_OK) st = check_vec_alias(a.w, wb, a.v, a.v ? (size_t)a.m * s : 0, "v");
    if (st != FP_OK) return st;
  }
  return FP_OK;
}

static fp_status check_dense(const PatternArgs& a) {
  fp_status st = check_common(a);
  if (st != FP_OK || a.n == 0) return st;
  FP_REQUIRE(a.ld >= a.n, FP_ERR_INVALID_ARG, "ld (%lld) < n (%lld)", (long long)a.ld, (long long)a.n);
  if (a.alpha != 0.0 && a.m > 0) {
    FP_REQUIRE(a.X != nullptr, FP_ERR_INVALID_ARG, "X is NULL");
    const size_t s = dtype_size(a.dtype);
    st = check_vec_alias(a.w, (size_t)a.n * s, a.X, (size_t)((a.m - 1) * a.ld + a.n) * s, "X");
  }
  return st;
}

static fp_status check_csr(const PatternArgs& a) {
  FP_REQUIRE(a.n <= INT32_MAX, FP_ERR_UNSUPPORTED, "n exceeds int32 column indices");
  fp_status st = check_common(a);
  if (st != FP_OK || a.n == 0) return st;
  FP_REQUIRE(a.nnz >= 0, FP_ERR_INVALID_ARG, "nnz < 0");
  if (a.alpha != 0.0 && a.m > 0) {
    FP_REQUIRE(a.rowptr != nullptr, FP_ERR_INVALID_ARG, "rowptr is NULL");
    FP_REQUIRE(a.nnz == 0 || (a.colidx && a.val), FP_ERR_INVALID_ARG, "colidx/val is NULL");
    const size_t s = dtype_size(a.dtype), wb = (size_t)a.n * s;
    st = check_vec_alias(a.w, wb, a.val, (size_t)a.nnz * s, "val");
    if (st == FP_OK) st = check_vec_alias(a.w, wb, a.colidx, (size_t)a.nnz * 4, "colidx");
    if (st == FP_OK) st = check_vec_alias(a.w, wb, a.rowptr, (size_t)(a.m + 1) * 8, "rowptr");
  }
  return st;
}

// Row-epilogue arguments (fp_*_epi): kind 1 needs y (the margins' weights) and v (labels);
// row_out / scalar_out need alpha != 0 (X must be read).  scalar_out is zeroed here.
static fp_status prepare_epilogue(const PatternArgs& a, cudaStream_t s) {
  FP_REQUIRE(a.epi_kind == 0 || a.epi_kind == 1, FP_ERR_INVALID_ARG, "unknown epilogue %d", a.epi_kind);
  if (a.epi_kind == 1) FP_REQUIRE(a.y && a.v, FP_ERR_INVALID_ARG, "logistic epilogue needs y (w) and v (labels)");
  if (a.epi_kind == 1 || a.row_out)
    FP_REQUIRE(a.alpha != 0.0, FP_ERR_INVALID_ARG, "row epilogue outputs need alpha != 0");
  if (a.scalar_out && !a.accumulate) FP_CUDA(cudaMemsetAsync(a.scalar_out, 0, sizeof(double), s));
  return FP_OK;
}

// Plan cache: the chooser queries the occupancy API and kernel attributes (host calls of a few
// microseconds); repeated calls with the same shape class reuse the plan.  The key holds
// everything a plan depends on (format, device, sizes, dtype, alignment class, y/epilogue
// mode, presence of y for the smem sizing).
namespace {
std::mutex g_plan_mu;
std::map<std::array<int64_t, 10>, fp_launch> g_plans;

std::array<int64_t, 10> plan_key(bool csr, const PatternArgs& a, int dev) {
  const int64_t s = (int64_t)dtype_size(a.dtype);
  const int64_t align = csr ? 0 : (((uintptr_t)a.X % 32 == 0 && (a.ld * s) % 32 == 0) ? 32 :
                                   (((uintptr_t)a.X % 16 == 0 && (a.ld * s) % 16 == 0) ? 16 : s));
  const int64_t ym = !a.y ? 0 : ((a.epi_kind == 0 && !a.row_out) ? 1 : 2);
  return {csr ? 1 : 0, dev, a.m, a.n, csr ? a.nnz : 0, (int64_t)a.dtype, align, ym, a.y ? 1 : 0, 0};
}
}  // namespace

static fp_status cached_plan(bool csr, const PatternArgs& a, fp_launch* L) {
  const int dev = current_device();
  const auto key = plan_key(csr, a, dev);
  {
    std::lock_guard<std::mutex> lk(g_plan_mu);
    auto it = g_plans.find(key);
    if (it != g_plans.end()) {
      *L = it->second;
      return FP_OK;
    }
  }
  fp_status st = csr ? plan_csr(a, dev, L) : plan_dense(a, dev, L);
  if (st != FP_OK) return st;
  std::lock_guard<std::mutex> lk(g_plan_mu);
  if (g_plans.size() > 4096) g_plans.clear();
  g_plans[key] = *L;
  return FP_OK;
}

fp_status run_dense(const PatternArgs& a, const fp_launch* override_, cudaStream_t s) {
  fp_status st = check_dense(a);
  if (st == FP_OK) st = prepare_epilogue(a, s);
  if (st != FP_OK || a.n == 0) return st;
  if (a.alpha == 0.0 || a.m == 0)
    return launch_scale_z(a.n, a.add_beta_z ? a.z : nullptr, a.add_beta_z ? a.beta : 0.0, a.w, a.dtype, s);
  fp_launch L;
  if (override_) {
    L = *override_;
  } else {
    st = cached_plan(false, a, &L);
    if (st != FP_OK) return st;
  }
  return launch_dense(a, L, s);
}

fp_status run_csr(const PatternArgs& a, const fp_launch* override_, cudaStream_t s) {
  fp_status st = check_csr(a);
  if (st == FP_OK) st = prepare_epilogue(a, s);
  if (st != FP_OK || a.n == 0) return st;
  if (a.alpha == 0.0 || a.m == 0)
    return launch_scale_z(a.n, a.add_beta_z ? a.z : nullptr, a.add_beta_z ? a.beta : 0.0, a.w, a.dtype, s);
  fp_launch L;
  if (override_) {
    L = *override_;
  } else {
    st = cached_plan(true, a, &L);
    if (st != FP_OK) return st;
  }
  return launch_csr(a, L, s);
}

PatternArgs dense_args(int64_t m, int64_t n, const void* X, int64_t ld, const void* y, const void* v, const void* z,
                       double alpha, double beta, void* w, fp_dtype dtype) {
  PatternArgs a;
  a.m = m; a.n = n; a.X = X; a.ld = ld; a.y = y; a.v = v; a.z = z;
  a.alpha = alpha; a.beta = beta; a.w = w; a.dtype = dtype;
  return a;
}

PatternArgs csr_args(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                     const void* val, const void* y, const void* v, const void* z, double alpha, double beta, void* w,
                     fp_dtype dtype) {
  PatternArgs a;
  a.m = m; a.n = n; a.nnz = nnz; a.rowptr = rowptr; a.colidx = colidx; a.val = val;
  a.y = y; a.v = v; a.z = z; a.alpha = alpha; a.beta = beta; a.w = w; a.dtype = dtype;
  return a;
}

}  // namespace fp

extern "C" {

const char* fp_status_string(fp_status s) {
  switch (s) {
    case FP_OK: return "FP_OK";
    case FP_ERR_INVALID_ARG: return "FP_ERR_INVALID_ARG";
    case FP_ERR_UNSUPPORTED: return "FP_ERR_UNSUPPORTED";
    case FP_ERR_ALIAS: return "FP_ERR_ALIAS";
    case FP_ERR_INVALID_CSR: return "FP_ERR_INVALID_CSR";
    case FP_ERR_CUDA: return "FP_ERR_CUDA";
    case FP_ERR_NCCL: return "FP_ERR_NCCL";
    case FP_ERR_NOMEM: return "FP_ERR_NOMEM";
  }
  return "FP_ERR_UNKNOWN";
}

#ifdef FP_EXPERIMENTAL_VARIANTS
const char* fp_version(void) { return "0.2.0 sm_100a +experimental"; }
#else
const char* fp_version(void) { return "0.2.0 sm_100a"; }
#endif

fp_status fp_dense(int64_t m, int64_t n, const void* X, int64_t ld, const void* y, const void* v, const void* z,
                   double alpha, double beta, void* w, fp_dtype dtype, fp_stream stream) {
  return fp::run_dense(fp::dense_args(m, n, X, ld, y, v, z, alpha, beta, w, dtype), nullptr, (cudaStream_t)stream);
}

fp_status fp_dense_ex(int64_t m, int64_t n, const void* X, int64_t ld, const void* y, const void* v, const void* z,
                      double alpha, double beta, void* w, fp_dtype dtype, const fp_launch* override_,
                      fp_stream stream) {
  return fp::run_dense(fp::dense_args(m, n, X, ld, y, v, z, alpha, beta, w, dtype), override_,
                       (cudaStream_t)stream);
}

fp_status fp_csr(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx, const void* val,
                 const void* y, const void* v, const void* z, double alpha, double beta, void* w, fp_dtype dtype,
                 fp_stream stream) {
  return fp::run_csr(fp::csr_args(m, n, nnz, rowptr, colidx, val, y, v, z, alpha, beta, w, dtype), nullptr,
                     (cudaStream_t)stream);
}

fp_status fp_csr_ex(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx, const void* val,
                    const void* y, const void* v, const void* z, double alpha, double beta, void* w, fp_dtype dtype,
                    const fp_launch* override_, fp_stream stream) {
  return fp::run_csr(fp::csr_args(m, n, nnz, rowptr, colidx, val, y, v, z, alpha, beta, w, dtype), override_,
                     (cudaStream_t)stream);
}

fp_status fp_dense_epi(int64_t m, int64_t n, const void* X, int64_t ld, const void* y, const void* v, const void* z,
                       double alpha, double beta, void* w, fp_dtype dtype, int epilogue, double c, void* row_out,
                       double* scalar_out, fp_stream stream) {
  fp::PatternArgs a = fp::dense_args(m, n, X, ld, y, v, z, alpha, beta, w, dtype);
  a.epi_kind = epilogue;
  a.epi_c = c;
  a.row_out = row_out;
  a.scalar_out = scalar_out;
  return fp::run_dense(a, nullptr, (cudaStream_t)stream);
}

fp_status fp_csr_epi(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                     const void* val, const void* y, const void* v, const void* z, double alpha, double beta, void* w,
                     fp_dtype dtype, int epilogue, double c, void* row_out, double* scalar_out, fp_stream stream) {
  fp::PatternArgs a = fp::csr_args(m, n, nnz, rowptr, colidx, val, y, v, z, alpha, beta, w, dtype);
  a.epi_kind = epilogue;
  a.epi_c = c;
  a.row_out = row_out;
  a.scalar_out = scalar_out;
  return fp::run_csr(a, nullptr, (cudaStream_t)stream);
}

fp_status fp_release_workspace(void) {
  fp::release_all_workspaces();
  return FP_OK;
}

}  // extern "C"
