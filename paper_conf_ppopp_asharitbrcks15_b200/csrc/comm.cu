// comm.cu -- multi-GPU row sharding: NCCL communicator, one in-place
// allreduce of w per evaluation, nnz-balanced shard bounds, the *_dist entry points.
//
// Eq. (1) is a sum over rows of X[r,:]^T (v[r] X[r,:] y) (Eq. 2/3), so a row
// partition needs exactly one exchange: the n-vector sum of per-rank partials.  beta*z is
// added on rank 0 only (reading R18).  The paper is single-GPU; this layer is new.
#include <nccl.h>
#include <string.h>

#include "kernels.cuh"

struct fp_comm {
  ncclComm_t nccl = nullptr;
  int rank = 0;
  int size = 1;
  int device = 0;
};

namespace fp {
fp_status run_dense(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
fp_status run_csr(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
PatternArgs dense_args(int64_t m, int64_t n, const void* X, int64_t ld, const void* y, const void* v, const void* z,
                       double alpha, double beta, void* w, fp_dtype dtype);
PatternArgs csr_args(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                     const void* val, const void* y, const void* v, const void* z, double alpha, double beta, void* w,
                     fp_dtype dtype);

static fp_status nccl_fail(ncclResult_t r, const char* what) {
  set_error("%s: %s", what, ncclGetErrorString(r));
  return FP_ERR_NCCL;
}
}  // namespace fp

#define FP_NCCL(call)                                      \
  do {                                                     \
    ncclResult_t r_ = (call);                              \
    if (r_ != ncclSuccess) return fp::nccl_fail(r_, #call); \
  } while (0)

extern "C" {

fp_status fp_comm_get_unique_id(unsigned char id[128]) {
  FP_REQUIRE(id, FP_ERR_INVALID_ARG, "fp_comm_get_unique_id: id is NULL");
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  ncclUniqueId u;
  FP_NCCL(ncclGetUniqueId(&u));
  memcpy(id, &u, 128);
  return FP_OK;
}

fp_status fp_comm_init(fp_comm** comm, int nranks, int rank, const unsigned char id[128], int device) {
  FP_REQUIRE(comm && id && nranks >= 1 && rank >= 0 && rank < nranks, FP_ERR_INVALID_ARG,
             "fp_comm_init: bad arguments (nranks=%d rank=%d)", nranks, rank);
  FP_CUDA(cudaSetDevice(device));
  ncclUniqueId u;
  memcpy(&u, id, 128);
  fp_comm* c = new fp_comm();
  c->rank = rank;
  c->size = nranks;
  c->device = device;
  ncclResult_t r = ncclCommInitRank(&c->nccl, nranks, u, rank);
  if (r != ncclSuccess) {
    delete c;
    return fp::nccl_fail(r, "ncclCommInitRank");
  }
  *comm = c;
  return FP_OK;
}

fp_status fp_comm_destroy(fp_comm* comm) {
  if (!comm) return FP_OK;
  ncclResult_t r = comm->nccl ? ncclCommDestroy(comm->nccl) : ncclSuccess;
  delete comm;
  if (r != ncclSuccess) return fp::nccl_fail(r, "ncclCommDestroy");
  return FP_OK;
}

int fp_comm_rank(const fp_comm* comm) { return comm ? comm->rank : -1; }
int fp_comm_size(const fp_comm* comm) { return comm ? comm->size : -1; }

fp_status fp_allreduce(fp_comm* comm, void* buf, int64_t n, fp_dtype dtype, fp_stream stream) {
  FP_REQUIRE(comm && fp::valid_dtype(dtype) && n >= 0 && (n == 0 || buf), FP_ERR_INVALID_ARG,
             "fp_allreduce: bad arguments");
  // no short cut for one rank: the collective runs (a copy in place) so that every *_dist call
  // exercises the same NCCL path at any world size
  if (n == 0) return FP_OK;
  FP_NCCL(ncclAllReduce(buf, buf, (size_t)n, dtype == FP_F64 ? ncclFloat64 : ncclFloat32, ncclSum, comm->nccl,
                        (cudaStream_t)stream));
  return FP_OK;
}

// ----------------------------------------------------------------------- shard bounds (host)
fp_status fp_shard_rows_dense(int64_t m, int nranks, int64_t* bounds) {
  FP_REQUIRE(m >= 0 && nranks >= 1 && bounds, FP_ERR_INVALID_ARG, "fp_shard_rows_dense: bad arguments");
  for (int k = 0; k <= nranks; ++k) bounds[k] = (m * k) / nranks;
  return FP_OK;
}

fp_status fp_shard_rows_csr(int64_t m, const int64_t* rowptr, int nranks, int64_t* bounds) {
  FP_REQUIRE(m >= 0 && nranks >= 1 && bounds && rowptr, FP_ERR_INVALID_ARG, "fp_shard_rows_csr: bad arguments");
  const int64_t base = rowptr[0], nnz = rowptr[m] - rowptr[0];
  FP_REQUIRE(nnz >= 0, FP_ERR_INVALID_CSR, "fp_shard_rows_csr: rowptr[m] < rowptr[0]");
  bounds[0] = 0;
  bounds[nranks] = m;
  for (int k = 1; k < nranks; ++k) {
    // first row r with rowptr[r] - base >= k*nnz/P (binary search; rows are never split)
    const int64_t t = (int64_t)(((long double)nnz * k) / nranks);
    int64_t lo = 0, hi = m;
    while (lo < hi) {
      int64_t mid = lo + (hi - lo) / 2;
      if (rowptr[mid] - base < t) lo = mid + 1;
      else hi = mid;
    }
    bounds[k] = lo < bounds[k - 1] ? bounds[k - 1] : lo;
  }
  return FP_OK;
}

// --------------------------------------------------------------------- distributed pattern
fp_status fp_dense_dist(int64_t m_local, int64_t n, const void* X, int64_t ld, const void* y, const void* v,
                        const void* z, double alpha, double beta, void* w, fp_dtype dtype, fp_comm* comm,
                        fp_stream stream) {
  FP_REQUIRE(comm, FP_ERR_INVALID_ARG, "fp_dense_dist: comm is NULL");
  fp::PatternArgs a = fp::dense_args(m_local, n, X, ld, y, v, z, alpha, beta, w, dtype);
  a.add_beta_z = comm->rank == 0;
  fp_status st = fp::run_dense(a, nullptr, (cudaStream_t)stream);
  if (st != FP_OK) return st;
  return fp_allreduce(comm, w, n, dtype, stream);
}

fp_status fp_csr_dist(int64_t m_local, int64_t n, int64_t nnz_local, const int64_t* rowptr, const int32_t* colidx,
                      const void* val, const void* y, const void* v, const void* z, double alpha, double beta,
                      void* w, fp_dtype dtype, fp_comm* comm, fp_stream stream) {
  FP_REQUIRE(comm, FP_ERR_INVALID_ARG, "fp_csr_dist: comm is NULL");
  fp::PatternArgs a = fp::csr_args(m_local, n, nnz_local, rowptr, colidx, val, y, v, z, alpha, beta, w, dtype);
  a.add_beta_z = comm->rank == 0;
  fp_status st = fp::run_csr(a, nullptr, (cudaStream_t)stream);
  if (st != FP_OK) return st;
  return fp_allreduce(comm, w, n, dtype, stream);
}

}  // extern "C"
