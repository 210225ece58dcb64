// csr_plan.cu -- fp_csr_plan_*: the once-per-matrix analysis of a CSR matrix (row statistics
// -> launch parameters) and, for n too wide for one SM's shared memory, the
// column split of the cluster kernel (csr_colsplit.cuh): CS-1 int32 segment offsets per row.
// The paper amortises its baseline's transpose the same way.
#include <cstdlib>
#include <new>

#include "csr_kernels.cuh"

struct fp_csr_plan {
  int64_t m = 0, n = 0, nnz = 0;
  const int64_t* rowptr = nullptr;
  const int32_t* colidx = nullptr;
  fp_dtype dtype = FP_F32;
  fp_launch L{};
  fp::CsrSplit split;
  int32_t* soff = nullptr;  // device, owned
  int device = 0;
  fp::Packed* packed = nullptr;  // fp_csr_plan_pack: the column-blocked copy (owned)
};

namespace {

// One thread per row: scans the row once, counts entries below each block bound (the segment
// offsets) and checks canonical order (strictly increasing columns; reading R7 allows
// non-canonical rows, which the split cannot serve).
__global__ void k_split_offsets(int64_t m, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ colidx,
                                int cs, fp::CsrSplit sp, int32_t* __restrict__ soff,
                                unsigned long long* __restrict__ bad) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t s = rowptr[r], e = rowptr[r + 1];
    int k = 1;  // next bound to pass
    int prev = -1;
    bool sorted = true;
    for (int64_t i = s; i < e; ++i) {
      const int c = colidx[i];
      sorted &= c > prev;
      prev = c;
      while (k < cs && c >= sp.cb[k]) {
        soff[(int64_t)(k - 1) * m + r] = (int32_t)(i - s);
        ++k;
      }
    }
    for (; k < cs; ++k) soff[(int64_t)(k - 1) * m + r] = (int32_t)(e - s);
    if (!sorted) atomicAdd(bad, 1ull);
  }
}

}  // namespace

namespace fp {
// One evaluation on a plan's matrix: the packed copy when a.val is NULL (fp_csr_plan_pack),
// else the unpacked plan.  a carries the call's vectors and the dist layer's flags (add_beta_z,
// w = a rank's partial buffer).
fp_status plan_run(const fp_csr_plan* p, PatternArgs& a, cudaStream_t s) {
  if (!a.val && p->nnz > 0) {
    FP_REQUIRE(p->packed, FP_ERR_INVALID_ARG, "fp_csr_plan_exec: val is NULL and the plan is not packed");
    FP_REQUIRE(p->n == 0 || a.w, FP_ERR_INVALID_ARG, "fp_csr_plan_exec: w is NULL");
    FP_REQUIRE(a.beta == 0.0 || a.z || !a.add_beta_z, FP_ERR_INVALID_ARG, "fp_csr_plan_exec: beta != 0 needs z");
    FP_REQUIRE(current_device() == p->device, FP_ERR_INVALID_ARG, "fp_csr_plan_exec: plan is on device %d",
               p->device);
    const size_t wb = (size_t)p->n * 4;
    FP_REQUIRE(!overlaps(a.w, wb, a.y, wb) && !overlaps(a.w, wb, a.v, (size_t)p->m * 4), FP_ERR_ALIAS,
               "fp_csr_plan_exec: w overlaps y or v");
    if (p->n == 0) return FP_OK;
    if (a.alpha == 0.0 || p->m == 0)
      return launch_scale_z(p->n, a.add_beta_z ? a.z : nullptr, a.add_beta_z ? a.beta : 0.0, a.w, p->dtype, s);
    return packed_exec(p->packed, a, s);
  }
  a.split = p->soff ? &p->split : nullptr;
  return run_csr(a, &p->L, s);
}
void plan_shape(const fp_csr_plan* p, int64_t* m, int64_t* n, int64_t* nnz, const int64_t** rowptr,
                const int32_t** colidx, fp_dtype* dt) {
  *m = p->m;
  *n = p->n;
  *nnz = p->nnz;
  *rowptr = p->rowptr;
  *colidx = p->colidx;
  *dt = p->dtype;
}
}  // namespace fp

extern "C" {

fp_status fp_csr_plan_create(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                             fp_dtype dtype, const fp_launch* override_, fp_csr_plan** out, fp_stream stream) {
  FP_REQUIRE(out, FP_ERR_INVALID_ARG, "fp_csr_plan_create: out is NULL");
  *out = nullptr;
  FP_REQUIRE(fp::valid_dtype(dtype), FP_ERR_INVALID_ARG, "fp_csr_plan_create: bad dtype");
  FP_REQUIRE(m >= 0 && n >= 0 && nnz >= 0, FP_ERR_INVALID_ARG, "fp_csr_plan_create: negative size");
  FP_REQUIRE(n <= INT32_MAX, FP_ERR_UNSUPPORTED, "fp_csr_plan_create: n exceeds int32 column indices");
  FP_REQUIRE(m == 0 || rowptr, FP_ERR_INVALID_ARG, "fp_csr_plan_create: rowptr is NULL");
  FP_REQUIRE(nnz == 0 || colidx, FP_ERR_INVALID_ARG, "fp_csr_plan_create: colidx is NULL");
  cudaStream_t s = (cudaStream_t)stream;
  // the once-per-matrix structure check (rowptr[0] == 0, monotone, rowptr[m] == nnz, 0 <= col
  // < n): the hot path trusts the plan's matrix, so an invalid one is refused here
  if (m > 0) {
    fp_status vs = fp_csr_validate(m, n, nnz, rowptr, colidx, stream);
    if (vs != FP_OK) return vs;
  }
  fp_csr_plan* p = new (std::nothrow) fp_csr_plan;
  FP_REQUIRE(p, FP_ERR_NOMEM, "fp_csr_plan_create: out of host memory");
  p->m = m;
  p->n = n;
  p->nnz = nnz;
  p->rowptr = rowptr;
  p->colidx = colidx;
  p->dtype = dtype;
  p->device = fp::current_device();
  fp::PatternArgs a;
  a.m = m;
  a.n = n;
  a.nnz = nnz;
  a.rowptr = rowptr;
  a.colidx = colidx;
  a.dtype = dtype;
  a.y = (const void*)(uintptr_t)256;  // plan the full pattern (with y)
  const bool force_split = override_ && override_->variant == FP_VAR_CSR_COLSPLIT;
  fp_status st = FP_OK;
  if (override_ && !force_split) p->L = *override_;
  else st = fp::plan_csr(a, p->device, &p->L);  // also the fallback of a forced split on an empty matrix
  // column split only when forced: measured on B200 it is correct but 2x slower than the flat
  // L2 plan (C4-like 10M x 100K: 7.3 vs 3.6 ms), so the chooser keeps L2
  if (st == FP_OK && m > 0 && nnz > 0 && force_split) {
    fp::CsrSplit sp;
    fp_launch Ls{};
    if (fp::plan_colsplit(a, p->device, force_split ? override_->cluster : 0, &sp, &Ls)) {
      int32_t* soff = nullptr;
      unsigned long long* bad = nullptr;
      cudaError_t e = cudaMalloc((void**)&soff, (size_t)(sp.cs - 1) * (size_t)m * sizeof(int32_t));
      if (e == cudaSuccess) e = cudaMallocAsync((void**)&bad, sizeof(*bad), s);
      if (e != cudaSuccess) {
        cudaGetLastError();
        if (soff) cudaFree(soff);
        delete p;
        fp::set_error("fp_csr_plan_create: cannot allocate the column split (%s)", cudaGetErrorString(e));
        return FP_ERR_NOMEM;
      }
      cudaMemsetAsync(bad, 0, sizeof(*bad), s);
      int grid = (int)std::min<int64_t>((m + 255) / 256, 148 * 16);
      k_split_offsets<<<grid, 256, 0, s>>>(m, rowptr, colidx, sp.cs, sp, soff, bad);
      unsigned long long hbad = 0;
      cudaMemcpyAsync(&hbad, bad, sizeof(hbad), cudaMemcpyDeviceToHost, s);
      cudaFreeAsync(bad, s);
      e = cudaStreamSynchronize(s);
      if (e != cudaSuccess) {
        cudaFree(soff);
        delete p;
        fp::set_error("fp_csr_plan_create: %s", cudaGetErrorString(e));
        return FP_ERR_CUDA;
      }
      if (hbad == 0) {
        sp.soff = soff;
        p->soff = soff;
        p->split = sp;
        p->L = Ls;
      } else {
        cudaFree(soff);
        if (force_split) {
          delete p;
          fp::set_error("fp_csr_plan_create: %llu rows are not canonical (column split needs sorted, unique columns)",
                        hbad);
          return FP_ERR_INVALID_CSR;
        }
      }
    } else if (force_split) {
      delete p;
      fp::set_error("fp_csr_plan_create: no cluster of %d CTAs fits n = %lld", override_->cluster, (long long)n);
      return FP_ERR_UNSUPPORTED;
    }
  }
  if (st != FP_OK) {
    delete p;
    return st;
  }
  *out = p;
  return FP_OK;
}

fp_status fp_csr_plan_exec(const fp_csr_plan* p, const void* val, const void* y, const void* v, const void* z,
                           double alpha, double beta, void* w, fp_stream stream) {
  FP_REQUIRE(p, FP_ERR_INVALID_ARG, "fp_csr_plan_exec: plan is NULL");
  fp::PatternArgs a = fp::csr_args(p->m, p->n, p->nnz, p->rowptr, p->colidx, val, y, v, z, alpha, beta, w, p->dtype);
  return fp::plan_run(p, a, (cudaStream_t)stream);
}

fp_status fp_csr_plan_launch(const fp_csr_plan* p, fp_launch* out) {
  FP_REQUIRE(p && out, FP_ERR_INVALID_ARG, "fp_csr_plan_launch: NULL argument");
  if (p->packed) fp::packed_launch(p->packed, out);
  else *out = p->L;
  return FP_OK;
}

fp_status fp_csr_plan_pack(fp_csr_plan* p, const void* val, fp_stream stream) {
  FP_REQUIRE(p, FP_ERR_INVALID_ARG, "fp_csr_plan_pack: plan is NULL");
  FP_REQUIRE(fp::current_device() == p->device, FP_ERR_INVALID_ARG, "fp_csr_plan_pack: plan is on device %d",
             p->device);
  fp::Packed* q = nullptr;
  const int cs_env = [] {
    const char* e = std::getenv("FP_PK_CS");  // force the column blocks (measurement)
    return e ? std::atoi(e) : 0;
  }();
  fp_status st = fp::packed_build(p->m, p->n, p->nnz, p->rowptr, p->colidx, val, p->dtype, cs_env, &q,
                                  (cudaStream_t)stream);
  if (st != FP_OK) return st;
  fp::packed_free(p->packed);
  p->packed = q;
  return FP_OK;
}

fp_status fp_csr_plan_pack_info(const fp_csr_plan* p, int64_t* ntiles, int64_t* entries, int* blocks, int* groups) {
  FP_REQUIRE(p, FP_ERR_INVALID_ARG, "fp_csr_plan_pack_info: plan is NULL");
  FP_REQUIRE(p->packed, FP_ERR_INVALID_ARG, "fp_csr_plan_pack_info: the plan is not packed");
  if (ntiles) *ntiles = p->packed->ntiles;
  if (entries) *entries = p->packed->entries;
  if (blocks) *blocks = p->packed->cs;
  if (groups) *groups = p->packed->groups;
  return FP_OK;
}

fp_status fp_csr_plan_pack_detail(const fp_csr_plan* p, int64_t out[8]) {
  FP_REQUIRE(p && out, FP_ERR_INVALID_ARG, "fp_csr_plan_pack_detail: NULL argument");
  FP_REQUIRE(p->packed, FP_ERR_INVALID_ARG, "fp_csr_plan_pack_detail: the plan is not packed");
  fp::packed_detail(p->packed, out);
  return FP_OK;
}

fp_status fp_csr_plan_destroy(fp_csr_plan* p) {
  if (!p) return FP_OK;
  if (p->soff) cudaFree(p->soff);
  fp::packed_free(p->packed);
  delete p;
  return FP_OK;
}

}  // extern "C"

// Measurement hook (not part of the ABI, tools/pk_trace.py): the per-warp timing of the last
// packed pass run with FP_PK_TRACE set, 8 uint64 per warp (start, end, tiles, prologue end,
// clocks polling, flagged entries, tiles on the check-free path, clocks in the dots).
extern "C" int fpx_pack_trace(const fp_csr_plan* p, unsigned long long* host, int64_t n) {
  if (!p || !p->packed || !p->packed->trace) return 0;
  const int64_t have = (int64_t)p->packed->groups * p->packed->cs * (p->packed->trace_warps) * 8;
  const int64_t k = n < have ? n : have;
  if (cudaMemcpy(host, p->packed->trace, (size_t)k * 8, cudaMemcpyDeviceToHost) != cudaSuccess) return -1;
  return (int)k;
}
