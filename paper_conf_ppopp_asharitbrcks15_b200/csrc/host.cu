// host.cu -- host-buffer entry points: the end-to-end path (P:467 counts the host-to-device
// transfer) built as the streaming design the paper names for X that does not stay resident
// ("adapted to a streaming design for out-of-core computation").
//
// Eq. (1) is a sum over rows, so X is cut into row chunks that are copied host->device into a
// double-buffered staging area on a copy stream while the fused kernel runs on the previous
// chunk on a compute stream; w accumulates across chunks (PatternArgs::accumulate), with
// beta*z folded into the first chunk only.  Pageable host memory is first memcpy'd into
// pinned bounce buffers by the calling thread (overlapped with the device copies); pinned
// memory is copied directly.
#include <string.h>

#include <algorithm>
#include <mutex>

#include "kernels.cuh"

namespace fp {
fp_status run_dense(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
fp_status run_csr(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
}  // namespace fp

namespace {

constexpr size_t kChunkBytes = 512ull << 20;  // X bytes per chunk (two chunks in flight)

struct Stager {
  int device = -1;
  cudaStream_t copy = nullptr, comp = nullptr;
  cudaEvent_t copied[2] = {nullptr, nullptr}, consumed[2] = {nullptr, nullptr};
  void* dbuf[2] = {nullptr, nullptr};    // device staging (X / colidx+val / v / rowptr)
  void* hbuf[2] = {nullptr, nullptr};    // pinned bounce buffers (pageable sources)
  size_t cap = 0;
  void* dvec = nullptr;                  // y, z, w on the device
  size_t vcap = 0;
};

std::mutex g_mu;
Stager g_st[16];

fp_status stager_get(int device, size_t chunk_cap, size_t vec_bytes, Stager** out) {
  FP_REQUIRE(device >= 0 && device < 16, FP_ERR_INVALID_ARG, "host path: device %d out of range", device);
  Stager& S = g_st[device];
  FP_CUDA(cudaSetDevice(device));
  if (S.device < 0) {
    FP_CUDA(cudaStreamCreateWithFlags(&S.copy, cudaStreamNonBlocking));
    FP_CUDA(cudaStreamCreateWithFlags(&S.comp, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      FP_CUDA(cudaEventCreateWithFlags(&S.copied[i], cudaEventDisableTiming));
      FP_CUDA(cudaEventCreateWithFlags(&S.consumed[i], cudaEventDisableTiming));
    }
    S.device = device;
  }
  if (chunk_cap > S.cap) {
    cudaDeviceSynchronize();
    for (int i = 0; i < 2; ++i) {
      cudaFree(S.dbuf[i]);
      cudaFreeHost(S.hbuf[i]);
      S.dbuf[i] = S.hbuf[i] = nullptr;
    }
    S.cap = 0;
    for (int i = 0; i < 2; ++i) {
      FP_CUDA(cudaMalloc(&S.dbuf[i], chunk_cap));
      FP_CUDA(cudaMallocHost(&S.hbuf[i], chunk_cap));
    }
    S.cap = chunk_cap;
  }
  if (vec_bytes > S.vcap) {
    cudaDeviceSynchronize();
    cudaFree(S.dvec);
    S.dvec = nullptr;
    S.vcap = 0;
    FP_CUDA(cudaMalloc(&S.dvec, vec_bytes));
    S.vcap = vec_bytes;
  }
  *out = &S;
  return FP_OK;
}

bool is_pinned(const void* p) {
  cudaPointerAttributes at{};
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeHost;
}

// One piece of a chunk: `bytes` from host `src` to device offset `doff` of the staging buffer.
struct Piece {
  const void* src;
  size_t bytes;
  size_t doff;
};

// Copy the pieces of chunk k into staging buffer b (waiting until chunk k-2 released it).
fp_status stage(Stager& S, int b, const Piece* pc, int np, bool pinned) {
  FP_CUDA(cudaStreamWaitEvent(S.copy, S.consumed[b], 0));
  if (!pinned) FP_CUDA(cudaEventSynchronize(S.consumed[b]));  // host reuses hbuf[b]
  for (int i = 0; i < np; ++i) {
    if (pc[i].bytes == 0) continue;
    const void* src = pc[i].src;
    if (!pinned) {
      memcpy((char*)S.hbuf[b] + pc[i].doff, src, pc[i].bytes);
      src = (char*)S.hbuf[b] + pc[i].doff;
    }
    FP_CUDA(cudaMemcpyAsync((char*)S.dbuf[b] + pc[i].doff, src, pc[i].bytes, cudaMemcpyHostToDevice, S.copy));
  }
  FP_CUDA(cudaEventRecord(S.copied[b], S.copy));
  return FP_OK;
}

__global__ void k_rebase(int64_t cnt, int64_t* rp, int64_t base) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < cnt; i += (int64_t)gridDim.x * blockDim.x)
    rp[i] -= base;
}

size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

}  // namespace

extern "C" {

fp_status fp_dense_host(int64_t m, int64_t n, const void* X, int64_t ld, const void* y, const void* v,
                        const void* z, double alpha, double beta, void* w, fp_dtype dtype, int device) {
  FP_REQUIRE(fp::valid_dtype(dtype) && m >= 0 && n >= 0 && ld >= n, FP_ERR_INVALID_ARG, "fp_dense_host: bad arguments");
  FP_REQUIRE(n == 0 || w, FP_ERR_INVALID_ARG, "fp_dense_host: w is NULL");
  FP_REQUIRE(beta == 0.0 || z, FP_ERR_INVALID_ARG, "fp_dense_host: beta != 0 requires z");
  if (n == 0) return FP_OK;
  std::lock_guard<std::mutex> lk(g_mu);
  const size_t s = fp::dtype_size(dtype);
  const size_t row_b = (size_t)ld * s;
  int64_t rows_per_chunk = (int64_t)(kChunkBytes / (row_b + s));
  if (rows_per_chunk < 1) rows_per_chunk = 1;
  if (rows_per_chunk > m) rows_per_chunk = m > 0 ? m : 1;
  const size_t xoff = 0, voff = align256((size_t)rows_per_chunk * row_b);
  const size_t cap = voff + align256((size_t)rows_per_chunk * s);
  Stager* S = nullptr;
  fp_status st = stager_get(device, cap, 3 * align256((size_t)n * s), &S);
  if (st != FP_OK) return st;
  char* dv = (char*)S->dvec;
  void* dy = dv;
  void* dz = dv + align256((size_t)n * s);
  void* dw = dv + 2 * align256((size_t)n * s);
  if (y) FP_CUDA(cudaMemcpyAsync(dy, y, (size_t)n * s, cudaMemcpyHostToDevice, S->comp));
  if (z && beta != 0.0) FP_CUDA(cudaMemcpyAsync(dz, z, (size_t)n * s, cudaMemcpyHostToDevice, S->comp));
  const bool pinned = is_pinned(X) && (!v || is_pinned(v));
  const int64_t nchunks = m > 0 ? (m + rows_per_chunk - 1) / rows_per_chunk : 0;
  for (int b = 0; b < 2; ++b) FP_CUDA(cudaEventRecord(S->consumed[b], S->comp));

  if (nchunks == 0 || alpha == 0.0) {  // w = beta z
    fp::PatternArgs a;
    a.m = 0; a.n = n; a.ld = ld; a.X = (const void*)(uintptr_t)256; a.z = dz; a.alpha = alpha; a.beta = beta;
    a.w = dw; a.dtype = dtype;
    st = fp::run_dense(a, nullptr, S->comp);
  }
  for (int64_t k = 0; st == FP_OK && alpha != 0.0 && k < nchunks; ++k) {
    const int b = (int)(k & 1);
    const int64_t r0 = k * rows_per_chunk, mc = (m - r0) < rows_per_chunk ? (m - r0) : rows_per_chunk;
    // the chunk's last row is copied as n elements, not ld: X may end right after it (its
    // extent is (m-1)*ld + n elements, check_dense), and padded columns are never read (R9)
    Piece pc[2] = {{(const char*)X + (size_t)r0 * row_b, (size_t)(mc - 1) * row_b + (size_t)n * s, xoff},
                   {v ? (const char*)v + (size_t)r0 * s : nullptr, v ? (size_t)mc * s : 0, voff}};
    st = stage(*S, b, pc, 2, pinned);
    if (st != FP_OK) break;
    FP_CUDA(cudaStreamWaitEvent(S->comp, S->copied[b], 0));
    fp::PatternArgs a;
    a.m = mc; a.n = n; a.ld = ld; a.X = (char*)S->dbuf[b] + xoff;
    a.y = y ? dy : nullptr; a.v = v ? (char*)S->dbuf[b] + voff : nullptr; a.z = dz;
    a.alpha = alpha; a.beta = beta; a.w = dw; a.dtype = dtype;
    a.add_beta_z = (k == 0);
    a.accumulate = (k > 0);
    st = fp::run_dense(a, nullptr, S->comp);
    FP_CUDA(cudaEventRecord(S->consumed[b], S->comp));
  }
  if (st == FP_OK) FP_CUDA(cudaMemcpyAsync(w, dw, (size_t)n * s, cudaMemcpyDeviceToHost, S->comp));
  FP_CUDA(cudaStreamSynchronize(S->comp));
  FP_CUDA(cudaStreamSynchronize(S->copy));
  return st;
}

fp_status fp_csr_host(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                      const void* val, const void* y, const void* v, const void* z, double alpha, double beta,
                      void* w, fp_dtype dtype, int device) {
  FP_REQUIRE(fp::valid_dtype(dtype) && m >= 0 && n >= 0 && nnz >= 0, FP_ERR_INVALID_ARG, "fp_csr_host: bad arguments");
  FP_REQUIRE(n == 0 || w, FP_ERR_INVALID_ARG, "fp_csr_host: w is NULL");
  FP_REQUIRE(beta == 0.0 || z, FP_ERR_INVALID_ARG, "fp_csr_host: beta != 0 requires z");
  FP_REQUIRE(m == 0 || rowptr, FP_ERR_INVALID_ARG, "fp_csr_host: rowptr is NULL");
  if (n == 0) return FP_OK;
  std::lock_guard<std::mutex> lk(g_mu);
  const size_t s = fp::dtype_size(dtype);
  // chunks: consecutive rows with <= nnz_cap nonzeros (a longer single row gets its own chunk)
  const int64_t nnz_cap = (int64_t)(kChunkBytes / (s + 4));
  const int64_t row_cap = (int64_t)(kChunkBytes / 64);
  // end of the chunk starting at row r0: the largest r1 in [r0 + 1, min(m, r0 + row_cap)] with
  // rowptr[r1] - rowptr[r0] <= nnz_cap (rowptr is monotone: a binary search, not a row scan --
  // the scan cost ~20 ms of host time per call on C3's 20M rows)
  auto chunk_end = [&](int64_t r0) -> int64_t {
    const int64_t lim = std::min(m, r0 + row_cap);
    const int64_t* p = std::upper_bound(rowptr + r0 + 1, rowptr + lim + 1, rowptr[r0] + nnz_cap);
    const int64_t r1 = (int64_t)(p - rowptr) - 1;
    return r1 > r0 ? r1 : r0 + 1;
  };
  int64_t max_chunk_nnz = 0, max_chunk_rows = 0;
  for (int64_t r0 = 0; r0 < m;) {  // pre-pass for the staging size (host rowptr, cheap)
    const int64_t r1 = chunk_end(r0);
    const int64_t cn = rowptr[r1] - rowptr[r0];
    if (cn > max_chunk_nnz) max_chunk_nnz = cn;
    if (r1 - r0 > max_chunk_rows) max_chunk_rows = r1 - r0;
    r0 = r1;
  }
  const size_t off_rp = 0, off_v = align256((size_t)(max_chunk_rows + 1) * 8);
  const size_t off_c = off_v + align256((size_t)max_chunk_rows * s);
  const size_t off_x = off_c + align256((size_t)max_chunk_nnz * 4);
  const size_t cap = off_x + align256((size_t)max_chunk_nnz * s) + 256;
  Stager* S = nullptr;
  fp_status st = stager_get(device, cap, 3 * align256((size_t)n * s), &S);
  if (st != FP_OK) return st;
  char* dv = (char*)S->dvec;
  void* dy = dv;
  void* dz = dv + align256((size_t)n * s);
  void* dw = dv + 2 * align256((size_t)n * s);
  if (y) FP_CUDA(cudaMemcpyAsync(dy, y, (size_t)n * s, cudaMemcpyHostToDevice, S->comp));
  if (z && beta != 0.0) FP_CUDA(cudaMemcpyAsync(dz, z, (size_t)n * s, cudaMemcpyHostToDevice, S->comp));
  const bool pinned = is_pinned(rowptr) && (nnz == 0 || (is_pinned(colidx) && is_pinned(val))) && (!v || is_pinned(v));
  for (int b = 0; b < 2; ++b) FP_CUDA(cudaEventRecord(S->consumed[b], S->comp));
  bool first = true;
  if (m == 0 || alpha == 0.0) {
    fp::PatternArgs a;
    a.m = 0; a.n = n; a.z = dz; a.alpha = alpha; a.beta = beta; a.w = dw; a.dtype = dtype;
    st = fp::run_csr(a, nullptr, S->comp);
  }
  int64_t k = 0;
  for (int64_t r0 = 0; st == FP_OK && alpha != 0.0 && r0 < m; ++k) {
    const int64_t r1 = chunk_end(r0);
    const int b = (int)(k & 1);
    const int64_t mc = r1 - r0, a0 = rowptr[r0], cn = rowptr[r1] - a0;
    Piece pc[4] = {{rowptr + r0, (size_t)(mc + 1) * 8, off_rp},
                   {v ? (const char*)v + (size_t)r0 * s : nullptr, v ? (size_t)mc * s : 0, off_v},
                   {colidx + a0, (size_t)cn * 4, off_c},
                   {(const char*)val + (size_t)a0 * s, (size_t)cn * s, off_x}};
    st = stage(*S, b, pc, 4, pinned);
    if (st != FP_OK) break;
    FP_CUDA(cudaStreamWaitEvent(S->comp, S->copied[b], 0));
    char* base = (char*)S->dbuf[b];
    k_rebase<<<(int)((mc + 1 + 255) / 256 < 1024 ? (mc + 1 + 255) / 256 : 1024), 256, 0, S->comp>>>(
        mc + 1, (int64_t*)(base + off_rp), a0);
    fp::PatternArgs a;
    a.m = mc; a.n = n; a.nnz = cn; a.rowptr = (const int64_t*)(base + off_rp);
    a.colidx = (const int32_t*)(base + off_c); a.val = base + off_x;
    a.y = y ? dy : nullptr; a.v = v ? base + off_v : nullptr; a.z = dz;
    a.alpha = alpha; a.beta = beta; a.w = dw; a.dtype = dtype;
    a.add_beta_z = first;
    a.accumulate = !first;
    first = false;
    st = fp::run_csr(a, nullptr, S->comp);
    FP_CUDA(cudaEventRecord(S->consumed[b], S->comp));
    r0 = r1;
  }
  if (st == FP_OK) FP_CUDA(cudaMemcpyAsync(w, dw, (size_t)n * s, cudaMemcpyDeviceToHost, S->comp));
  FP_CUDA(cudaStreamSynchronize(S->comp));
  FP_CUDA(cudaStreamSynchronize(S->copy));
  return st;
}

}  // extern "C"
