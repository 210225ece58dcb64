/*
 * synth_cuda.cu -- device implementation of the counter-based generator in synth_core.h.
 * Same functions as synth_host.c (bit-identical outputs); used so that bench.py and the
 * full-size GPU tests can create multi-GB synthetic inputs directly in HBM.  This is
 * input generation only: it computes nothing of Eq. (1) and shares no code with
 * libfusedpat (the product) or the oracle beyond the generator spec itself.
 */
#include "synth_core.h"
#include <cub/device/device_scan.cuh>
#include <cuda_runtime.h>
#include <math.h>

#define SYN_F32 0
#define SYN_F64 1

template <typename T>
__device__ __forceinline__ T syn_value(uint64_t h, int kind, int colexp);
template <>
__device__ __forceinline__ double syn_value<double>(uint64_t h, int kind, int colexp) { return syn_value_f64(h, kind, colexp); }
template <>
__device__ __forceinline__ float syn_value<float>(uint64_t h, int kind, int colexp) { return syn_value_f32(h, kind, colexp); }

template <typename T>
__global__ void k_dense(int64_t m, int64_t n, int64_t ld, int64_t row0, int kind, uint64_t seed, uint64_t stream, T* out) {
  int64_t total = m * ld;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t r = i / ld, c = i - r * ld;
    out[i] = c < n ? syn_value<T>(syn_hash(seed, stream, (uint64_t)((row0 + r) * n + c)), kind, syn_colscale_exp(seed, (uint64_t)c))
                   : (T)NAN;
  }
}

template <typename T>
__global__ void k_vector(int64_t len, int64_t i0, int kind, uint64_t seed, uint64_t stream, T* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < len; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = syn_value<T>(syn_hash(seed, stream, (uint64_t)(i0 + i)), kind, 0);
}

__global__ void k_row_lengths(int64_t m, int64_t row0, const uint64_t* thr, int64_t lmax, uint64_t seed, int64_t* len) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x)
    len[r] = syn_row_length(syn_hash(seed, SYN_S_LEN, (uint64_t)(row0 + r)), thr, lmax);
}

/* one warp per row (heavy power-law rows reach 1e5 entries) */
template <typename T>
__global__ void k_csr_fill(int64_t m, int64_t n, int64_t nnz0, const int64_t* rowptr, int kind, int col_skew,
                           uint64_t seed, int32_t* colidx, T* val) {
  int lane = threadIdx.x & 31;
  int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = warp; r < m; r += nwarps) {
    int64_t a = rowptr[r], L = rowptr[r + 1] - a;
    for (int64_t k = lane; k < L; k += 32) {
      uint64_t g = (uint64_t)(nnz0 + a + k);
      uint64_t hc = syn_hash(seed, SYN_S_COL, g);
      int32_t c = col_skew > 0 ? syn_column_skew(hc, k, L, n, col_skew)
                                 : (col_skew < 0 ? syn_column_iid(hc, n) : syn_column(hc, k, L, n));
      colidx[a + k] = c;
      val[a + k] = syn_value<T>(syn_hash(seed, SYN_S_VAL, g), kind, syn_colscale_exp(seed, (uint64_t)c));
    }
  }
}

static int grid_for(int64_t work) {
  int64_t g = (work + 255) / 256;
  if (g > 148 * 32) g = 148 * 32;
  if (g < 1) g = 1;
  return (int)g;
}

extern "C" {

int synth_dense_cuda(int64_t m, int64_t n, int64_t ld, int64_t row0, int dtype, int kind, uint64_t seed, uint64_t stream, void* out,
                     cudaStream_t s) {
  if (m < 0 || n < 0 || ld < n) return 1;
  if (m == 0 || ld == 0) return 0;
  if (dtype == SYN_F64) k_dense<double><<<grid_for(m * ld), 256, 0, s>>>(m, n, ld, row0, kind, seed, stream, (double*)out);
  else k_dense<float><<<grid_for(m * ld), 256, 0, s>>>(m, n, ld, row0, kind, seed, stream, (float*)out);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

int synth_vector_cuda(int64_t len, int64_t i0, int dtype, int kind, uint64_t seed, uint64_t stream, void* out,
                      cudaStream_t s) {
  if (len < 0) return 1;
  if (len == 0) return 0;
  if (dtype == SYN_F64) k_vector<double><<<grid_for(len), 256, 0, s>>>(len, i0, kind, seed, stream, (double*)out);
  else k_vector<float><<<grid_for(len), 256, 0, s>>>(len, i0, kind, seed, stream, (float*)out);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

int synth_row_lengths_cuda(int64_t m, int64_t row0, const uint64_t* thr_dev, int64_t lmax, uint64_t seed,
                           int64_t* len_out, cudaStream_t s) {
  if (m < 0 || lmax < 0) return 1;
  if (m == 0) return 0;
  k_row_lengths<<<grid_for(m), 256, 0, s>>>(m, row0, thr_dev, lmax, seed, len_out);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

/* rowptr[0] = 0; rowptr[1..m] = inclusive scan of len.  temp: caller-provided scratch of
   *temp_bytes (query with temp == NULL). */
int synth_rowptr_cuda(int64_t m, const int64_t* len, int64_t* rowptr, void* temp, size_t* temp_bytes, cudaStream_t s) {
  if (temp == nullptr) {
    size_t tb = 0;
    cub::DeviceScan::InclusiveSum(nullptr, tb, len, rowptr + 1, (int64_t)m, s);
    *temp_bytes = tb;
    return 0;
  }
  cudaMemsetAsync(rowptr, 0, sizeof(int64_t), s);
  if (m > 0) cub::DeviceScan::InclusiveSum(temp, *temp_bytes, len, rowptr + 1, (int64_t)m, s);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

int synth_csr_fill_cuda(int64_t m, int64_t n, int64_t nnz0, const int64_t* rowptr, int dtype, int kind, int col_skew,
                        uint64_t seed, int32_t* colidx, void* val, cudaStream_t s) {
  if (m < 0 || n < 0) return 1;
  if (m == 0) return 0;
  int g = grid_for(m * 32);
  if (dtype == SYN_F64) k_csr_fill<double><<<g, 256, 0, s>>>(m, n, nnz0, rowptr, kind, col_skew, seed, colidx, (double*)val);
  else k_csr_fill<float><<<g, 256, 0, s>>>(m, n, nnz0, rowptr, kind, col_skew, seed, colidx, (float*)val);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

}  // extern "C"
