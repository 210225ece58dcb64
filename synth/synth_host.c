/*
 * synth_host.c -- host (OpenMP) implementation of the counter-based generator in
 * synth_core.h.  Bit-identical to synth_cuda.cu by construction (same integer hash,
 * exact value mappings).  Shared by tests, the oracle side and bench.py input setup;
 * holds none of the method's arithmetic (Eq. 1 of PAPER.md is NOT computed here).
 */
#include "synth_core.h"
#include <math.h>
#include <stddef.h>

#define SYN_F32 0
#define SYN_F64 1

/* Dense row-major matrix: rows [row0, row0+m) of the seeded matrix, n logical columns, row
   stride ld >= n (elements).  Element (r, c) = value(hash(seed, stream, r*n + c)); padding columns c >= n hold NaN
   so that any read of padding by a consumer shows up in its result. */
int synth_dense(int64_t m, int64_t n, int64_t ld, int64_t row0, int dtype, int kind, uint64_t seed,
                uint64_t stream, void* out) {
  if (m < 0 || n < 0 || ld < n) return 1;
#pragma omp parallel for schedule(static)
  for (int64_t r = 0; r < m; ++r) {
    for (int64_t c = 0; c < ld; ++c) {
      if (dtype == SYN_F64) {
        double* o = (double*)out;
        o[r * ld + c] = c < n ? syn_value_f64(syn_hash(seed, stream, (uint64_t)((row0 + r) * n + c)), kind,
                                              syn_colscale_exp(seed, (uint64_t)c))
                              : NAN;
      } else {
        float* o = (float*)out;
        o[r * ld + c] = c < n ? syn_value_f32(syn_hash(seed, stream, (uint64_t)((row0 + r) * n + c)), kind,
                                              syn_colscale_exp(seed, (uint64_t)c))
                              : NAN;
      }
    }
  }
  return 0;
}

/* Dense vector of length len starting at global index i0. */
int synth_vector(int64_t len, int64_t i0, int dtype, int kind, uint64_t seed, uint64_t stream,
                 void* out) {
  if (len < 0) return 1;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < len; ++i) {
    uint64_t h = syn_hash(seed, stream, (uint64_t)(i0 + i));
    if (dtype == SYN_F64) ((double*)out)[i] = syn_value_f64(h, kind, 0);
    else ((float*)out)[i] = syn_value_f32(h, kind, 0);
  }
  return 0;
}

/* Row lengths of rows [row0, row0+m) from an inverse-CDF threshold table. */
int synth_row_lengths(int64_t m, int64_t row0, const uint64_t* thr, int64_t lmax, uint64_t seed,
                      int64_t* len_out) {
  if (m < 0 || lmax < 0) return 1;
#pragma omp parallel for schedule(static)
  for (int64_t r = 0; r < m; ++r)
    len_out[r] = syn_row_length(syn_hash(seed, SYN_S_LEN, (uint64_t)(row0 + r)), thr, lmax);
  return 0;
}

/* Exclusive prefix sum: rowptr[0] = 0, rowptr[r+1] = rowptr[r] + len[r]. */
int synth_rowptr(int64_t m, const int64_t* len, int64_t* rowptr) {
  rowptr[0] = 0;
  for (int64_t r = 0; r < m; ++r) rowptr[r + 1] = rowptr[r] + len[r];
  return 0;
}

/* Fill colidx/val of rows [row0, row0+m) given their (local) rowptr.  The global nnz index
   of local entry k is nnz0 + k, so a row shard is bit-identical to the slice of the full
   matrix when nnz0 = global rowptr[row0]. */
int synth_csr_fill(int64_t m, int64_t n, int64_t row0, int64_t nnz0, const int64_t* rowptr,
                   int dtype, int kind, int col_skew, uint64_t seed, int32_t* colidx, void* val) {
  if (m < 0 || n < 0) return 1;
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t r = 0; r < m; ++r) {
    int64_t a = rowptr[r], L = rowptr[r + 1] - rowptr[r];
    (void)row0;
    for (int64_t k = 0; k < L; ++k) {
      uint64_t g = (uint64_t)(nnz0 + a + k);
      uint64_t hc = syn_hash(seed, SYN_S_COL, g);
      int32_t c = col_skew > 0 ? syn_column_skew(hc, k, L, n, col_skew)
                                 : (col_skew < 0 ? syn_column_iid(hc, n) : syn_column(hc, k, L, n));
      colidx[a + k] = c;
      uint64_t h = syn_hash(seed, SYN_S_VAL, g);
      if (dtype == SYN_F64) ((double*)val)[a + k] = syn_value_f64(h, kind, syn_colscale_exp(seed, (uint64_t)c));
      else ((float*)val)[a + k] = syn_value_f32(h, kind, syn_colscale_exp(seed, (uint64_t)c));
    }
  }
  return 0;
}

/* FNV-1a checksum over a byte range (generator self-check, host vs device). */
uint64_t synth_fnv1a(const void* p, int64_t nbytes) {
  const unsigned char* b = (const unsigned char*)p;
  uint64_t h = 0xcbf29ce484222325ULL;
  for (int64_t i = 0; i < nbytes; ++i) { h ^= b[i]; h *= 0x100000001b3ULL; }
  return h;
}
