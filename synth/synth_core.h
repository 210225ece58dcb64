/*
 * synth_core.h -- counter-based synthetic input generator (the ONE module shared by
 * the oracle side and the CUDA side; it holds none of the method's arithmetic).
 *
 * Every element is a pure function of (seed, stream, global index), so a shard, a
 * host copy and a device copy of the same array are bit-identical by construction.
 * Used by synth_host.c (host, OpenMP) and synth_cuda.cu (device).  Workload recipe:
 * DESIGN.md "Input recipe" (mirrors PAPER.md P:411 synthetic CSR, P:465 HIGGS-like
 * tall-skinny dense, P:427 KDD-like skew).
 */
#ifndef SYNTH_CORE_H
#define SYNTH_CORE_H
#include <stdint.h>

#ifdef __CUDACC__
#define SYNTH_HD __host__ __device__ __forceinline__
#else
#define SYNTH_HD static inline
#endif

/* stream ids: one independent sequence per array role */
enum {
  SYN_S_X = 1, SYN_S_Y = 2, SYN_S_V = 3, SYN_S_Z = 4, SYN_S_LEN = 5, SYN_S_COL = 6,
  SYN_S_VAL = 7, SYN_S_COLSCALE = 8, SYN_S_LABEL = 9, SYN_S_AUX = 10
};

/* value kinds (how a 64-bit hash becomes a number; every mapping is exact) */
enum {
  SYN_K_UNIFORM = 0,   /* U[-1,1): fp64 ((h>>11)*2^-53)*2-1, fp32 ((h>>40)*2^-24)*2-1     */
  SYN_K_POS = 1,       /* U(0,1/4]: fp64 ((h>>11)+1)*2^-55, fp32 ((h>>40)+1)*2^-26        */
  SYN_K_INT_PM12 = 2,  /* {-2,-1,1,2}  (integer twin of X)                                  */
  SYN_K_INT_SMALL = 3, /* {-3..3}      (integer twin of y, z)                               */
  SYN_K_INT_POS = 4,   /* {1,2,3}      (integer twin of v)                                  */
  SYN_K_COLSCALED = 5, /* U[-1,1) * 2^k, k = colscale(col) in {-4..4} (C5 conditioning)      */
  SYN_K_DYADIC = 6     /* k/8, k in {-8..8}: tiny-dyadic inputs for exact-arithmetic pins  */
};

SYNTH_HD uint64_t syn_mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

/* SplitMix64-style counter hash of (seed, stream, index). */
SYNTH_HD uint64_t syn_hash(uint64_t seed, uint64_t stream, uint64_t i) {
  uint64_t key = syn_mix64(seed + stream * 0x9E3779B97F4A7C15ULL);
  return syn_mix64(key + (i + 1) * 0x9E3779B97F4A7C15ULL);
}

SYNTH_HD int syn_colscale_exp(uint64_t seed, uint64_t col) {
  return (int)(syn_hash(seed, SYN_S_COLSCALE, col) % 9ULL) - 4;
}

SYNTH_HD double syn_value_f64(uint64_t h, int kind, int colexp) {
  switch (kind) {
    case SYN_K_UNIFORM: return (double)(h >> 11) * 0x1.0p-53 * 2.0 - 1.0;
    case SYN_K_POS: return (double)((h >> 11) + 1) * 0x1.0p-55;
    case SYN_K_INT_PM12: { double mag = (double)(1 + ((h >> 1) & 1)); return (h & 1) ? -mag : mag; }
    case SYN_K_INT_SMALL: return (double)((int)((h >> 8) % 7ULL) - 3);
    case SYN_K_INT_POS: return (double)(1 + (int)((h >> 8) % 3ULL));
    case SYN_K_COLSCALED: {
      double u = (double)(h >> 11) * 0x1.0p-53 * 2.0 - 1.0;
      double s = 1.0;
      for (int e = colexp; e > 0; --e) s *= 2.0;
      for (int e = colexp; e < 0; ++e) s *= 0.5;
      return u * s;
    }
    case SYN_K_DYADIC: return (double)((int)((h >> 8) % 17ULL) - 8) * 0.125;
    default: return 0.0;
  }
}

SYNTH_HD float syn_value_f32(uint64_t h, int kind, int colexp) {
  switch (kind) {
    case SYN_K_UNIFORM: return (float)(h >> 40) * 0x1.0p-24f * 2.0f - 1.0f;
    case SYN_K_POS: return (float)((h >> 40) + 1) * 0x1.0p-26f;
    case SYN_K_COLSCALED: {
      float u = (float)(h >> 40) * 0x1.0p-24f * 2.0f - 1.0f;
      float s = 1.0f;
      for (int e = colexp; e > 0; --e) s *= 2.0f;
      for (int e = colexp; e < 0; ++e) s *= 0.5f;
      return u * s;
    }
    default: return (float)syn_value_f64(h, kind, colexp); /* integer / dyadic kinds are exact */
  }
}

/* Row length from an inverse-CDF table of uint64 thresholds: smallest L with h < thr[L].
   thr has lmax+1 entries, nondecreasing, thr[lmax] == UINT64_MAX. */
SYNTH_HD int64_t syn_row_length(uint64_t h, const uint64_t* thr, int64_t lmax) {
  int64_t lo = 0, hi = lmax;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (h < thr[mid]) hi = mid; else lo = mid + 1;
  }
  return lo;
}

/* k-th column (0 <= k < L) of a row with L distinct columns drawn from [0, n):
   stratified-uniform -- stratum [floor(k n / L), floor((k+1) n / L)), one uniform
   pick inside.  Sorted and distinct by construction (n >= L). */
SYNTH_HD int32_t syn_column(uint64_t h, int64_t k, int64_t L, int64_t n) {
  int64_t b0 = (k * n) / L, b1 = ((k + 1) * n) / L;
  return (int32_t)(b0 + (int64_t)(h % (uint64_t)(b1 - b0)));
}

/* Skewed ("Zipf-like") variant: popularity decreasing with the column index.  The k-th of L
   columns is k + floor((n - L) * g(u_k)), u_k = (k + frac(h)) / L in 32-bit fixed point and
   g(u) = u^(2^skew_log2) (repeated squaring) -- strictly increasing in k, so sorted and
   distinct; density of column c ~ c^(1/2^skew_log2 - 1).  Integer arithmetic only. */
SYNTH_HD int32_t syn_column_skew(uint64_t h, int64_t k, int64_t L, int64_t n, int skew_log2) {
  uint64_t u = (((uint64_t)k << 32) + (h >> 32)) / (uint64_t)L;  /* in [0, 2^32) */
  for (int i = 0; i < skew_log2; ++i) u = (u * u) >> 32;
  return (int32_t)(k + (int64_t)((((uint64_t)(n - L)) * u) >> 32));
}

/* i.i.d. uniform columns (col_skew < 0): column k of a row is uniform on [0, n) independently
   of the others -- unsorted, repeats possible (summed, reading R7).  The un-stratified
   pattern for measuring the kernels on truly random column positions. */
SYNTH_HD int32_t syn_column_iid(uint64_t h, int64_t n) { return (int32_t)(h % (uint64_t)n); }

#endif
