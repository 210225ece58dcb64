// fixacc.cuh -- exact-integer partial w in shared memory for the CSR scale-back (rows a7/a9 of
// SURVEY 8; the paper's "SD" shared partial of Alg. 1 l.12 / Alg. 2 l.14).
//
// Why: the paper aggregates the per-nonzero products X[r,j] q_r into a shared-memory partial
// with atomicAdd.  On sm_100a a floating-point shared atomic is a CAS loop
// (ATOMS.CAST.SPIN: 1.44 fp64 updates / clk / SM measured, tools/microbench/smem_scatter2.cu);
// the only native shared atomic add is 32-bit integer (ATOMS.ADD: 11.1 / clk / SM).  So each
// term is converted to a 64-bit fixed-point integer and added as two 32-bit limbs (low limb
// with return value for the carry, then high limb): 5.55 updates / clk / SM, 3.9x the CAS.
//
// Representation, per column j (three shared arrays):
//     partial_j = sp[j] + (hi[j] * 2^32 + lo[j]) * 2^(e - kFixBits)
// e is the CTA's cap exponent: terms with |t| < 2^e take the fixed path, rounded to the
// nearest multiple of 2^(e - kFixBits) (|integer| < 2^50); e is set ONCE per CTA, lazily, by
// the first warp that has a nonzero finite term: e = exponent(max |t| of that warp's batch) +
// kFixMargin.  Terms >= 2^e, and non-finite terms (IEEE semantics, DESIGN reading R8), go to
// the fp64 spill partial sp (CAS atomicAdd: rare).  The high limb never overflows: an add
// that leaves |hi| above 2^29 moves 2^28 high units (= 2^(e+10), exact) from hi to sp with a
// 32-bit CAS that applies only while |hi| is still above the limit (value-preserving, bounded).
// Accuracy: the absolute error per term is <= 2^(e - kFixBits - 1) = 2^(e-51), i.e. the
// rounding error of an fp64 sum whose magnitude is ~2^e; the normwise bound of DESIGN R21.
#pragma once
#include <climits>
#include <cstdint>

namespace fpd {

constexpr int kFixUnset = INT_MIN;
constexpr int kFixBits = 50;    // |fixed integer of a term| < 2^50
constexpr int kFixMargin = 6;   // a later term may be 64x the setting batch's max and stay fixed
constexpr int kFixHiLimit = 1 << 29;
constexpr int kFixHiMove = 1 << 28;

struct FixAcc {
  uint32_t* lo;
  int32_t* hi;
  double* sp;
  int* e;  // shared cap exponent (kFixUnset until set)
};

// Per-warp view of the CTA scale (registers).  Warp-uniform.
struct FixScale {
  int e = kFixUnset;
  double scale = 0.0, cap = 0.0, hi_unit = 0.0;
  float scalef = 0.f, capf = 0.f;
  bool fok = false;  // scale representable in fp32 (else fp32 terms convert through fp64)
  __device__ __forceinline__ void set(int ee) {
    e = ee;
    scale = ldexp(1.0, kFixBits - ee);
    cap = ldexp(1.0, ee);
    hi_unit = ldexp(1.0, ee - kFixBits + 32);
    scalef = (float)scale;
    capf = ee >= 128 ? __int_as_float(0x7f800000) : (float)cap;
    fok = kFixBits - ee < 127 && kFixBits - ee > -126;
  }
};

template <int BS>
__device__ __forceinline__ void fix_init(const FixAcc& A, int64_t n) {
  for (int64_t j = threadIdx.x; j < n; j += BS) {
    A.lo[j] = 0u;
    A.hi[j] = 0;
    A.sp[j] = 0.0;
  }
  if (threadIdx.x == 0) *A.e = kFixUnset;
}

// Called by the whole warp before a batch of adds while the scale is still unset: tmax is the
// lane's largest |term| of the batch (finite terms only).  Sets the CTA's e if nobody has.
__device__ __forceinline__ void fix_try_set(const FixAcc& A, FixScale& S, double tmax) {
  if (S.e != kFixUnset) return;
  int cur = __shfl_sync(0xffffffffu, *(volatile int*)A.e, 0);
  if (cur == kFixUnset) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) tmax = fmax(tmax, __shfl_xor_sync(0xffffffffu, tmax, off));
    if (tmax > 0.0) {
      int ee = ilogb(tmax) + 1 + kFixMargin;
      ee = ee < -900 ? -900 : (ee > 1000 ? 1000 : ee);
      if ((threadIdx.x & 31) == 0) atomicCAS(A.e, kFixUnset, ee);
      __syncwarp();
      cur = *(volatile int*)A.e;
    }
  }
  cur = __shfl_sync(0xffffffffu, cur, 0);
  if (cur != kFixUnset) S.set(cur);
}

__device__ __forceinline__ bool fix_finite_abs(double t, double& a) {
  a = fabs(t);
  return a < __longlong_as_double(0x7ff0000000000000ll);
}

// Rare path (|hi| above 2^29): move 2^28 high units into the spill.  Out of line so that the
// hot path keeps its register budget.
static __device__ __noinline__ void fix_move(int32_t* hi, double* sp, int32_t cur, double hi_unit) {
  // a CAS that applies only while |hi| is still above the limit: concurrent movers can never
  // push hi past the opposite limit (a plain subtract by every thread that saw the excess could)
  while (cur > kFixHiLimit || cur < -kFixHiLimit) {
    const int32_t mv = cur > 0 ? kFixHiMove : -kFixHiMove;
    const int32_t prev = atomicCAS(hi, cur, cur - mv);
    if (prev == cur) {
      atomicAdd(sp, (double)mv * hi_unit);
      return;
    }
    cur = prev;
  }
}

__device__ __forceinline__ void fix_limbs(const FixAcc& A, const FixScale& S, int c, long long T) {
  const uint32_t l = (uint32_t)T;
  int32_t h = (int32_t)(T >> 32);
  const uint32_t old = atomicAdd(A.lo + c, l);
  h += (old + l < old) ? 1 : 0;  // carry out of the low limb
  if (h != 0) {
    const int32_t cur = atomicAdd(A.hi + c, h) + h;
    if ((uint32_t)(cur + kFixHiLimit) > (uint32_t)(2 * kFixHiLimit)) fix_move(A.hi + c, A.sp + c, cur, S.hi_unit);
  }
}

// partial_j += t  (fp64 term)
__device__ __forceinline__ void fix_add(const FixAcc& A, const FixScale& S, int c, double t) {
  if (t == 0.0) return;
  if (!(fabs(t) < S.cap)) {  // unset scale, >= cap, NaN or Inf
    atomicAdd(A.sp + c, t);
    return;
  }
  fix_limbs(A, S, c, __double2ll_rn(t * S.scale));
}

// partial_j += t  (fp32 term: the float -> int64 conversion of t * 2^k is exact)
__device__ __forceinline__ void fix_add(const FixAcc& A, const FixScale& S, int c, float t) {
  if (t == 0.f) return;
  if (!(fabsf(t) < S.capf)) {
    atomicAdd(A.sp + c, (double)t);
    return;
  }
  fix_limbs(A, S, c, S.fok ? __float2ll_rn(t * S.scalef) : __double2ll_rn((double)t * S.scale));
}

// After the CTA's last add (caller synchronises): sp[j] += fixed value, in place, so sp is
// the CTA's fp64 partial w for grid_finalize.
template <int BS>
__device__ __forceinline__ void fix_to_double(const FixAcc& A, int64_t n) {
  const int e = *A.e;
  if (e == kFixUnset) return;  // nothing took the fixed path (all terms zero / spilled)
  const double unit = ldexp(1.0, e - kFixBits);
  for (int64_t j = threadIdx.x; j < n; j += BS) {
    const long long I = (long long)(((unsigned long long)(long long)A.hi[j] << 32) | (unsigned long long)A.lo[j]);
    A.sp[j] += (double)I * unit;
  }
}

}  // namespace fpd
