// csr_kernels.cuh -- fused CSR kernels for Eq. (1), re-designing
// Algorithms 1-2 for sm_100a.
//
// Kept from the paper: CSR-vector ([3]) -- a vector of VS lanes per row, VS from the
// mean row length (Eq. 4); the row's dot with y reduced inside the vector
// (Alg. 2 l.10-12) and multiplied by v[row] by the vector; the same lanes then
// scatter X[r,:]^T q into a partial w (l.13-14) -- the second touch of the row comes from the
// registers that loaded it, not from HBM; partial w in shared memory when n fits
// ("inter-vector aggregation") and in global memory for large n.
// Changed for B200:
//   - each warp owns a contiguous row range balanced by nnz + per-row cost, found with a
//     32-ary warp-cooperative search of rowptr (no coarsening factor C to tune, no tail
//     imbalance on power-law rows; correctness never depends on it);
//   - rowptr is fetched 32 rows at a time with one coalesced load and broadcast by shuffle;
//     RPV row groups are in flight per warp iteration;
//   - y is staged in shared memory when it fits (the paper bound y to texture);
//   - the inter-vector aggregation has three modes:
//       MODE_PRIVATE: one partial w per WARP in shared memory, updated with plain
//         load-add-store (no atomics: float shared atomics are CAS loops on sm_100a); lanes of
//         different vectors that hit the same column in one instruction are serialised with
//         __match_any_sync; the NW warp partials are summed in fixed order at the end;
//       MODE_SHARED: one partial w per CTA, shared-memory atomicAdd (the paper's SD);
//       MODE_L2: fire-and-forget red.global.add into the L2-resident w, alpha folded
//         into q, w pre-written with beta*z by a tiny kernel.
//     Small-n modes finish with the fp64 grid accumulator + last-CTA finalize (aggregate.cuh).
#pragma once
#include "aggregate.cuh"
#include "fixacc.cuh"
#include "kernels.cuh"

namespace fp {

struct CsrKArgs {
  int64_t m, n, nnz;
  const int64_t* rowptr;
  const int32_t* colidx;
  const void* val;
  const void* y;
  const void* v;
  const void* z;
  double alpha, beta;
  void* w;
  double* acc;
  unsigned long long* counter;
  int add_beta_z;
  int accumulate;
  int y_in_smem;  // MODE_L2 only: number of leading y entries staged in shared memory (0: none;
                  // >= n: all -- the only case the CSR-vector kernel accepts)
  fpd::RowEpi epi;
  int phase_iters;  // owner-computes kernel: row-group iterations between queue drains
  // MODE_L2: the CTAs reduce into nrep copies of w (copy 0 = w, copies 1.. = wrep, stride n,
  // all-zero on entry; folded into w by k_fold_replicas) to spread the random reds over more
  // L2 lines / slices
  void* wrep;
  int nrep;
};

// MODE_L2 target of this CTA's reds
template <typename T>
__device__ __forceinline__ T* l2_target(const CsrKArgs& a) {
  if (a.nrep <= 1) return (T*)a.w;
  const int r = (int)(blockIdx.x % (unsigned)a.nrep);
  return r == 0 ? (T*)a.w : (T*)a.wrep + (int64_t)(r - 1) * a.n;
}

enum { MODE_L2 = 0, MODE_SHARED = 1, MODE_PRIVATE = 2, MODE_FIXED = 8 };

// shared-memory layout of the MODE_FIXED partial behind y_s (fixacc.cuh): [sp: n f64][lo: n u32][hi: n u32]
__device__ __forceinline__ fpd::FixAcc fix_layout(unsigned char* base, int64_t n, int* e) {
  fpd::FixAcc A;
  A.sp = reinterpret_cast<double*>(base);
  A.lo = reinterpret_cast<uint32_t*>(A.sp + n);
  A.hi = reinterpret_cast<int32_t*>(A.lo + n);
  A.e = e;
  return A;
}
__host__ __device__ constexpr int64_t fix_y_bytes(int64_t n, int s) { return (n * s + 15) / 16 * 16; }

constexpr int64_t kRowCost = 4;  // a row costs about as much as 4 nonzeros (rowptr, v, reduce)

// First row r in [0, m] with rowptr[r] + kRowCost*r >= t (monotone in r).  Warp-cooperative
// 32-ary search: ~log32(m) dependent loads instead of log2(m).
__device__ __forceinline__ int64_t warp_search_rows(const int64_t* __restrict__ rowptr, int64_t m, int64_t t,
                                                    int lane) {
  int64_t lo = 0, hi = m;  // answer in [lo, hi]
  while (hi - lo > 32) {
    const int64_t span = hi - lo;
    const int64_t p = lo + (span * (lane + 1)) / 33;
    const bool below = __ldg(rowptr + p) + kRowCost * p < t;
    const unsigned bal = __ballot_sync(0xffffffffu, below);
    const int cnt = __popc(bal);
    const int64_t plo = __shfl_sync(0xffffffffu, p, cnt > 0 ? cnt - 1 : 0);
    const int64_t phi = __shfl_sync(0xffffffffu, p, cnt < 32 ? cnt : 31);
    if (cnt > 0) lo = plo + 1;
    if (cnt < 32) hi = phi;
  }
  const int64_t p = lo + lane;
  const bool below = p < hi && (__ldg(rowptr + p) + kRowCost * p < t);
  const unsigned bal = __ballot_sync(0xffffffffu, below);
  return lo + __popc(bal);
}

// Warp-private partial update wp[c] += val (plain load-add-store, no atomics).  Lanes of
// DIFFERENT vectors may hit the same column, so the VPW vectors of the warp update one after
// the other.  Inside a vector the lanes hold one row's entries; their columns are distinct
// when the row is canonical (strictly increasing across lanes -- one shuffle + vote checks
// it); a non-canonical row (duplicates, reading R7) is serialised lane by lane.
template <int VS, typename T>
__device__ __forceinline__ void warp_private_add(T* wp, int c, T val, bool act, int lane) {
  constexpr int VPW = 32 / VS;
  const int lid = lane & (VS - 1), vid = lane / VS;
  bool ok = true;
  if constexpr (VS > 1) {
    const int cn = __shfl_down_sync(0xffffffffu, c, 1);
    const bool nact = __shfl_down_sync(0xffffffffu, (int)act, 1) != 0;
    ok = !(act && nact && lid + 1 < VS && cn <= c);
  }
  if (__all_sync(0xffffffffu, ok)) {
#pragma unroll
    for (int u = 0; u < VPW; ++u) {
      if (act && vid == u) wp[c] += val;
      __syncwarp();
    }
  } else {
    for (int l = 0; l < 32; ++l) {
      if (act && lane == l) wp[c] += val;
      __syncwarp();
    }
  }
}

// VS lanes per row, K nonzeros per lane cached in registers (rows up to VS*K are read from
// HBM exactly once; longer rows re-read their tail from L1/L2 for the scatter, the paper's
// "likely a cache hit"), RPV row groups per warp iteration.
template <typename T, int VS, int K, int RPV, int YM, int MODE, int BS>
__global__ void __launch_bounds__(BS) k_csr_vector(const CsrKArgs a) {
  constexpr int VPW = 32 / VS;
  constexpr int NW = BS / 32;
  constexpr int GROUP = VPW * RPV;  // rows per warp iteration
  static_assert(GROUP <= 32, "rowptr batch holds 32 rows");
  const int64_t* __restrict__ rowptr = a.rowptr;
  const int32_t* __restrict__ colidx = a.colidx;
  const T* __restrict__ val = (const T*)a.val;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int lid = lane & (VS - 1), vid = lane / VS;
  const int64_t m = a.m, n = a.n;

  // shared memory: [y_s: n] [w partials: n (SHARED) or NW*n (PRIVATE)]
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* y_s = reinterpret_cast<T*>(smem_raw);
  constexpr bool HAS_Y = YM != 0;
  const bool ysm = HAS_Y && (MODE != MODE_L2 || a.y_in_smem);
  T* w_s = y_s + (ysm ? n : 0);
  T* w_mine = MODE == MODE_PRIVATE ? w_s + (int64_t)warp * n : w_s;
  __shared__ int fix_e;
  const fpd::FixAcc FA = fix_layout(smem_raw + (ysm ? fix_y_bytes(n, sizeof(T)) : 0), n, &fix_e);
  fpd::FixScale FS;
  {
    const int64_t nw_copies = MODE == MODE_PRIVATE ? NW : (MODE == MODE_SHARED ? 1 : 0);
    for (int64_t j = threadIdx.x; j < nw_copies * n; j += BS) w_s[j] = T(0);
    if constexpr (MODE == MODE_FIXED) fpd::fix_init<BS>(FA, n);
    if (ysm)
      for (int64_t j = threadIdx.x; j < n; j += BS) y_s[j] = y[j];
    if (nw_copies > 0 || ysm || MODE == MODE_FIXED) __syncthreads();
  }
  // alpha: folded into q on the L2 path, applied once by the finaliser on the smem paths
  const T qscale = MODE == MODE_L2 ? (T)a.alpha : T(1);
  auto Y = [&](int c) -> T { return ysm ? y_s[c] : fpd::ld_keep(y + c); };
  T* const wl2 = l2_target<T>(a);
  auto W_ADD = [&](int c, T val_, bool act) {
    if constexpr (MODE == MODE_PRIVATE) {
      warp_private_add<VS>(w_mine, c, val_, act, lane);
    } else if constexpr (MODE == MODE_SHARED) {
      if (act) atomicAdd(w_s + c, val_);
    } else if constexpr (MODE == MODE_FIXED) {
      if (act) fpd::fix_add(FA, FS, c, val_);
    } else {
      if (act) fpd::red_add(wl2 + c, val_);
    }
  };

  // ---- this warp's row range, balanced by nnz + kRowCost*rows
  const int64_t gw = (int64_t)blockIdx.x * NW + warp, tw = (int64_t)gridDim.x * NW;
  const int64_t total = a.nnz + kRowCost * m;
  const int64_t r0 = warp_search_rows(rowptr, m, (total * gw) / tw, lane);
  const int64_t r1 = warp_search_rows(rowptr, m, (total * (gw + 1)) / tw, lane);

  int64_t bstart = r0;  // rows [bstart, bstart+32) have their rowptr in `rp` (lane i: row bstart+i)
  int64_t rp = (bstart + lane <= m) ? __ldg(rowptr + bstart + lane) : 0;
  int64_t rp32 = (bstart + 32 <= m) ? __ldg(rowptr + bstart + 32) : 0;

  double loss_acc = 0.0;  // logistic epilogue only
  for (int64_t rb = r0; rb < r1; rb += GROUP) {
    if (rb + GROUP > bstart + 32) {  // refill the rowptr batch (warp-uniform)
      bstart = rb;
      rp = (bstart + lane <= m) ? __ldg(rowptr + bstart + lane) : 0;
      rp32 = (bstart + 32 <= m) ? __ldg(rowptr + bstart + 32) : 0;
    }
    int64_t start[RPV], len[RPV];
    T vr[RPV];
    bool okr[RPV];
    bool any_long = false;
#pragma unroll
    for (int i = 0; i < RPV; ++i) {
      const int64_t row = rb + i * VPW + vid;
      const int o = (int)(row - bstart);
      const int64_t s0 = __shfl_sync(0xffffffffu, rp, o & 31);
      const int64_t s1n = __shfl_sync(0xffffffffu, rp, (o + 1) & 31);
      const int64_t s1 = (o + 1 == 32) ? rp32 : s1n;
      const bool ok = row < r1;
      okr[i] = ok;
      start[i] = ok ? s0 : 0;
      len[i] = ok ? s1 - s0 : 0;
      vr[i] = ok ? (v ? v[row] : T(1)) : T(0);
      any_long |= len[i] > VS * K;
    }
    any_long = __any_sync(0xffffffffu, any_long);

    // ---- first touch: (col, val) into registers
    int cc[RPV][K];
    T xv[RPV][K];
#pragma unroll
    for (int i = 0; i < RPV; ++i)
#pragma unroll
      for (int k = 0; k < K; ++k) {
        const int64_t idx = lid + k * VS;
        if (idx < len[i]) {
          cc[i][k] = fpd::ld_once(colidx + start[i] + idx);
          xv[i][k] = fpd::ld_once(val + start[i] + idx);
        } else {
          cc[i][k] = 0;
          xv[i][k] = T(0);
        }
      }
    int64_t lmax = 0;
    if (any_long) {
#pragma unroll
      for (int i = 0; i < RPV; ++i) lmax = len[i] > lmax ? len[i] : lmax;
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        const int64_t o = __shfl_xor_sync(0xffffffffu, lmax, off);
        lmax = o > lmax ? o : lmax;
      }
    }

    T q[RPV];
    if constexpr (HAS_Y) {
      T p[RPV];
      T yv[RPV][K];  // every gather issued before the first use (latencies overlap)
      if (ysm) {
#pragma unroll
        for (int i = 0; i < RPV; ++i)
#pragma unroll
          for (int k = 0; k < K; ++k) yv[i][k] = y_s[cc[i][k]];
      } else {
#pragma unroll
        for (int i = 0; i < RPV; ++i)
#pragma unroll
          for (int k = 0; k < K; ++k) yv[i][k] = fpd::ld_keep(y + cc[i][k]);
      }
#pragma unroll
      for (int i = 0; i < RPV; ++i) {  // Eq. (2) / Alg. 2 l.10-11
        p[i] = T(0);
#pragma unroll
        for (int k = 0; k < K; ++k)
          if (lid + k * VS < len[i]) p[i] = fma(xv[i][k], yv[i][k], p[i]);
      }
      if (any_long) {  // tails of rows longer than VS*K (warp-uniform loop)
        for (int64_t seg = VS * K; seg < lmax; seg += VS * K) {
#pragma unroll
          for (int i = 0; i < RPV; ++i)
#pragma unroll
            for (int k = 0; k < K; ++k) {
              const int64_t idx = seg + lid + k * VS;
              if (idx < len[i]) {
                const int c = __ldg(colidx + start[i] + idx);
                p[i] = fma(__ldg(val + start[i] + idx), Y(c), p[i]);
              }
            }
        }
      }
#pragma unroll
      for (int i = 0; i < RPV; ++i)  // l.12: q = v[r] * reduce(p) (or the row epilogue)
        if constexpr (YM == 2)
          q[i] = fpd::row_epilogue<T>(fpd::vector_allreduce<VS>(p[i]), vr[i], okr[i], rb + i * VPW + vid, lid == 0,
                                      a.epi, loss_acc) *
                 qscale;
        else
          q[i] = fpd::vector_allreduce<VS>(p[i]) * vr[i] * qscale;
    } else {
#pragma unroll
      for (int i = 0; i < RPV; ++i) q[i] = vr[i] * qscale;
    }

    // ---- second touch from registers: Eq. (3) / Alg. 2 l.13-14
    if constexpr (MODE == MODE_FIXED) {
      if (FS.e == fpd::kFixUnset) {  // warp-uniform; until the CTA's fixed-point scale is set
        double tmax = 0.0;
#pragma unroll
        for (int i = 0; i < RPV; ++i)
#pragma unroll
          for (int k = 0; k < K; ++k) {
            double at;
            if (lid + k * VS < len[i] && fpd::fix_finite_abs((double)(xv[i][k] * q[i]), at)) tmax = fmax(tmax, at);
          }
        fpd::fix_try_set(FA, FS, tmax);
      }
    }
#pragma unroll
    for (int i = 0; i < RPV; ++i)
#pragma unroll
      for (int k = 0; k < K; ++k) W_ADD(cc[i][k], xv[i][k] * q[i], lid + k * VS < len[i]);
    if (any_long) {
      for (int64_t seg = VS * K; seg < lmax; seg += VS * K) {
#pragma unroll
        for (int i = 0; i < RPV; ++i)
#pragma unroll
          for (int k = 0; k < K; ++k) {
            const int64_t idx = seg + lid + k * VS;
            const bool act = idx < len[i];
            int c = 0;
            T x = T(0);
            if (act) {
              c = __ldg(colidx + start[i] + idx);
              x = __ldg(val + start[i] + idx);
            }
            W_ADD(c, x * q[i], act);
          }
      }
    }
  }
  if constexpr (YM == 2) fpd::flush_loss(a.epi, loss_acc);

  if constexpr (MODE == MODE_PRIVATE) {
    __syncthreads();
    for (int64_t j = threadIdx.x; j < n; j += BS) {  // fixed warp order: deterministic in the CTA
      T s = w_s[j];
#pragma unroll
      for (int ww = 1; ww < NW; ++ww) s += w_s[(int64_t)ww * n + j];
      w_s[j] = s;
    }
    __syncthreads();
    fpd::grid_finalize<T, T>(w_s, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z,
                             a.accumulate);
  } else if constexpr (MODE == MODE_SHARED) {
    __syncthreads();
    fpd::grid_finalize<T, T>(w_s, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z,
                             a.accumulate);
  } else if constexpr (MODE == MODE_FIXED) {
    __syncthreads();
    fpd::fix_to_double<BS>(FA, n);
    __syncthreads();
    fpd::grid_finalize<T, double>(FA.sp, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z,
                                  a.accumulate);
  }
}

// ------------------------------------------------------------------------------ dispatch
constexpr int kCsrBS = 256;
using CsrKFn = void (*)(const CsrKArgs);

}  // namespace fp
#include "csr_colsplit.cuh"
#include "csr_flat.cuh"
#include "csr_owner.cuh"
#include "csr_stream.cuh"
namespace fp {

// column-split cluster kernels (csr_colsplit.cuh): 512 threads, NB in {8, 16} register tiles
constexpr int kSplitBS = 512;
using SplitKFn = void (*)(const SplitKArgs);

template <typename T, int YM, int NB>
SplitKFn csr_pick_colsplit_y(int cs) {
  switch (cs) {
    case 2: return k_csr_colsplit<T, 2, NB, YM, kSplitBS>;
    case 4: return k_csr_colsplit<T, 4, NB, YM, kSplitBS>;
    case 8: return k_csr_colsplit<T, 8, NB, YM, kSplitBS>;
    default: return nullptr;
  }
}
template <typename T, int NB>
SplitKFn csr_pick_colsplit_nb(int ym, int cs) {
  switch (ym) {
    case 0: return csr_pick_colsplit_y<T, 0, NB>(cs);
    case 1: return csr_pick_colsplit_y<T, 1, NB>(cs);
    case 2: return csr_pick_colsplit_y<T, 2, NB>(cs);
    default: return nullptr;
  }
}
template <typename T>
SplitKFn csr_pick_colsplit_t(int ym, int cs, int nb) {
  return nb == 8 ? csr_pick_colsplit_nb<T, 8>(ym, cs) : (nb == 16 ? csr_pick_colsplit_nb<T, 16>(ym, cs) : nullptr);
}
SplitKFn csr_pick_colsplit_f32(int ym, int cs, int nb);  // csr_split_f32.cu
SplitKFn csr_pick_colsplit_f64(int ym, int cs, int nb);  // csr_split_f64.cu
inline size_t colsplit_smem(fp_dtype dt, int cs, int width, bool has_y) {
  const size_t s = dt == FP_F64 ? 8 : 4;
  return (size_t)(kSplitBS / 32) * (2 * cs + 1) * 32 * s + (size_t)width * s * (has_y ? 2 : 1);
}

template <typename T, int YM, int NPT>
CsrKFn csr_pick_owner_n(int vs, int k) {
#define FP_CSR_OW(VS_, K_, RPV_) \
  if (vs == VS_ && k == K_) return k_csr_owner<T, VS_, K_, RPV_, YM, NPT, kCsrBS>;
  FP_CSR_OW(4, 4, 2) FP_CSR_OW(8, 2, 2) FP_CSR_OW(16, 2, 2) FP_CSR_OW(32, 4, 2)
#undef FP_CSR_OW
  return nullptr;
}

// dispatch modes of the flat kernel (aggregation as MODE_SHARED / MODE_L2); k = NB tiles
enum { DMODE_FLAT_SHARED = 3, DMODE_FLAT_L2 = 4, DMODE_FLAT_PRIVATE = 5, DMODE_OWNER4 = 6, DMODE_OWNER8 = 7,
       DMODE_FLAT_FIXED = 9, DMODE_STREAM_SHARED = 10, DMODE_STREAM_FIXED = 11, DMODE_FLAT_L2_WIDE = 12 };
constexpr int kWideBS = 1024;  // variant 16: one 1024-thread CTA per SM, a y prefix in shared memory

// stream kernels (csr_stream.cuh): (VS, K) as for CSR-vector; no row epilogues (YM 2)
template <typename T, int YM, int MODE>
CsrKFn csr_pick_stream(int vs, int k) {
  if constexpr (YM == 2) {
    return nullptr;
  } else {
#define FP_CSR_S(VS_, K_) \
  if (vs == VS_ && k == K_) return k_csr_stream<T, VS_, K_, YM, MODE, kCsrBS>;
    FP_CSR_S(2, 4) FP_CSR_S(4, 4) FP_CSR_S(8, 2) FP_CSR_S(16, 2) FP_CSR_S(32, 4)
#undef FP_CSR_S
    return nullptr;
  }
}

template <typename T, int YM, int MODE>
CsrKFn csr_pick_flat(int nb) {
  switch (nb) {
    case 2: return k_csr_flat<T, 2, YM, MODE, kCsrBS>;
    case 4: return k_csr_flat<T, 4, YM, MODE, kCsrBS>;
    case 8: return k_csr_flat<T, 8, YM, MODE, kCsrBS>;
    default: return nullptr;
  }
}

// (VS, K) -> kernel: a vector caches VS*K nonzeros of a row in registers; RPV row groups per
// warp iteration (1 for VS <= 2, else 2).  K is fp_launch.tl for the CSR variants.
template <typename T, int YM, int MODE>
CsrKFn csr_pick_vs(int vs, int k) {
#define FP_CSR_K(VS_, K_, RPV_) \
  if (vs == VS_ && k == K_) return k_csr_vector<T, VS_, K_, RPV_, YM, MODE, kCsrBS>;
  FP_CSR_K(1, 2, 1) FP_CSR_K(1, 4, 1) FP_CSR_K(1, 12, 1) FP_CSR_K(1, 16, 1) FP_CSR_K(2, 2, 1) FP_CSR_K(2, 4, 1)
  FP_CSR_K(2, 8, 1) FP_CSR_K(4, 4, 1)
  FP_CSR_K(4, 2, 2) FP_CSR_K(8, 1, 2) FP_CSR_K(8, 2, 2)
  FP_CSR_K(16, 1, 2) FP_CSR_K(16, 2, 2) FP_CSR_K(32, 2, 2) FP_CSR_K(32, 4, 2)
#undef FP_CSR_K
  return nullptr;
}

template <typename T, int YM>
CsrKFn csr_pick_m(int mode, int vs, int k) {
  switch (mode) {
    case MODE_L2: return csr_pick_vs<T, YM, MODE_L2>(vs, k);
    case MODE_SHARED: return csr_pick_vs<T, YM, MODE_SHARED>(vs, k);
    case MODE_PRIVATE: return csr_pick_vs<T, YM, MODE_PRIVATE>(vs, k);
    case MODE_FIXED: return csr_pick_vs<T, YM, MODE_FIXED>(vs, k);
#ifdef FP_EXPERIMENTAL_VARIANTS
    // measured and never chosen: built only with FP_EXPERIMENTAL=1
    case DMODE_FLAT_FIXED: return csr_pick_flat<T, YM, MODE_FIXED>(k);
    case DMODE_OWNER4: return csr_pick_owner_n<T, YM, 4>(vs, k);
    case DMODE_OWNER8: return csr_pick_owner_n<T, YM, 8>(vs, k);
    case DMODE_STREAM_SHARED: return csr_pick_stream<T, YM, MODE_SHARED>(vs, k);
    case DMODE_STREAM_FIXED: return csr_pick_stream<T, YM, MODE_FIXED>(vs, k);
#endif
    case DMODE_FLAT_SHARED: return csr_pick_flat<T, YM, MODE_SHARED>(k);
    case DMODE_FLAT_L2: return csr_pick_flat<T, YM, MODE_L2>(k);
    case DMODE_FLAT_PRIVATE: return csr_pick_flat<T, YM, MODE_PRIVATE>(k);
    case DMODE_FLAT_L2_WIDE: return k == 8 ? k_csr_flat<T, 8, YM, MODE_L2, kWideBS> : nullptr;
    default: return nullptr;
  }
}

// ym: 0 = no y (Table 1 row 1), 1 = Eq. (1), 2 = Eq. (1) with a row epilogue
template <typename T>
CsrKFn csr_pick_t(int ym, int mode, int vs, int k) {
  switch (ym) {
    case 0: return csr_pick_m<T, 0>(mode, vs, k);
    case 1: return csr_pick_m<T, 1>(mode, vs, k);
    case 2: return csr_pick_m<T, 2>(mode, vs, k);
    default: return nullptr;
  }
}

CsrKFn csr_pick_f32(int ym, int mode, int vs, int k);  // csr_f32.cu
CsrKFn csr_pick_f64(int ym, int mode, int vs, int k);  // csr_f64.cu

}  // namespace fp
