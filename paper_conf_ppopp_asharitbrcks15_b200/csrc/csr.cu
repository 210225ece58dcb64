// csr.cu -- fused CSR kernels for Eq. (1), re-designing Algorithms 1-2
// for sm_100a.
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
//   - y is staged in shared memory when n fits (the paper bound y to texture);
//   - large n: beta*z (rank 0) / 0 pre-written by a tiny kernel, then fire-and-forget
//     REDG.E.ADD into the L2-resident w (alpha folded into q); small n: shared partial +
//     fp64 grid accumulator + last-CTA finalize (aggregate.cuh).
#include "aggregate.cuh"
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
};

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

// VS lanes per row, K nonzeros per lane cached in registers (rows up to VS*K are read from
// HBM exactly once; longer rows re-read their tail from L1/L2 for the scatter, the paper's
// "likely a cache hit"), RPV row groups per warp iteration.
// SMEM: partial w (and y) in shared memory; else L2 path (REDG into w).
template <typename T, int VS, int K, int RPV, bool HAS_Y, bool SMEM, int BS>
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

  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* w_s = reinterpret_cast<T*>(smem_raw);  // [n] partial w   (SMEM only)
  T* y_s = w_s + n;                         // [n] staged y    (SMEM && HAS_Y)
  if constexpr (SMEM) {
    for (int64_t j = threadIdx.x; j < n; j += BS) {
      w_s[j] = T(0);
      if constexpr (HAS_Y) y_s[j] = y[j];
    }
    __syncthreads();
  }
  // alpha: folded into q on the L2 path, applied once by the finaliser on the smem path
  const T qscale = SMEM ? T(1) : (T)a.alpha;

  // ---- this warp's row range, balanced by nnz + kRowCost*rows
  const int64_t gw = (int64_t)blockIdx.x * NW + warp, tw = (int64_t)gridDim.x * NW;
  const int64_t total = a.nnz + kRowCost * m;
  const int64_t r0 = warp_search_rows(rowptr, m, (total * gw) / tw, lane);
  const int64_t r1 = warp_search_rows(rowptr, m, (total * (gw + 1)) / tw, lane);

  int64_t bstart = r0;  // rows [bstart, bstart+32) have their rowptr in `rp` (lane i: row bstart+i)
  int64_t rp = (bstart + lane <= m) ? __ldg(rowptr + bstart + lane) : 0;
  int64_t rp32 = (bstart + 32 <= m) ? __ldg(rowptr + bstart + 32) : 0;

  for (int64_t rb = r0; rb < r1; rb += GROUP) {
    if (rb + GROUP > bstart + 32) {  // refill the rowptr batch (warp-uniform)
      bstart = rb;
      rp = (bstart + lane <= m) ? __ldg(rowptr + bstart + lane) : 0;
      rp32 = (bstart + 32 <= m) ? __ldg(rowptr + bstart + 32) : 0;
    }
    int64_t start[RPV], len[RPV];
    T vr[RPV];
    bool any_long = false;
#pragma unroll
    for (int i = 0; i < RPV; ++i) {
      const int64_t row = rb + i * VPW + vid;
      const int o = (int)(row - bstart);
      const int64_t s0 = __shfl_sync(0xffffffffu, rp, o & 31);
      const int64_t s1n = __shfl_sync(0xffffffffu, rp, (o + 1) & 31);
      const int64_t s1 = (o + 1 == 32) ? rp32 : s1n;
      const bool ok = row < r1;
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
#pragma unroll
      for (int i = 0; i < RPV; ++i) {  // Eq. (2) / Alg. 2 l.10-11
        p[i] = T(0);
#pragma unroll
        for (int k = 0; k < K; ++k)
          if (lid + k * VS < len[i]) p[i] = fma(xv[i][k], SMEM ? y_s[cc[i][k]] : __ldg(y + cc[i][k]), p[i]);
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
                p[i] = fma(__ldg(val + start[i] + idx), SMEM ? y_s[c] : __ldg(y + c), p[i]);
              }
            }
        }
      }
#pragma unroll
      for (int i = 0; i < RPV; ++i) q[i] = fpd::vector_allreduce<VS>(p[i]) * vr[i] * qscale;  // l.12
    } else {
#pragma unroll
      for (int i = 0; i < RPV; ++i) q[i] = vr[i] * qscale;
    }

    // ---- second touch from registers: Eq. (3) / Alg. 2 l.13-14
#pragma unroll
    for (int i = 0; i < RPV; ++i)
#pragma unroll
      for (int k = 0; k < K; ++k) {
        if (lid + k * VS < len[i]) {
          if constexpr (SMEM) atomicAdd(w_s + cc[i][k], xv[i][k] * q[i]);
          else fpd::red_add((T*)a.w + cc[i][k], xv[i][k] * q[i]);
        }
      }
    if (any_long) {
      for (int64_t seg = VS * K; seg < lmax; seg += VS * K) {
#pragma unroll
        for (int i = 0; i < RPV; ++i)
#pragma unroll
          for (int k = 0; k < K; ++k) {
            const int64_t idx = seg + lid + k * VS;
            if (idx < len[i]) {
              const int c = __ldg(colidx + start[i] + idx);
              const T x = __ldg(val + start[i] + idx);
              if constexpr (SMEM) atomicAdd(w_s + c, x * q[i]);
              else fpd::red_add((T*)a.w + c, x * q[i]);
            }
          }
      }
    }
  }

  if constexpr (SMEM) {
    __syncthreads();
    fpd::grid_finalize<T, T>(w_s, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z, a.accumulate);
  }
}

// ------------------------------------------------------------------------------ dispatch
namespace {

constexpr int kBS = 256;
using KFn = void (*)(const CsrKArgs);

// VS -> (K, RPV): a vector caches VS*K nonzeros per row; RPV row groups per iteration.
template <typename T, bool HY, bool SM>
KFn pick_vs(int vs) {
  switch (vs) {
    case 1: return k_csr_vector<T, 1, 2, 1, HY, SM, kBS>;
    case 2: return k_csr_vector<T, 2, 2, 1, HY, SM, kBS>;
    case 4: return k_csr_vector<T, 4, 2, 2, HY, SM, kBS>;
    case 8: return k_csr_vector<T, 8, 2, 2, HY, SM, kBS>;
    case 16: return k_csr_vector<T, 16, 2, 2, HY, SM, kBS>;
    case 32: return k_csr_vector<T, 32, 4, 2, HY, SM, kBS>;
    default: return nullptr;
  }
}

KFn pick_any(const PatternArgs& a, const fp_launch& L) {
  const bool hy = a.y != nullptr;
  const bool sm = L.variant == FP_VAR_CSR_VECTOR;
  if (L.variant != FP_VAR_CSR_VECTOR && L.variant != FP_VAR_CSR_VECTOR_L2) return nullptr;
  if (a.dtype == FP_F64) {
    if (hy) return sm ? pick_vs<double, true, true>(L.vs) : pick_vs<double, true, false>(L.vs);
    return sm ? pick_vs<double, false, true>(L.vs) : pick_vs<double, false, false>(L.vs);
  }
  if (hy) return sm ? pick_vs<float, true, true>(L.vs) : pick_vs<float, true, false>(L.vs);
  return sm ? pick_vs<float, false, true>(L.vs) : pick_vs<float, false, false>(L.vs);
}

size_t smem_for(const PatternArgs& a, int variant) {
  if (variant != FP_VAR_CSR_VECTOR) return 0;
  return (size_t)a.n * dtype_size(a.dtype) * (a.y ? 2 : 1);
}

}  // namespace

// Eq. (4): VS = 32 if mu > 32; 2^i if 2^(i+1) >= mu > 2^i (i in 1..4); else 1.
int eq4_vector_size(double mu) {
  if (mu > 32) return 32;
  for (int i = 4; i >= 1; --i)
    if (mu > (double)(1 << i)) return 1 << i;
  return 1;
}

constexpr size_t kSmemBudget = 64 * 1024;  // y + partial w per CTA for the smem variant

fp_status plan_csr(const PatternArgs& a, int device, fp_launch* out) {
  const DeviceInfo& di = device_info(device);
  fp_launch L{};
  const double mu = a.m > 0 ? (double)a.nnz / (double)a.m : 0.0;
  L.vs = eq4_vector_size(mu);
  L.bs = kBS;
  L.variant = ((size_t)a.n * dtype_size(a.dtype) * (a.y ? 2 : 1) <= kSmemBudget) ? FP_VAR_CSR_VECTOR
                                                                                    : FP_VAR_CSR_VECTOR_L2;
  L.smem_bytes = (int)smem_for(a, L.variant);
  KFn f = pick_any(a, L);
  FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_csr: no kernel for vs=%d", L.vs);
  if (L.smem_bytes > 48 * 1024) cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, L.smem_bytes);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, f, L.bs, L.smem_bytes);
  if (per_sm < 1) per_sm = 1;
  cudaFuncAttributes fa{};
  cudaFuncGetAttributes(&fa, f);
  L.regs_per_thread = fa.numRegs;
  L.blocks_per_sm = per_sm;
  L.concurrent_warps = per_sm * L.bs / 32;
  L.tl = 0;
  int64_t grid = (int64_t)di.sm_count * per_sm;
  int64_t need = (a.m + (L.bs / L.vs) - 1) / (L.bs / L.vs);  // one row per vector at least
  if (need < 1) need = 1;
  if (grid > need) grid = need;
  L.grid = (int)grid;
  const int64_t vectors = grid * (L.bs / L.vs);
  L.rows_per_vector = (a.m + vectors - 1) / vectors;
  *out = L;
  return FP_OK;
}

fp_status launch_csr(const PatternArgs& a, const fp_launch& L, cudaStream_t s) {
  KFn f = pick_any(a, L);
  FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_csr: launch plan (variant=%d vs=%d) has no kernel", L.variant, L.vs);
  FP_REQUIRE(L.bs == kBS, FP_ERR_UNSUPPORTED, "fp_csr: block size %d not supported", L.bs);
  FP_REQUIRE(L.grid >= 1, FP_ERR_INVALID_ARG, "fp_csr: grid must be >= 1");
  const bool smem_path = L.variant == FP_VAR_CSR_VECTOR;
  const size_t smem = smem_for(a, L.variant);
  Workspace* ws = workspace(s, smem_path ? (size_t)a.n : 0, 0);
  if (!ws) return FP_ERR_NOMEM;
  if (!smem_path && !a.accumulate) {  // L2 path: w <- beta z (or 0) first, kernel reduces alpha X^T q into it
    fp_status st = launch_scale_z(a.n, a.add_beta_z ? a.z : nullptr, a.add_beta_z ? a.beta : 0.0, a.w, a.dtype, s);
    if (st != FP_OK) return st;
  }
  CsrKArgs k{a.m, a.n, a.nnz, a.rowptr, a.colidx, a.val, a.y, a.v, a.z, a.alpha, a.beta, a.w,
             ws->acc, ws->counters, a.add_beta_z ? 1 : 0, a.accumulate ? 1 : 0};
  if (smem > 48 * 1024) FP_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  f<<<L.grid, L.bs, smem, s>>>(k);
  FP_CUDA(cudaGetLastError());
  return FP_OK;
}

}  // namespace fp
