// dense.cu -- fused dense kernels for Eq. (1), re-designing Algorithm 3
// and its generated form, Listing 2, for sm_100a.
//
// What is kept from the paper: a "vector" of VS threads per row, TL elements of the row per
// thread held in registers (l_X), y held in registers (l_y), the row's partial dot
// reduced inside the vector and scaled by v[row] (Alg. 3 l.10-22), the row immediately
// streamed back from the same registers into the thread's register partial of w (l_w,
// l.23-24), coarsening over rows (l.25), and full unrolling of every TL loop, which the
// paper obtains by code generation and we obtain by C++ template instantiation.
// What changed for B200:
//   - rows are fetched with 256-bit LDG.E.256 streaming loads (L1 no-allocate, L2
//     evict-first); RPV rows per vector are loaded before any is reduced, so each lane keeps
//     RPV*32 bytes in flight (memory-level parallelism instead of occupancy alone);
//   - the vector reduction is an xor-shuffle all-reduce, so every lane gets p[r]*v[r]
//     without the warp-synchronous volatile smem broadcast of Listing 2, which
//     is a race on Volta+ independent thread scheduling;
//   - no zero padding of X or y: predicated tails;
//   - aggregation: warp xor-shuffle across vectors -> CTA smem (fixed warp order) ->
//     fp64 grid accumulator + last-CTA finalize (aggregate.cuh) instead of per-thread
//     atomicAdd into a w pre-initialised with beta*z (Alg. 3 l.6-7, l.26-27).
//   - VS > 32 (Alg. 3 l.16-22) is the CTA variant: warp shuffle + smem across warps.
#include "aggregate.cuh"
#include "kernels.cuh"

namespace fp {

struct DenseKArgs {
  int64_t m, n, ld;
  const void* X;
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

// Warp-granular vector kernel: VS in {1,2,4,8,16,32} lanes per row, NCH chunks of E
// elements per lane (thread load TL = NCH*E), RPV rows per vector per iteration.
template <typename T, int VS, int NCH, int E, int RPV, bool HAS_Y, int BS>
__global__ void __launch_bounds__(BS) k_dense_vector(const DenseKArgs a) {
  constexpr int VPW = 32 / VS;       // vectors per warp
  constexpr int NW = BS / 32;        // warps per CTA
  constexpr int RPW = VPW * RPV;     // rows per warp iteration
  const T* __restrict__ X = (const T*)a.X;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int lid = lane & (VS - 1), vid = lane / VS;
  const int64_t m = a.m, n = a.n, ld = a.ld;
  const int64_t nfull = n / E;  // chunks lying completely inside the row

  T ly[NCH][E], lw[NCH][E];
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t col = (int64_t)(k * VS + lid) * E + e;
      ly[k][e] = (HAS_Y && col < n) ? y[col] : T(0);
      lw[k][e] = T(0);
    }

  const int64_t nwarps = (int64_t)gridDim.x * NW;
  for (int64_t base = ((int64_t)blockIdx.x * NW + warp) * RPW; base < m; base += nwarps * RPW) {
    T x[RPV][NCH][E];
    T vr[RPV];
    bool okr[RPV];
#pragma unroll
    for (int i = 0; i < RPV; ++i) {
      const int64_t row = base + vid * RPV + i;
      const bool ok = row < m;
      okr[i] = ok;
      vr[i] = ok ? (v ? v[row] : T(1)) : T(0);
      const T* xr = X + (ok ? row : 0) * ld;
#pragma unroll
      for (int k = 0; k < NCH; ++k) {
        const int64_t c = k * VS + lid;
        if (ok && c < nfull) {
          fpd::ld_chunk<E * (int)sizeof(T)>(xr + c * E, x[i][k]);
        } else {
#pragma unroll
          for (int e = 0; e < E; ++e) {
            const int64_t col = c * E + e;
            x[i][k][e] = (ok && col < n) ? xr[col] : T(0);
          }
        }
      }
    }
#pragma unroll
    for (int i = 0; i < RPV; ++i) {
      T q;
      if constexpr (HAS_Y) {
        T p = T(0);  // Eq. (2): X[r,:] . y, TL products per lane
#pragma unroll
        for (int k = 0; k < NCH; ++k)
#pragma unroll
          for (int e = 0; e < E; ++e) p = fma(x[i][k][e], ly[k][e], p);
        p = fpd::vector_allreduce<VS>(p);  // intra-vector reduce, every lane gets p[r]
        q = okr[i] ? p * vr[i] : T(0);     // rows past m contribute nothing (even if y has Inf)
      } else {
        q = vr[i];  // Table 1 row 1: alpha X^T v
      }
#pragma unroll
      for (int k = 0; k < NCH; ++k)  // Eq. (3): l_w += X[r,:]^T q, same registers
#pragma unroll
        for (int e = 0; e < E; ++e) lw[k][e] = fma(x[i][k][e], q, lw[k][e]);
    }
  }

  // ---- aggregation: vectors of a warp (xor over the vector-id lane bits) -> CTA -> grid
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e)
#pragma unroll
      for (int off = VS; off < 32; off <<= 1) lw[k][e] += __shfl_xor_sync(0xffffffffu, lw[k][e], off);

  extern __shared__ double sw[];  // n doubles
  for (int64_t j = threadIdx.x; j < n; j += BS) sw[j] = 0.0;
  __syncthreads();
  for (int ww = 0; ww < NW; ++ww) {  // fixed warp order: deterministic within the CTA
    if (warp == ww && vid == 0) {
#pragma unroll
      for (int k = 0; k < NCH; ++k)
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const int64_t col = (int64_t)(k * VS + lid) * E + e;
          if (col < n) sw[col] += (double)lw[k][e];
        }
    }
    __syncthreads();
  }
  fpd::grid_finalize<T, double>(sw, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z, a.accumulate);
}

// CTA-wide vector (VS = BS > 32; Alg. 3 l.16-22): all BS threads share one row at a time;
// intra-warp shuffle reduce, then the NW warp sums through double-buffered smem (one
// barrier per row).  Thread t owns chunks t, t+BS, ... (NCH of them).
template <typename T, int NCH, int E, bool HAS_Y, int BS>
__global__ void __launch_bounds__(BS) k_dense_cta(const DenseKArgs a) {
  constexpr int NW = BS / 32;
  const T* __restrict__ X = (const T*)a.X;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t m = a.m, n = a.n, ld = a.ld;
  const int64_t nfull = n / E;
  __shared__ T red[2][NW];

  T ly[NCH][E], lw[NCH][E];
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t col = (int64_t)(k * BS + tid) * E + e;
      ly[k][e] = (HAS_Y && col < n) ? y[col] : T(0);
      lw[k][e] = T(0);
    }
  int buf = 0;
  for (int64_t row = blockIdx.x; row < m; row += gridDim.x) {
    T x[NCH][E];
    const T* xr = X + row * ld;
    const T vr = v ? v[row] : T(1);
#pragma unroll
    for (int k = 0; k < NCH; ++k) {
      const int64_t c = k * BS + tid;
      if (c < nfull) {
        fpd::ld_chunk<E * (int)sizeof(T)>(xr + c * E, x[k]);
      } else {
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const int64_t col = c * E + e;
          x[k][e] = col < n ? xr[col] : T(0);
        }
      }
    }
    T q;
    if constexpr (HAS_Y) {
      T p = T(0);
#pragma unroll
      for (int k = 0; k < NCH; ++k)
#pragma unroll
        for (int e = 0; e < E; ++e) p = fma(x[k][e], ly[k][e], p);
      p = fpd::vector_allreduce<32>(p);  // intra-warp (Alg. 3 l.17)
      if (lane == 0) red[buf][warp] = p;
      __syncthreads();                   // l.18-19
      p = T(0);
#pragma unroll
      for (int i = 0; i < NW; ++i) p += red[buf][i];  // inter-warp (l.20), same order everywhere
      buf ^= 1;
      q = p * vr;
    } else {
      q = vr;
    }
#pragma unroll
    for (int k = 0; k < NCH; ++k)
#pragma unroll
      for (int e = 0; e < E; ++e) lw[k][e] = fma(x[k][e], q, lw[k][e]);
  }
  extern __shared__ double sw[];
  __syncthreads();
  // every column has exactly one owner thread in the CTA: no intra-CTA reduction needed
  for (int64_t j = tid; j < n; j += BS) sw[j] = 0.0;
  __syncthreads();
#pragma unroll
  for (int k = 0; k < NCH; ++k)
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const int64_t col = (int64_t)(k * BS + tid) * E + e;
      if (col < n) sw[col] = (double)lw[k][e];
    }
  __syncthreads();
  fpd::grid_finalize<T, double>(sw, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z, a.accumulate);
}

template <typename T>
__global__ void k_scale_z(int64_t n, const T* z, double beta, T* w) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
    w[j] = (beta != 0.0 && z) ? (T)(beta * (double)z[j]) : T(0);
}

fp_status launch_scale_z(int64_t n, const void* z, double beta, void* w, fp_dtype dt, cudaStream_t s) {
  if (n <= 0) return FP_OK;
  int grid = (int)((n + 255) / 256);
  if (grid > 4096) grid = 4096;
  if (dt == FP_F64) k_scale_z<double><<<grid, 256, 0, s>>>(n, (const double*)z, beta, (double*)w);
  else k_scale_z<float><<<grid, 256, 0, s>>>(n, (const float*)z, beta, (float*)w);
  FP_CUDA(cudaGetLastError());
  return FP_OK;
}

// ------------------------------------------------------------------------------ dispatch
namespace {

constexpr int kBS = 256;  // dense vector kernel block size
constexpr int kBSCta = 256;

using KFn = void (*)(const DenseKArgs);

// Rows per vector per iteration: keep ~64-128 B per lane in flight.
constexpr int rpv_for(int nch, int eb) { return nch * eb <= 32 ? 4 : (nch * eb <= 64 ? 2 : 1); }

template <typename T, int E, bool HY>
KFn pick_vector(int vs, int nch) {
  constexpr int EB = E * (int)sizeof(T);
  switch (vs) {
    case 1: return k_dense_vector<T, 1, 1, E, 4, HY, kBS>;
    case 2: return k_dense_vector<T, 2, 1, E, 4, HY, kBS>;
    case 4: return k_dense_vector<T, 4, 1, E, 4, HY, kBS>;
    case 8: return k_dense_vector<T, 8, 1, E, 4, HY, kBS>;
    case 16: return k_dense_vector<T, 16, 1, E, rpv_for(1, EB), HY, kBS>;
    case 32:
      switch (nch) {
        case 1: return k_dense_vector<T, 32, 1, E, rpv_for(1, EB), HY, kBS>;
        case 2: return k_dense_vector<T, 32, 2, E, rpv_for(2, EB), HY, kBS>;
        case 3: return k_dense_vector<T, 32, 3, E, rpv_for(3, EB), HY, kBS>;
        case 4: return k_dense_vector<T, 32, 4, E, rpv_for(4, EB), HY, kBS>;
        case 6: return k_dense_vector<T, 32, 6, E, rpv_for(6, EB), HY, kBS>;
        case 8: return k_dense_vector<T, 32, 8, E, rpv_for(8, EB), HY, kBS>;
        default: return nullptr;
      }
    default: return nullptr;
  }
}

template <typename T, int E, bool HY>
KFn pick_cta(int nch) {
  switch (nch) {
    case 1: return k_dense_cta<T, 1, E, HY, kBSCta>;
    case 2: return k_dense_cta<T, 2, E, HY, kBSCta>;
    case 4: return k_dense_cta<T, 4, E, HY, kBSCta>;
    case 8: return k_dense_cta<T, 8, E, HY, kBSCta>;
    default: return nullptr;
  }
}

// E32 = elements per 32-byte chunk; scalar path E = 1.
template <typename T, bool HY>
KFn pick(int variant, int chunk_elems, int vs, int nch) {
  constexpr int E32 = 32 / (int)sizeof(T);
  if (variant == FP_VAR_DENSE_VECTOR) {
    if (chunk_elems == E32) return pick_vector<T, E32, HY>(vs, nch);
    if (chunk_elems == 1) return pick_vector<T, 1, HY>(vs, nch);
  } else if (variant == FP_VAR_DENSE_CTA) {
    if (chunk_elems == E32) return pick_cta<T, E32, HY>(nch);
    if (chunk_elems == 1) return pick_cta<T, 1, HY>(nch);
  }
  return nullptr;
}

KFn pick_any(const PatternArgs& a, const fp_launch& L) {
  const bool hy = a.y != nullptr;
  // L.tl = thread load (elements per thread) = nch * chunk_elems; chunk_elems from alignment
  const int e32 = 32 / (int)dtype_size(a.dtype);
  const bool aligned = ((uintptr_t)a.X % 32 == 0) && ((a.ld * (int64_t)dtype_size(a.dtype)) % 32 == 0);
  const int ce = aligned ? e32 : 1;
  if (L.tl % ce != 0) return nullptr;
  const int nch = L.tl / ce;
  if (a.dtype == FP_F64) return hy ? pick<double, true>(L.variant, ce, L.vs, nch) : pick<double, false>(L.variant, ce, L.vs, nch);
  return hy ? pick<float, true>(L.variant, ce, L.vs, nch) : pick<float, false>(L.variant, ce, L.vs, nch);
}

int round_nch(int need, bool cta) {
  static const int vec_set[] = {1, 2, 3, 4, 6, 8};
  static const int cta_set[] = {1, 2, 4, 8};
  const int* s = cta ? cta_set : vec_set;
  int cnt = cta ? 4 : 6;
  for (int i = 0; i < cnt; ++i)
    if (s[i] >= need) return s[i];
  return -1;
}

}  // namespace

// B200 dense plan.  Chunk = 32 bytes when X and ld*sizeof(T) are 32-byte aligned (LDG.256),
// else 1 element.  chunks/row = ceil(n / E).  VS = next power of two >= chunks (one chunk per
// lane) up to 32 -- Eq. (6) with TL = E; beyond 32 chunks VS = 32 and TL grows
// (NCH chunks per lane, NCH in {2,3,4,6,8}); beyond that the CTA variant (VS = BS, P:400
// first case).  grid = SMs x resident CTAs (persistent; coarsening C = rows / vectors).
fp_status plan_dense(const PatternArgs& a, int device, fp_launch* out) {
  const DeviceInfo& di = device_info(device);
  const int s = (int)dtype_size(a.dtype);
  const bool aligned = ((uintptr_t)a.X % 32 == 0) && ((a.ld * (int64_t)s) % 32 == 0);
  const int ce = aligned ? 32 / s : 1;
  const int64_t chunks = (a.n + ce - 1) / ce;
  fp_launch L{};
  if (chunks <= 32) {
    int vs = 1;
    while (vs < chunks) vs <<= 1;
    L.variant = FP_VAR_DENSE_VECTOR;
    L.vs = vs;
    L.tl = ce;
    L.bs = kBS;
  } else {
    int nch = round_nch((int)((chunks + 31) / 32), false);
    if (nch > 0 && (int64_t)nch * ce * s <= 256) {  // <= 64 fp32 / 32 fp64 elements per lane
      L.variant = FP_VAR_DENSE_VECTOR;
      L.vs = 32;
      L.tl = nch * ce;
      L.bs = kBS;
    } else {
      nch = round_nch((int)((chunks + kBSCta - 1) / kBSCta), true);
      if (nch < 0 || (int64_t)nch * ce * s > 256) {
        set_error("fp_dense: n=%lld exceeds the register-resident row limit (%d B per thread x %d threads); "
                  "wide-n dense is not implemented (DESIGN.md NEXT-4)",
                  (long long)a.n, 256, kBSCta);
        return FP_ERR_UNSUPPORTED;
      }
      L.variant = FP_VAR_DENSE_CTA;
      L.vs = kBSCta;
      L.tl = nch * ce;
      L.bs = kBSCta;
    }
  }
  KFn f = pick_any(a, L);
  if (!f) {
    set_error("fp_dense: no kernel instantiation for vs=%d tl=%d", L.vs, L.tl);
    return FP_ERR_UNSUPPORTED;
  }
  L.smem_bytes = (int)(a.n * sizeof(double));
  int per_sm = 0;
  if (L.smem_bytes > 48 * 1024) cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, L.smem_bytes);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, f, L.bs, L.smem_bytes);
  if (per_sm < 1) per_sm = 1;
  cudaFuncAttributes fa{};
  cudaFuncGetAttributes(&fa, f);
  L.regs_per_thread = fa.numRegs;
  L.blocks_per_sm = per_sm;
  L.concurrent_warps = per_sm * L.bs / 32;
  int64_t vectors_per_cta = L.variant == FP_VAR_DENSE_CTA ? 1 : L.bs / L.vs;
  int64_t need_ctas = (a.m + vectors_per_cta - 1) / vectors_per_cta;
  int64_t grid = (int64_t)di.sm_count * per_sm;
  if (need_ctas < grid) grid = need_ctas > 0 ? need_ctas : 1;
  L.grid = (int)grid;
  L.rows_per_vector = (a.m + grid * vectors_per_cta - 1) / (grid * vectors_per_cta);
  *out = L;
  return FP_OK;
}

int dense_kernel_regs(const PatternArgs& a, const fp_launch& L) {
  KFn f = pick_any(a, L);
  if (!f) return 0;
  cudaFuncAttributes fa{};
  if (cudaFuncGetAttributes(&fa, f) != cudaSuccess) return 0;
  return fa.numRegs;
}

fp_status launch_dense(const PatternArgs& a, const fp_launch& L, cudaStream_t s) {
  KFn f = pick_any(a, L);
  FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_dense: launch plan (variant=%d vs=%d tl=%d) has no kernel", L.variant, L.vs,
             L.tl);
  FP_REQUIRE(L.bs == (L.variant == FP_VAR_DENSE_CTA ? kBSCta : kBS), FP_ERR_UNSUPPORTED,
             "fp_dense: block size %d not supported by the selected kernel", L.bs);
  FP_REQUIRE(L.grid >= 1, FP_ERR_INVALID_ARG, "fp_dense: grid must be >= 1");
  Workspace* ws = workspace(s, (size_t)a.n, 0);
  if (!ws) return FP_ERR_NOMEM;
  DenseKArgs k{a.m, a.n, a.ld, a.X, a.y, a.v, a.z, a.alpha, a.beta, a.w, ws->acc, ws->counters, a.add_beta_z ? 1 : 0,
                 a.accumulate ? 1 : 0};
  size_t smem = (size_t)a.n * sizeof(double);
  if (smem > 48 * 1024) FP_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  f<<<L.grid, L.bs, smem, s>>>(k);
  FP_CUDA(cudaGetLastError());
  return FP_OK;
}

}  // namespace fp
