// csr.cu -- B200 plan and launch of the fused CSR kernels (csr_kernels.cuh).
#include <algorithm>
#include <cstdlib>

#include "csr_kernels.cuh"

namespace fp {

namespace {

bool is_flat(int variant) {
  return (variant >= FP_VAR_CSR_FLAT && variant <= FP_VAR_CSR_FLAT_PRIVATE) || variant == FP_VAR_CSR_FLAT_FIXED ||
         variant == FP_VAR_CSR_FLAT_L2_WIDE || variant == FP_VAR_CSR_BINNED;
}

int mode_of(int variant) {
  switch (variant) {
    case FP_VAR_CSR_VECTOR: return MODE_SHARED;
    case FP_VAR_CSR_VECTOR_L2: return MODE_L2;
    case FP_VAR_CSR_VECTOR_PRIVATE: return MODE_PRIVATE;
    case FP_VAR_CSR_FLAT: return DMODE_FLAT_SHARED;
    case FP_VAR_CSR_FLAT_L2: return DMODE_FLAT_L2;
    case FP_VAR_CSR_FLAT_PRIVATE: return DMODE_FLAT_PRIVATE;
    case FP_VAR_CSR_VECTOR_FIXED: return MODE_FIXED;
    case FP_VAR_CSR_FLAT_FIXED: return DMODE_FLAT_FIXED;
    case FP_VAR_CSR_STREAM: return DMODE_STREAM_SHARED;
    case FP_VAR_CSR_STREAM_FIXED: return DMODE_STREAM_FIXED;
    case FP_VAR_CSR_FLAT_L2_WIDE: return DMODE_FLAT_L2_WIDE;
    default: return -1;
  }
}

// entries per lane cached in registers: VS*K covers ~1.6x the mean row for the VS Eq. (4) picks
int default_k(int vs) { return (vs == 8 || vs == 16) ? 2 : (vs == 32 ? 4 : 4); }

CsrKFn pick_any(const PatternArgs& a, const fp_launch& L) {
  int mode = mode_of(L.variant);
  if (L.variant == FP_VAR_CSR_OWNER) mode = a.n <= 4 * kCsrBS ? DMODE_OWNER4 : (a.n <= 8 * kCsrBS ? DMODE_OWNER8 : -1);
  if (mode < 0) return nullptr;
  const int ym = !a.y ? 0 : ((a.epi_kind == 0 && !a.row_out) ? 1 : 2);
  const bool flat = is_flat(L.variant);
  const int k = L.tl > 0 ? L.tl : (flat ? 4 : default_k(L.vs));
  return a.dtype == FP_F64 ? csr_pick_f64(ym, mode, L.vs, k) : csr_pick_f32(ym, mode, L.vs, k);
}

constexpr size_t kPrivateBudget = 100 * 1024;  // y + NW warp partials per CTA
constexpr size_t kSharedBudget = 64 * 1024;    // y + one CTA partial
constexpr size_t kYBudget = 96 * 1024;         // y staged in smem on the L2 path
constexpr int64_t kBinMinNnz = 1 << 24;         // variant 17 only from 16M nonzeros

// w += sum of the replicas; the replicas are re-zeroed (the workspace invariant)
template <typename T>
__global__ void k_fold_replicas(T* __restrict__ w, T* __restrict__ rep, int64_t n, int nr) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    T s = w[j];
    for (int r = 0; r < nr; ++r) {
      s += rep[(int64_t)r * n + j];
      rep[(int64_t)r * n + j] = T(0);
    }
    w[j] = s;
  }
}

// Copies of w for the L2 path: the random reds of all CTAs into ONE n-vector leave some L2
// slices near saturation while others idle (C4 ncu: lts__t_tag_requests avg 62 %, max 84 %,
// min 32 %); 8 copies (CTA b reduces into copy b mod 8) measured 20.3 -> 18.7 ms on C4.  Only
// while the copies stay small against L2 (126 MB).  FP_L2_REPLICAS overrides (measurement).
constexpr int kL2Replicas = 8;
constexpr size_t kL2ReplicaBudget = 16u << 20;
int l2_replicas(const PatternArgs& a) {
  static const int env = [] {
    const char* e = std::getenv("FP_L2_REPLICAS");
    return e ? std::atoi(e) : 0;
  }();
  if (env > 0) return std::min(env, 16);
  return (size_t)kL2Replicas * a.n * dtype_size(a.dtype) <= kL2ReplicaBudget ? kL2Replicas : 1;
}

bool y_in_smem_l2(const PatternArgs& a) { return a.y && (size_t)a.n * dtype_size(a.dtype) <= kYBudget; }

// variant 16: shared memory of the 1024-thread CTA left for a y prefix: 227 KB minus the
// static per-warp row sums (32 warps x 32 x s) and a little slack
int64_t wide_y_entries(const PatternArgs& a) {
  if (!a.y) return 0;
  const size_t budget = 227 * 1024 - (size_t)(kWideBS / 32) * 32 * dtype_size(a.dtype) - 512;
  const int64_t cap = (int64_t)(budget / dtype_size(a.dtype)) / 4 * 4;
  return a.n < cap ? a.n : cap;
}
// entries of y the L2-path kernels stage in shared memory (CsrKArgs::y_in_smem)
int l2_y_entries(const PatternArgs& a, int variant) {
  if (variant == FP_VAR_CSR_FLAT_L2_WIDE) return (int)wide_y_entries(a);
  return y_in_smem_l2(a) ? (int)a.n : 0;
}

size_t smem_for(const PatternArgs& a, int variant) {
  const size_t vb = (size_t)a.n * dtype_size(a.dtype);
  const size_t yb = a.y ? vb : 0;
  switch (variant) {
    case FP_VAR_CSR_VECTOR_PRIVATE:
    case FP_VAR_CSR_FLAT_PRIVATE: return yb + (size_t)(kCsrBS / 32) * vb;
    case FP_VAR_CSR_OWNER:  // y + spill partial + queues (values, 1-byte hi, counters)
      return yb + vb + (size_t)kOwnerQ * kCsrBS * (dtype_size(a.dtype) + 1) + (size_t)kCsrBS * 4;
    case FP_VAR_CSR_VECTOR:
    case FP_VAR_CSR_FLAT: return yb + vb;
    case FP_VAR_CSR_VECTOR_FIXED:  // y (16-byte aligned) + fp64 spill + two 32-bit limbs per column
    case FP_VAR_CSR_FLAT_FIXED: return (size_t)(a.y ? fix_y_bytes(a.n, (int)dtype_size(a.dtype)) : 0) + (size_t)a.n * 16;
    case FP_VAR_CSR_VECTOR_L2:
    case FP_VAR_CSR_FLAT_L2: return y_in_smem_l2(a) ? vb : 0;
    case FP_VAR_CSR_FLAT_L2_WIDE:
    case FP_VAR_CSR_BINNED: return (size_t)wide_y_entries(a) * dtype_size(a.dtype);
    case FP_VAR_CSR_STREAM:  // y (16-byte padded) + partial + two stages per warp
    case FP_VAR_CSR_STREAM_FIXED: {
      const size_t s = dtype_size(a.dtype);
      const size_t part = variant == FP_VAR_CSR_STREAM_FIXED ? (size_t)a.n * 16 : (vb + 15) / 16 * 16;
      const size_t stage = s == 8 ? (size_t)stream_stage_bytes<double>() : (size_t)stream_stage_bytes<float>();
      return (a.y ? (size_t)fix_y_bytes(a.n, (int)s) : 0) + part + (size_t)(kCsrBS / 32) * 2 * stage;
    }
    default: return 0;
  }
}

// owner-computes: row-group iterations per phase so that one phase fills the queues to about
// half (BS * kOwnerQ / 2 entries per CTA) at the mean row length
int phase_iters_for(const PatternArgs& a, const fp_launch& L) {
  if (L.variant != FP_VAR_CSR_OWNER) return 0;
  const double mu = a.m > 0 ? (double)a.nnz / (double)a.m : 1.0;
  const int rpv = 2;
  const double per_iter = (double)(kCsrBS / 32) * (32 / (L.vs > 0 ? L.vs : 32)) * rpv * (mu > 1.0 ? mu : 1.0);
  int pi = (int)((kCsrBS * kOwnerQ / 2) / per_iter);
  return pi < 1 ? 1 : pi;
}


}  // namespace

// Eq. (4): VS = 32 if mu > 32; 2^i if 2^(i+1) >= mu > 2^i (i in 1..4); else 1.
int eq4_vector_size(double mu) {
  if (mu > 32) return 32;
  for (int i = 4; i >= 1; --i)
    if (mu > (double)(1 << i)) return 1 << i;
  return 1;
}

// B200 CSR plan: VS by Eq. (4); aggregation mode by what fits on chip -- per-warp private
// partials (no atomics) when y + 8 warp copies fit in 100 KB, else one shared CTA partial
// when y + w fit in 64 KB, else red into the L2-resident w.  Persistent grid
// = SMs x resident CTAs from the occupancy API.
fp_status plan_csr(const PatternArgs& a, int device, fp_launch* out) {
  const DeviceInfo& di = device_info(device);
  fp_launch L{};
  const double mu = a.m > 0 ? (double)a.nnz / (double)a.m : 0.0;
  L.vs = eq4_vector_size(mu);
  L.bs = kCsrBS;
  // Measured on B200 (tools/sweep.py, profiles/r01_sweep_*.json): with y + w on chip the
  // paper's CSR-vector with the CTA-shared partial and Eq. (4)'s VS is within 2 % of the best
  // of ~300 settings (C3); the per-warp private and flat variants lose to it because fp64
  // shared-memory updates cost per instruction.  For large n the flat layout (lanes on
  // consecutive nonzeros, L2 reds) is best (C4: 17.3 ms vs 19.8 ms for CSR-vector).
  // Round-1 re-sweep after the y gathers were hoisted ahead of their use (every gather of a
  // row group in flight at once; profiles/r01_sweep2_{C3,S3}.json): with Eq. (4)'s VS = 8 bin
  // (8 < mu <= 16) the same 16 cached entries per row are faster as VS = 4 lanes x K = 4 than
  // as 8 x 2 (C3 fp64 1.14 vs 1.28 ms, S3 fp32 0.92 vs 1.06 ms: more independent loads per
  // lane, half the shuffle-reduce steps).  The fixed-point partial (variant 11) at 4 x 4 is 3 %
  // faster on fp64 and slower on fp32; the paper's shared partial is kept.
  if (smem_for(a, FP_VAR_CSR_VECTOR) <= kSharedBudget) L.variant = FP_VAR_CSR_VECTOR;
  else L.variant = FP_VAR_CSR_FLAT_L2;
  (void)kPrivateBudget;
  L.smem_bytes = (int)smem_for(a, L.variant);
  L.tl = is_flat(L.variant) ? 8 : default_k(L.vs);
  if (!is_flat(L.variant) && L.vs == 8) {
    L.vs = 4;
    L.tl = 4;
  }
  // Wide y on the L2 path: one 1024-thread CTA per SM with a y prefix in shared memory takes
  // that share of the gathers off the L2 request stream, the bound of this path (C4: 18.5 ->
  // 17.2 ms with 56 % of y staged).  Only when the prefix is a sizeable share of y; the
  // decision depends on (n, dtype) only, so a CSR plan made without y picks the same.
  if (L.variant == FP_VAR_CSR_FLAT_L2) {
    PatternArgs ay = a;
    ay.y = reinterpret_cast<const void*>(uintptr_t(256));
    if (4 * wide_y_entries(ay) >= a.n) {
      L.variant = FP_VAR_CSR_FLAT_L2_WIDE;
      L.bs = kWideBS;
      L.smem_bytes = (int)smem_for(a, L.variant);
    }
  }
  // Binned scatter (variant 17, csr_binned.cu): for fp32 and n up to 4 column blocks of one
  // SM's shared memory, when the matrix is large enough that the ~4 extra launches and the
  // message round trip (6 B per nonzero written and read) are repaid by removing the per-lane
  // global reds, and the message workspace fits in free device memory with 1 GB to spare.
  // FP_NO_BINNED=1 keeps variant 16 (A/B measurement).
  if (L.variant == FP_VAR_CSR_FLAT_L2_WIDE && a.dtype == FP_F32 && binned_nbin(a.n) > 0 && a.nnz >= kBinMinNnz &&
      a.epi_kind == 0 && !a.row_out && !std::getenv("FP_NO_BINNED")) {
    const int nb = binned_nbin(a.n);
    size_t fr = 0, tot = 0;
    const size_t need = binned_ws_bytes(a.n, a.nnz, nb, di.sm_count, di.sm_count);
    if (cudaMemGetInfo(&fr, &tot) == cudaSuccess && need + (1ull << 30) <= fr) {
      L.variant = FP_VAR_CSR_BINNED;
      L.cluster = nb;
    } else {
      cudaGetLastError();
    }
  }
  // fp64, y + w on chip, short rows: the flat-4 kernel with the fixed-point CTA partial
  // (variant 18) -- the best of 936 settings on C3 (profiles/r02_sweep_C3.json), 3.5 % ahead of
  // the CSR-vector / shared-partial plan; for fp32 the CSR-vector plan stays best (S3 sweep)
  if (L.variant == FP_VAR_CSR_VECTOR && a.dtype == FP_F64 && mu <= 32.0 && a.epi_kind == 0 && !a.row_out &&
      flat4_fixed_smem(a.n, a.dtype, true) <= kSharedBudget && !std::getenv("FP_NO_FLAT4")) {
    L.variant = FP_VAR_CSR_FLAT4_FIXED;
    L.vs = 32;
    L.tl = 8;
    L.bs = 256;
    const int occ = flat4_fixed_blocks_per_sm(a.n, a.dtype, true);
    L.blocks_per_sm = occ > 0 ? occ : 1;
    L.concurrent_warps = L.blocks_per_sm * L.bs / 32;
    L.grid = di.sm_count * L.blocks_per_sm;
    L.smem_bytes = (int)flat4_fixed_smem(a.n, a.dtype, true);
    L.rows_per_vector = (a.m + (int64_t)L.grid * 8 - 1) / ((int64_t)L.grid * 8);
    *out = L;
    return FP_OK;
  }
  if (L.variant == FP_VAR_CSR_BINNED) {  // one producer CTA of 1024 threads per SM
    L.regs_per_thread = binned_producer_regs(a.y != nullptr);
    L.blocks_per_sm = 1;
    L.concurrent_warps = L.bs / 32;
    L.grid = di.sm_count;
    L.rows_per_vector = (a.m + (int64_t)L.grid * 32 - 1) / ((int64_t)L.grid * 32);
    *out = L;
    return FP_OK;
  }
  CsrKFn f = pick_any(a, L);
  FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_csr: no kernel for vs=%d", L.vs);
  set_max_dynamic_smem((const void*)f);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, f, L.bs, L.smem_bytes);
  if (per_sm < 1) per_sm = 1;
  cudaFuncAttributes fa{};
  cudaFuncGetAttributes(&fa, f);
  L.regs_per_thread = fa.numRegs;
  L.blocks_per_sm = per_sm;
  L.concurrent_warps = per_sm * L.bs / 32;
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

namespace {
int ym_of(const PatternArgs& a) { return !a.y ? 0 : ((a.epi_kind == 0 && !a.row_out) ? 1 : 2); }

SplitKFn pick_split(const PatternArgs& a, int cs, int nb) {
  return a.dtype == FP_F64 ? csr_pick_colsplit_f64(ym_of(a), cs, nb) : csr_pick_colsplit_f32(ym_of(a), cs, nb);
}

// register tiles per warp batch: 16 when the mean block segment of a 32-row batch exceeds 8 tiles
int split_nb(const PatternArgs& a, int cs) {
  const double seg = a.m > 0 ? 32.0 * (double)a.nnz / (double)a.m / cs : 0.0;
  return seg > 0.8 * 8 * 32 ? 16 : 8;
}

cudaLaunchConfig_t split_config(const PatternArgs& a, const CsrSplit& sp, int grid, cudaLaunchAttribute* attr,
                                cudaStream_t s) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3((unsigned)kSplitBS);
  cfg.dynamicSmemBytes = colsplit_smem(a.dtype, sp.cs, sp.width, a.y != nullptr);
  cfg.stream = s;
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)sp.cs;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cfg;
}

// co-resident clusters of the split kernel (0 if it does not fit)
int split_capacity(const PatternArgs& a, const CsrSplit& sp, int nb) {
  SplitKFn f = pick_split(a, sp.cs, nb);
  if (!f) return 0;
  const size_t smem = colsplit_smem(a.dtype, sp.cs, sp.width, a.y != nullptr);
  if (smem > 227 * 1024) return 0;
  set_max_dynamic_smem((const void*)f);
  cudaLaunchAttribute attr[1];
  cudaLaunchConfig_t cfg = split_config(a, sp, sp.cs * 64, attr, 0);
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, (const void*)f, &cfg) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}
}  // namespace

// Column-split plan (FP_VAR_CSR_COLSPLIT): the smallest cluster (2, 4, 8 CTAs, one per SM)
// whose column blocks of y and w fit one CTA's shared memory; equal-width column blocks.
bool plan_colsplit(const PatternArgs& a, int device, int cs_force, CsrSplit* sp, fp_launch* L) {
  (void)device;
  if (a.n < 2 || a.n > INT32_MAX) return false;
  for (int cs = 2; cs <= kSplitMaxCS; cs *= 2) {
    if (cs_force && cs != cs_force) continue;
    CsrSplit t;
    t.cs = cs;
    for (int k = 0; k <= cs; ++k) t.cb[k] = (int)((a.n * k) / cs);
    t.width = 0;
    for (int k = 0; k < cs; ++k) t.width = std::max(t.width, t.cb[k + 1] - t.cb[k]);
    if (colsplit_smem(a.dtype, cs, t.width, a.y != nullptr) > 227 * 1024) continue;
    const int nb = split_nb(a, cs);
    const int nc = split_capacity(a, t, nb);
    if (nc < 1) continue;
    *sp = t;
    fp_launch o{};
    o.variant = FP_VAR_CSR_COLSPLIT;
    o.vs = 32;
    o.bs = kSplitBS;
    o.tl = nb;
    o.cluster = cs;
    o.grid = nc * cs;
    o.blocks_per_sm = 1;
    o.concurrent_warps = kSplitBS / 32;
    o.smem_bytes = (int)colsplit_smem(a.dtype, cs, t.width, a.y != nullptr);
    cudaFuncAttributes fa{};
    if (cudaFuncGetAttributes(&fa, (const void*)pick_split(a, cs, nb)) == cudaSuccess) o.regs_per_thread = fa.numRegs;
    const int64_t vectors = (int64_t)o.grid / cs * (kSplitBS / 32);
    o.rows_per_vector = vectors > 0 ? (a.m + vectors - 1) / vectors : 0;
    *L = o;
    return true;
  }
  return false;
}

// The stream variants copy colidx / val in 16-byte chunks and have no row epilogue; otherwise
// the same (VS, K) runs as plain CSR-vector with the same partial (identical arithmetic).
fp_launch stream_fallback(const PatternArgs& a, const fp_launch& L) {
  fp_launch o = L;
  if (L.variant == FP_VAR_CSR_FLAT4_FIXED) {
    // the chooser picks variant 18 without seeing val: colidx / val aligned differently (or a
    // row epilogue) run the paper's CSR-vector with the CTA-shared partial instead
    const size_t es = dtype_size(a.dtype);
    const bool alike = ((uintptr_t)a.colidx % 4 == 0) && ((uintptr_t)a.val % es == 0) &&
                       (((uintptr_t)a.colidx / 4) % 4 == ((uintptr_t)a.val / es) % 4);
    const bool epi = a.y && !(a.epi_kind == 0 && !a.row_out);
    if (!alike || epi) {
      o.variant = FP_VAR_CSR_VECTOR;
      o.vs = 4;
      o.tl = 4;
      o.grid = 0;
    }
    return o;
  }
  if (L.variant != FP_VAR_CSR_STREAM && L.variant != FP_VAR_CSR_STREAM_FIXED) return o;
  const bool aligned = ((uintptr_t)a.colidx % 16 == 0) && ((uintptr_t)a.val % 16 == 0);
  const bool epi = a.y && !(a.epi_kind == 0 && !a.row_out);
  if (!aligned || epi) o.variant = L.variant == FP_VAR_CSR_STREAM ? FP_VAR_CSR_VECTOR : FP_VAR_CSR_VECTOR_FIXED;
  return o;
}

fp_status launch_csr(const PatternArgs& a, const fp_launch& L_in, cudaStream_t s) {
  const fp_launch L = stream_fallback(a, L_in);
  if (L.variant == FP_VAR_CSR_BINNED) return launch_binned(a, L, wide_y_entries(a), s);
  if (L.variant == FP_VAR_CSR_FLAT4_FIXED) return launch_flat4_fixed(a, L, s);
  if (L.variant == FP_VAR_CSR_COLSPLIT) {
    FP_REQUIRE(a.split && a.split->soff && a.split->cs == L.cluster, FP_ERR_UNSUPPORTED,
               "fp_csr: variant %d (column split) runs from a CSR plan (fp_csr_plan_create)", L.variant);
    const CsrSplit& sp = *a.split;
    SplitKFn f = pick_split(a, sp.cs, L.tl);
    FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_csr: no column-split kernel for cluster %d, %d tiles", sp.cs, L.tl);
    FP_REQUIRE(L.grid >= sp.cs && L.grid % sp.cs == 0, FP_ERR_INVALID_ARG, "fp_csr: split grid must be k x %d",
               sp.cs);
    Workspace* ws = workspace(s, (size_t)a.n, 0);
    if (!ws) return FP_ERR_NOMEM;
    SplitKArgs k{};
    k.k = CsrKArgs{a.m, a.n, a.nnz, a.rowptr, a.colidx, a.val, a.y, a.v, a.z, a.alpha, a.beta, a.w,
                   ws->acc, ws->counters, a.add_beta_z ? 1 : 0, a.accumulate ? 1 : 0, 0,
                   {a.epi_kind, a.epi_c, a.row_out, a.scalar_out}, 0};
    k.soff = sp.soff;
    for (int i = 0; i <= kSplitMaxCS; ++i) k.cb[i] = sp.cb[i];
    k.width = sp.width;
    const size_t smem = colsplit_smem(a.dtype, sp.cs, sp.width, a.y != nullptr);
    set_max_dynamic_smem((const void*)f);
    cudaLaunchAttribute attr[1];
    cudaLaunchConfig_t cfg = split_config(a, sp, L.grid, attr, s);
    FP_CUDA(cudaLaunchKernelEx(&cfg, f, k));
    return FP_OK;
  }
  CsrKFn f = pick_any(a, L);
  FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_csr: launch plan (variant=%d vs=%d) has no kernel", L.variant, L.vs);
  const int bs_need = L.variant == FP_VAR_CSR_FLAT_L2_WIDE ? kWideBS : kCsrBS;
  FP_REQUIRE(L.bs == bs_need, FP_ERR_UNSUPPORTED, "fp_csr: block size %d not supported (variant %d runs %d)", L.bs,
             L.variant, bs_need);
  FP_REQUIRE(L.grid >= 0, FP_ERR_INVALID_ARG, "fp_csr: grid must be >= 0 (0 = one resident wave)");
  const bool l2 = L.variant == FP_VAR_CSR_VECTOR_L2 || L.variant == FP_VAR_CSR_FLAT_L2 ||
                  L.variant == FP_VAR_CSR_FLAT_L2_WIDE;
  const size_t smem = smem_for(a, L.variant);
  FP_REQUIRE(smem <= 227 * 1024, FP_ERR_UNSUPPORTED, "fp_csr: variant %d needs %zu B shared memory (n too large)",
             L.variant, smem);
  // L2 path: number of copies of w the CTAs spread their reds over (copies 1.. live in the
  // all-zero workspace accumulator and are folded into w after the kernel)
  // copies of w for the L2 reds: the chooser's rule, or an explicit plan's cluster field (1..16;
  // the sweep varies it -- fp_launch.cluster is otherwise unused by the L2 variants)
  const int nrep = !l2 ? 1 : (L.cluster > 0 ? std::min(L.cluster, 16) : l2_replicas(a));
  const size_t rep_doubles = nrep > 1 ? ((size_t)(nrep - 1) * a.n * dtype_size(a.dtype) + 7) / 8 : 0;
  Workspace* ws = workspace(s, l2 ? rep_doubles : (size_t)a.n, 0);
  if (!ws) return FP_ERR_NOMEM;
  if (l2 && !a.accumulate) {  // L2 path: w <- beta z (or 0) first, the kernel reduces alpha X^T q into it
    fp_status st = launch_scale_z(a.n, a.add_beta_z ? a.z : nullptr, a.add_beta_z ? a.beta : 0.0, a.w, a.dtype, s);
    if (st != FP_OK) return st;
  }
  CsrKArgs k{a.m, a.n, a.nnz, a.rowptr, a.colidx, a.val, a.y, a.v, a.z, a.alpha, a.beta, a.w,
             ws->acc, ws->counters, a.add_beta_z ? 1 : 0, a.accumulate ? 1 : 0, l2 ? l2_y_entries(a, L.variant) : 0,
             {a.epi_kind, a.epi_c, a.row_out, a.scalar_out}, phase_iters_for(a, L), ws->acc, nrep};
  set_max_dynamic_smem((const void*)f);
  // L2 path without y in shared memory: prefer the largest L1 so the random y gathers hit it
  // (X itself streams with L1::no_allocate and never displaces y)
  if (l2 && smem == 0) cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, 0);
  int grid = L.grid;
  if (grid == 0) {  // one full resident wave: SMs x occupancy of this kernel
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, f, L.bs, (int)smem);
    grid = device_info(current_device()).sm_count * (per_sm > 0 ? per_sm : 1);
  }
  f<<<grid, L.bs, smem, s>>>(k);
  FP_CUDA(cudaGetLastError());
  if (nrep > 1) {
    const int fb = 256;
    const int fg = (int)std::min<int64_t>((a.n + fb - 1) / fb, 4 * device_info(current_device()).sm_count);
    if (a.dtype == FP_F64)
      k_fold_replicas<double><<<fg, fb, 0, s>>>((double*)a.w, (double*)ws->acc, a.n, nrep - 1);
    else
      k_fold_replicas<float><<<fg, fb, 0, s>>>((float*)a.w, (float*)ws->acc, a.n, nrep - 1);
    FP_CUDA(cudaGetLastError());
  }
  return FP_OK;
}

}  // namespace fp
