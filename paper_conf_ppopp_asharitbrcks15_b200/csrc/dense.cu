// dense.cu -- B200 plan and launch of the fused dense kernels (dense_kernels.cuh), and the
// beta*z / zero-fill kernel shared by the alpha == 0 path and the CSR L2 path.
#include <stdlib.h>

#include <algorithm>

#include "dense_kernels.cuh"

namespace fp {

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

namespace {

// bytes per load the alignment of X and of the row stride allows
int chunk_bytes_for(const PatternArgs& a) {
  const int64_t s = (int64_t)dtype_size(a.dtype);
  const uintptr_t x = (uintptr_t)a.X;
  if (x % 32 == 0 && (a.ld * s) % 32 == 0) return 32;
  if (x % 16 == 0 && (a.ld * s) % 16 == 0) return 16;
  return (int)s;
}

// Bulk-copy (TMA) ring for the cluster kernel: on unless FP_CLUSTER_TMA=0 (A/B measurement).
bool cluster_tma_enabled() {
  static const bool on = [] {
    const char* e = getenv("FP_CLUSTER_TMA");
    return !(e && e[0] == '0');
  }();
  return on;
}

// The cluster plan runs the bulk-copy ring kernel for 16/32-byte-aligned rows and thread slices
// of at most 128 bytes; 256-byte slices (rows up to 2x wider) and unaligned rows run the
// register kernel.
bool uses_tma(const PatternArgs& a, const fp_launch& L, int cb) {
  return L.variant == FP_VAR_DENSE_CLUSTER && cb >= 16 && cluster_tma_enabled() &&
         L.tl * (int)dtype_size(a.dtype) <= 128;
}

// Ring depth of the TMA cluster kernel: 3 slices (two rows in flight beyond the one being
// consumed; 3 x 32 KB -> two CTAs per SM).  FP_CLUSTER_RING=2..8 overrides (measurement),
// clamped to the 227 KB opt-in limit.
int cluster_ring_depth(const PatternArgs& a, const fp_launch& L) {
  const int slice = L.tl * (int)dtype_size(a.dtype) * L.bs;
  int d = 3;
  static const int env = [] {
    const char* e = getenv("FP_CLUSTER_RING");
    return e ? atoi(e) : 0;
  }();
  if (env >= 2 && env <= 8) d = env;
  while (d > 2 && d * slice > 220 * 1024) --d;
  return d;
}

// dynamic shared memory of a plan: the fp64 w row (vector/CTA kernels), the D-row ring of the
// TMA cluster kernel (D x TL elements x BS threads), 0 for the register-only cluster kernel
int dense_smem_bytes(const PatternArgs& a, const fp_launch& L) {
  const int cb = chunk_bytes_for(a);
  if (L.variant != FP_VAR_DENSE_CLUSTER) return (int)(a.n * sizeof(double));
  if (!uses_tma(a, L, cb)) return 0;
  return cluster_ring_depth(a, L) * L.tl * (int)dtype_size(a.dtype) * L.bs;
}

DenseKFn pick_any(const PatternArgs& a, const fp_launch& L) {
  const int cb = chunk_bytes_for(a);
  const int ce = cb / (int)dtype_size(a.dtype);
  if (L.tl <= 0 || L.tl % ce != 0) return nullptr;
  const int nch = L.tl / ce;
  // 0: no y (Table 1 row 1); 1: Eq. (1) fast path; 2: Eq. (1) + row epilogue (outputs / logistic)
  const int ym = !a.y ? 0 : ((a.epi_kind == 0 && !a.row_out) ? 1 : 2);
  const int tma = uses_tma(a, L, cb) ? 1 : 0;
  return a.dtype == FP_F64 ? dense_pick_f64(ym, L.variant, cb, L.vs, nch, tma)
                           : dense_pick_f32(ym, L.variant, cb, L.vs, nch, tma);
}


// Clusters of plan C that can be co-resident on the device (0 if the kernel is missing or the
// query fails).
int cluster_capacity(const PatternArgs& a, const fp_launch& C) {
  DenseKFn f = pick_any(a, C);
  if (!f) return 0;
  const int dsm = dense_smem_bytes(a, C);
  if (dsm > (int)device_info(current_device()).smem_optin_per_block) return 0;
  set_max_dynamic_smem((const void*)f);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3((unsigned)(C.cluster * 64));
  cfg.blockDim = dim3((unsigned)C.bs);
  cfg.dynamicSmemBytes = (size_t)dsm;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)C.cluster;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, (const void*)f, &cfg) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}

int round_up_in(int need, const int* set, int cnt) {
  for (int i = 0; i < cnt; ++i)
    if (set[i] >= need) return set[i];
  return -1;
}

}  // namespace

// B200 dense plan.  chunks/row = ceil(n / E) with E the elements of one (32/16-byte or
// scalar) load.  Up to 32 chunks: one chunk per lane, VS = next power of two >= chunks --
// Eq. (6) with TL = E.  Beyond: VS = 32 and NCH chunks per lane (TL = NCH*E, at most
// 256 bytes per thread -- the register budget that replaces the paper's TL <= 40).
// Beyond that: the CTA variant, VS = BS (Eq. 6 first case).  grid = SMs x resident CTAs
// (persistent, each vector strides over rows: Alg. 3 l.25 with C = rows / vectors).
fp_status plan_dense(const PatternArgs& a, int device, fp_launch* out) {
  const DeviceInfo& di = device_info(device);
  const int s = (int)dtype_size(a.dtype);
  const int cb = chunk_bytes_for(a);
  const int ce = cb / s;
  const int64_t chunks = (a.n + ce - 1) / ce;
  static const int vec_set[] = {1, 2, 3, 4, 6, 8, 12, 16, 32, 64};
  static const int cta_set[] = {1, 2, 4, 8, 16, 32, 64};
  fp_launch L{};
  if (chunks <= 32) {
    int vs = 1;
    while (vs < chunks) vs <<= 1;
    L.variant = FP_VAR_DENSE_VECTOR;
    L.vs = vs;
    L.tl = ce;
    L.bs = kBS;
  } else {
    int nch = round_up_in((int)((chunks + 31) / 32), vec_set, 10);
    if (nch > 0 && nch * cb <= 256) {
      L.variant = FP_VAR_DENSE_VECTOR;
      L.vs = 32;
      L.tl = nch * ce;
      L.bs = kBS;
    } else {
      nch = round_up_in((int)((chunks + kBSCta - 1) / kBSCta), cta_set, 7);
      if (nch > 0 && nch * cb <= 256) {
        L.variant = FP_VAR_DENSE_CTA;
        L.vs = kBSCta;
        L.tl = nch * ce;
        L.bs = kBSCta;
      } else {
        // a cluster of CS CTAs (BS = 256 each) shares the row (VS = CS x BS).  Candidates in
        // preference order, each with the smallest CS in {2,4,8} covering n: bulk-copy ring
        // kernel with 128- / 64-byte thread slices (16-byte-aligned rows), register kernel with
        // 256-byte, then (rows not aligned, or ring disabled) 128-byte slices.  The one keeping
        // the most SMs streaming wins (co-resident clusters x CS / CTAs per SM, occupancy API:
        // an 8-CTA cluster must fit one GPC, so only 15 fit 148 SMs at one CTA per SM); ties
        // keep the earlier.
        const bool ring = cb >= 16 && cluster_tma_enabled();
        struct Cand { int tb; };
        Cand cands[4];
        int nc = 0;
        if (ring) {
          cands[nc++] = {128};
          cands[nc++] = {64};
          cands[nc++] = {256};
        } else {
          cands[nc++] = {256};
          cands[nc++] = {128};
        }
        int best_sms = -1;
        static const int force_tb = [] {  // FP_CLUSTER_TB=<bytes per thread>: pin (measurement)
          const char* e = getenv("FP_CLUSTER_TB");
          return e ? atoi(e) : 0;
        }();
        for (int ci = 0; ci < nc; ++ci) {
          const int tb = cands[ci].tb;
          if (force_tb && tb != force_tb) continue;
          const int64_t per_cta = (int64_t)kBSCta * (tb / s);
          int cs = 2;
          while (cs < 8 && (int64_t)cs * per_cta < a.n) cs <<= 1;
          if ((int64_t)cs * per_cta < a.n) continue;
          fp_launch C{};
          C.variant = FP_VAR_DENSE_CLUSTER;
          C.vs = cs * kBSCta;
          C.tl = tb / s;
          C.bs = kBSCta;
          C.cluster = cs;
          const int clusters = cluster_capacity(a, C);
          DenseKFn fc = pick_any(a, C);
          int bps = 1;
          if (fc) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, fc, C.bs, dense_smem_bytes(a, C));
          if (bps < 1) bps = 1;
          const int sms = std::min((clusters * cs + bps - 1) / bps, di.sm_count);  // SMs streaming
          if (clusters > 0 && sms > best_sms) {
            best_sms = sms;
            L = C;
          }
        }
        if (L.variant != FP_VAR_DENSE_CLUSTER) {
          const int64_t per_cta = (int64_t)kBSCta * (256 / s);
          set_error("fp_dense: n=%lld exceeds the cluster-resident row limit (%lld elements = 8 CTAs x %d "
                    "threads x 256 B); wider dense rows are not implemented (DESIGN.md NEXT-4)",
                    (long long)a.n, (long long)(8 * per_cta), kBSCta);
          return FP_ERR_UNSUPPORTED;
        }
      }
    }
  }
  DenseKFn f = pick_any(a, L);
  if (!f) {
    set_error("fp_dense: no kernel instantiation for vs=%d tl=%d (chunk %d B)", L.vs, L.tl, cb);
    return FP_ERR_UNSUPPORTED;
  }
  const bool clu = L.variant == FP_VAR_DENSE_CLUSTER;
  L.smem_bytes = dense_smem_bytes(a, L);
  set_max_dynamic_smem((const void*)f);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, f, L.bs, L.smem_bytes);
  if (per_sm < 1) per_sm = 1;
  cudaFuncAttributes fa{};
  cudaFuncGetAttributes(&fa, f);
  L.regs_per_thread = fa.numRegs;
  L.blocks_per_sm = per_sm;
  L.concurrent_warps = per_sm * L.bs / 32;
  const int64_t vectors_per_cta = (L.variant == FP_VAR_DENSE_CTA || clu) ? 1 : L.bs / L.vs;
  // rows a CTA consumes per iteration: vectors x RPV (rows in flight per vector)
  const int64_t rpv = (L.variant == FP_VAR_DENSE_CTA || clu) ? 1 : rpv_for(L.tl / (cb / s), cb);
  int64_t need_ctas = (a.m + vectors_per_cta * rpv - 1) / (vectors_per_cta * rpv);
  if (clu) need_ctas = a.m * L.cluster;  // a cluster of CS CTAs per row
  int64_t grid = (int64_t)di.sm_count * per_sm;
  if (need_ctas < grid) grid = need_ctas > 0 ? need_ctas : 1;
  if (clu) {  // co-resident clusters only: a second wave would double the time of the first
    int64_t nc = cluster_capacity(a, L);
    if (nc < 1) nc = 1;
    if (nc > a.m) nc = a.m > 0 ? a.m : 1;
    grid = nc * L.cluster;
  }
  L.grid = (int)grid;
  L.rows_per_vector = (a.m + grid * vectors_per_cta - 1) / (grid * vectors_per_cta);
  *out = L;
  return FP_OK;
}

int dense_kernel_regs(const PatternArgs& a, const fp_launch& L) {
  DenseKFn f = pick_any(a, L);
  if (!f) return 0;
  cudaFuncAttributes fa{};
  if (cudaFuncGetAttributes(&fa, f) != cudaSuccess) return 0;
  return fa.numRegs;
}

fp_status launch_dense(const PatternArgs& a, const fp_launch& L, cudaStream_t s) {
  DenseKFn f = pick_any(a, L);
  FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_dense: launch plan (variant=%d vs=%d tl=%d) has no kernel", L.variant, L.vs,
             L.tl);
  const bool clu = L.variant == FP_VAR_DENSE_CLUSTER;
  const int want_bs = (clu || L.variant == FP_VAR_DENSE_CTA) ? kBSCta : kBS;
  FP_REQUIRE(L.bs == want_bs, FP_ERR_UNSUPPORTED,
             "fp_dense: block size %d not supported by the selected kernel", L.bs);
  FP_REQUIRE(L.grid >= 1, FP_ERR_INVALID_ARG, "fp_dense: grid must be >= 1");
  const int cs = clu ? L.vs / L.bs : 1;
  FP_REQUIRE(!clu || ((cs == 2 || cs == 4 || cs == 8) && L.vs == cs * L.bs), FP_ERR_INVALID_ARG,
             "fp_dense: cluster plan needs vs = CS x bs with CS in {2,4,8}");
  FP_REQUIRE(!clu || (L.grid % cs == 0), FP_ERR_INVALID_ARG, "fp_dense: grid must be a multiple of the cluster size");
  Workspace* ws = workspace(s, (size_t)a.n, 0);
  if (!ws) return FP_ERR_NOMEM;
  DenseKArgs k{a.m, a.n, a.ld, a.X, a.y, a.v, a.z, a.alpha, a.beta, a.w, ws->acc, ws->counters, a.add_beta_z ? 1 : 0,
               a.accumulate ? 1 : 0, {a.epi_kind, a.epi_c, a.row_out, a.scalar_out}};
  if (clu) {  // thread-block cluster launch: CS CTAs share one row through DSMEM
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)L.grid);
    cfg.blockDim = dim3((unsigned)L.bs);
    const int dsm = dense_smem_bytes(a, L);
    set_max_dynamic_smem((const void*)f);
    cfg.dynamicSmemBytes = (size_t)dsm;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)cs;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    FP_CUDA(cudaLaunchKernelEx(&cfg, f, k));
    return FP_OK;
  }
  const size_t smem = (size_t)a.n * sizeof(double);
  set_max_dynamic_smem((const void*)f);
  f<<<L.grid, L.bs, smem, s>>>(k);
  FP_CUDA(cudaGetLastError());
  return FP_OK;
}

}  // namespace fp
