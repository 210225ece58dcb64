// dense.cu -- B200 plan and launch of the fused dense kernels (dense_kernels.cuh), and the
// beta*z / zero-fill kernel shared by the alpha == 0 path and the CSR L2 path.
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

DenseKFn pick_any(const PatternArgs& a, const fp_launch& L) {
  const int cb = chunk_bytes_for(a);
  const int ce = cb / (int)dtype_size(a.dtype);
  if (L.tl <= 0 || L.tl % ce != 0) return nullptr;
  const int nch = L.tl / ce;
  // 0: no y (Table 1 row 1); 1: Eq. (1) fast path; 2: Eq. (1) + row epilogue (outputs / logistic)
  const int ym = !a.y ? 0 : ((a.epi_kind == 0 && !a.row_out) ? 1 : 2);
  return a.dtype == FP_F64 ? dense_pick_f64(ym, L.variant, cb, L.vs, nch) : dense_pick_f32(ym, L.variant, cb, L.vs, nch);
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
        // a cluster of CS CTAs shares the row (VS = CS x BS); 128-byte thread load when 8 CTAs
        // cover the row with it (two resident CTAs per SM), else the full 256-byte load
        const int64_t half_cta = (int64_t)kBSCta * (128 / s);
        if ((int64_t)8 * half_cta >= a.n) {
          int cs = 2;
          while (cs < 8 && (int64_t)cs * half_cta < a.n) cs <<= 1;
          L.variant = FP_VAR_DENSE_CLUSTER;
          L.vs = cs * kBSCta;
          L.tl = 128 / s;
          L.bs = kBSCta;
          L.cluster = cs;
        }
        if (L.variant != FP_VAR_DENSE_CLUSTER) {
          const int64_t per_cta = (int64_t)kBSCta * (256 / s);  // elements of a row per CTA
          int cs = 2;
          while (cs < 8 && (int64_t)cs * per_cta < a.n) cs <<= 1;
          if ((int64_t)cs * per_cta < a.n) {
            set_error("fp_dense: n=%lld exceeds the cluster-resident row limit (%lld elements = 8 CTAs x %d "
                      "threads x 256 B); wider dense rows are not implemented (DESIGN.md NEXT-4)",
                      (long long)a.n, (long long)(8 * per_cta), kBSCta);
            return FP_ERR_UNSUPPORTED;
          }
          L.variant = FP_VAR_DENSE_CLUSTER;
          L.vs = cs * kBSCta;
          L.tl = 256 / s;
          L.bs = kBSCta;
          L.cluster = cs;
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
  L.smem_bytes = clu ? 0 : (int)(a.n * sizeof(double));
  if (L.smem_bytes > 48 * 1024) cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, L.smem_bytes);
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
  if (clu) grid = (grid / L.cluster > 0 ? grid / L.cluster : 1) * L.cluster;
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
  FP_REQUIRE(L.bs == ((L.variant == FP_VAR_DENSE_CTA || clu) ? kBSCta : kBS), FP_ERR_UNSUPPORTED,
             "fp_dense: block size %d not supported by the selected kernel", L.bs);
  FP_REQUIRE(L.grid >= 1, FP_ERR_INVALID_ARG, "fp_dense: grid must be >= 1");
  const int cs = clu ? L.vs / kBSCta : 1;
  FP_REQUIRE(!clu || (L.grid % cs == 0), FP_ERR_INVALID_ARG, "fp_dense: grid must be a multiple of the cluster size");
  Workspace* ws = workspace(s, (size_t)a.n, 0);
  if (!ws) return FP_ERR_NOMEM;
  DenseKArgs k{a.m, a.n, a.ld, a.X, a.y, a.v, a.z, a.alpha, a.beta, a.w, ws->acc, ws->counters, a.add_beta_z ? 1 : 0,
               a.accumulate ? 1 : 0, {a.epi_kind, a.epi_c, a.row_out, a.scalar_out}};
  if (clu) {  // thread-block cluster launch: CS CTAs share one row through DSMEM
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)L.grid);
    cfg.blockDim = dim3((unsigned)L.bs);
    cfg.dynamicSmemBytes = 0;
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
  if (smem > 48 * 1024) FP_CUDA(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  f<<<L.grid, L.bs, smem, s>>>(k);
  FP_CUDA(cudaGetLastError());
  return FP_OK;
}

}  // namespace fp
