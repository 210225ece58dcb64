// plan.cu -- launch-parameter chooser (Section 3.3) and row statistics.
//
// fp_choose_paper: the paper's analytical model written out as stated (Eq. 4, the
//   occupancy rule of P:377-388, Eq. 5, the dense TL/VS rule with the wasted-warp
//   refinement of P:396-403 and Eq. 6), parameterised by a device profile so that its worked
//   example (Kepler GK110: VS=8, BS=640, 28 blocks, 8,832 B smem, 223 rows/vector)
//   can be reproduced exactly (tests/golden/chooser_p457.json).
// fp_choose: what the B200 kernels actually launch (dense.cu plan_dense, csr.cu plan_csr):
//   same inputs, real register counts from cudaFuncGetAttributes and the CUDA occupancy API.
#include <math.h>
#include <string.h>

#include "kernels.cuh"

namespace fp {
int eq4_vector_size(double mu);  // csr.cu
}

namespace {

int ceil_div(int a, int b) { return (a + b - 1) / b; }
int round_up(int a, int b) { return ceil_div(a, b) * b; }

// Concurrent blocks per SM for one block shape (the NVIDIA occupancy-calculator rules the
// paper cites, P:388 [30]): limited by threads, blocks, registers (allocated per warp in
// reg_alloc_unit chunks, warps rounded to warp_alloc_granularity) and shared memory
// (smem_alloc_unit chunks).
int blocks_per_sm(const fp_device_profile& p, int bs, int regs_per_thread, int smem_bytes) {
  if (bs <= 0 || bs > p.max_threads_per_block) return 0;
  if (regs_per_thread > p.max_regs_per_thread) return 0;
  if (smem_bytes > p.smem_per_block) return 0;
  int by_threads = p.max_threads_per_sm / bs;
  int by_blocks = p.max_blocks_per_sm;
  int warps = ceil_div(bs, p.warp_size);
  int warps_alloc = round_up(warps, p.warp_alloc_granularity);
  int regs_per_warp = round_up(regs_per_thread * p.warp_size, p.reg_alloc_unit);
  int by_regs = regs_per_thread > 0 ? p.regs_per_sm / (regs_per_warp * warps_alloc) : by_blocks;
  int smem_alloc = smem_bytes > 0 ? round_up(smem_bytes, p.smem_alloc_unit) : 0;
  int by_smem = smem_alloc > 0 ? p.smem_per_sm / smem_alloc : by_blocks;
  int b = by_threads;
  if (by_blocks < b) b = by_blocks;
  if (by_regs < b) b = by_regs;
  if (by_smem < b) b = by_smem;
  return b;
}

// Eq. (6): VS = BS if n/TL > 32; 2^i if 2^i >= n/TL > 2^(i-1), i in 1..5; else 1.
int eq6_vector_size(int64_t n, int tl, int bs) {
  double r = (double)n / (double)tl;
  if (r > 32) return bs;
  for (int i = 1; i <= 5; ++i)
    if ((double)(1 << i) >= r && r > (double)(1 << (i - 1))) return 1 << i;
  return 1;
}

}  // namespace

extern "C" {

fp_status fp_device_profile_kepler(fp_device_profile* out) {
  FP_REQUIRE(out, FP_ERR_INVALID_ARG, "fp_device_profile_kepler: out is NULL");
  // (64K registers, 48KB), (1,024 and 2,048 threads), (8 blocks), (256 registers and
  // 4 warps allocation granularity), (255 registers/thread), (256 B smem allocation unit);
  // 14 SMs (GTX Titan).
  fp_device_profile p{};
  p.sm_count = 14;
  p.max_threads_per_sm = 2048;
  p.max_threads_per_block = 1024;
  p.max_blocks_per_sm = 8;
  p.regs_per_sm = 65536;
  p.max_regs_per_thread = 255;
  p.reg_alloc_unit = 256;
  p.warp_alloc_granularity = 4;
  p.smem_per_sm = 48 * 1024;
  p.smem_per_block = 48 * 1024;
  p.smem_alloc_unit = 256;
  p.warp_size = 32;
  *out = p;
  return FP_OK;
}

fp_status fp_device_profile_query(int device, fp_device_profile* out) {
  FP_REQUIRE(out, FP_ERR_INVALID_ARG, "fp_device_profile_query: out is NULL");
  cudaDeviceProp pr{};
  FP_CUDA(cudaGetDeviceProperties(&pr, device));
  fp_device_profile p{};
  p.sm_count = pr.multiProcessorCount;
  p.max_threads_per_sm = pr.maxThreadsPerMultiProcessor;
  p.max_threads_per_block = pr.maxThreadsPerBlock;
  p.max_blocks_per_sm = pr.maxBlocksPerMultiProcessor;
  p.regs_per_sm = pr.regsPerMultiprocessor;
  p.max_regs_per_thread = 255;
  p.reg_alloc_unit = 256;
  p.warp_alloc_granularity = 4;
  p.smem_per_sm = (int)pr.sharedMemPerMultiprocessor;
  p.smem_per_block = (int)pr.sharedMemPerBlockOptin;
  p.smem_alloc_unit = 128;
  p.warp_size = pr.warpSize;
  *out = p;
  return FP_OK;
}

fp_status fp_row_stats_dense(int64_t m, int64_t n, fp_row_stats* out) {
  FP_REQUIRE(out && m >= 0 && n >= 0, FP_ERR_INVALID_ARG, "fp_row_stats_dense: bad arguments");
  memset(out, 0, sizeof(*out));
  out->m = m;
  out->n = n;
  out->nnz = m * n;
  out->mean = (double)n;
  out->max_len = m > 0 ? n : 0;
  out->min_len = m > 0 ? n : 0;
  out->empty_rows = n == 0 ? m : 0;
  int b = 0;
  while (b < 63 && ((int64_t)1 << b) <= n) ++b;
  if (m > 0) out->hist_log2[n == 0 ? 0 : b] = m;
  return FP_OK;
}

static inline int len_bin(int64_t L) {
  if (L <= 0) return 0;
  int b = 0;
  while (b < 63 && ((int64_t)1 << b) <= L) ++b;
  return b;  // L in [2^(b-1), 2^b)
}

fp_status fp_row_stats_host(int64_t m, const int64_t* rowptr, fp_row_stats* out) {
  FP_REQUIRE(out && m >= 0 && (m == 0 || rowptr), FP_ERR_INVALID_ARG, "fp_row_stats_host: bad arguments");
  memset(out, 0, sizeof(*out));
  out->m = m;
  out->n = -1;
  out->min_len = m > 0 ? INT64_MAX : 0;
  for (int64_t r = 0; r < m; ++r) {
    int64_t L = rowptr[r + 1] - rowptr[r];
    FP_REQUIRE(L >= 0, FP_ERR_INVALID_CSR, "fp_row_stats_host: rowptr decreases at row %lld", (long long)r);
    if (L > out->max_len) out->max_len = L;
    if (L < out->min_len) out->min_len = L;
    if (L == 0) out->empty_rows++;
    out->hist_log2[len_bin(L)]++;
  }
  out->nnz = m > 0 ? rowptr[m] - rowptr[0] : 0;
  out->mean = m > 0 ? (double)out->nnz / (double)m : 0.0;
  return FP_OK;
}

fp_status fp_choose_paper(int is_csr, const fp_row_stats* st, fp_dtype dtype, const fp_device_profile* prof,
                          int regs_per_thread, int regs_dense_tl1, int regs_dense_tl40, fp_launch* out) {
  FP_REQUIRE(st && prof && out, FP_ERR_INVALID_ARG, "fp_choose_paper: NULL argument");
  FP_REQUIRE(fp::valid_dtype(dtype), FP_ERR_INVALID_ARG, "fp_choose_paper: bad dtype");
  const fp_device_profile& p = *prof;
  const int s = (int)fp::dtype_size(dtype);
  fp_launch L{};
  if (is_csr) {
    // Eq. (4): VS from mu = NNZ / m
    L.variant = FP_VAR_CSR_VECTOR;
    L.vs = fp::eq4_vector_size(st->mean);
    // BS from {1x32 .. 32x32} maximising concurrent warps NW, smem (BS/VS + n)*s;
    // ties go to the largest BS ("increase ... the block size to their maximum")
    int best_nw = -1;
    for (int bs = p.warp_size; bs <= 32 * p.warp_size; bs += p.warp_size) {
      if (bs % L.vs != 0) continue;
      int smem = (int)((bs / L.vs + st->n) * s);
      int b = blocks_per_sm(p, bs, regs_per_thread, smem);
      int nw = b * bs / p.warp_size;
      if (b > 0 && nw >= best_nw) {
        best_nw = nw;
        L.bs = bs;
        L.blocks_per_sm = b;
        L.smem_bytes = smem;
      }
    }
    FP_REQUIRE(best_nw > 0, FP_ERR_UNSUPPORTED, "fp_choose_paper: no block size fits (n too large for smem)");
    L.concurrent_warps = best_nw;
    L.regs_per_thread = regs_per_thread;
    L.tl = 0;
  } else {
    // Dense: BS = 128 (register-allocation multiple, minimal sync), TL in 1..40
    // with registers interpolated between the two profiled points, maximise
    // concurrent warps excluding wasted warp-loads per vector; VS by Eq. (6).
    if (st->n <= 32) {  // exception
      L.bs = 1024;
      L.tl = 1;
      L.vs = eq6_vector_size(st->n, 1, L.bs);
      L.regs_per_thread = regs_dense_tl1;
      L.blocks_per_sm = blocks_per_sm(p, L.bs, L.regs_per_thread, 0);
      L.concurrent_warps = L.blocks_per_sm * L.bs / p.warp_size;
    } else {
      L.bs = 128;
      double best = -1.0;
      for (int tl = 1; tl <= 40; ++tl) {
        int vs = eq6_vector_size(st->n, tl, L.bs);
        if ((int64_t)tl * vs < st->n) continue;  // the vector must cover the row
        int regs = (int)ceil(regs_dense_tl1 + (double)(tl - 1) * (regs_dense_tl40 - regs_dense_tl1) / 39.0);
        int smem = (L.bs / (vs < p.warp_size ? vs : p.warp_size)) * s;  // per-vector broadcast slots
        int b = blocks_per_sm(p, L.bs, regs, smem);
        if (b <= 0) continue;
        int nw = b * L.bs / p.warp_size;
        int64_t loads = (int64_t)tl * vs / p.warp_size;               // warp-loads per vector
        int64_t wasted = ((int64_t)tl * vs - st->n) / p.warp_size;    // floor((TL*VS - n)/32)
        double useful = loads > 0 ? nw * (1.0 - (double)wasted / (double)loads) : nw;
        if (useful > best + 1e-9) {
          best = useful;
          L.tl = tl;
          L.vs = vs;
          L.regs_per_thread = regs;
          L.blocks_per_sm = b;
          L.concurrent_warps = nw;
          L.smem_bytes = smem;
        }
      }
      FP_REQUIRE(best > 0, FP_ERR_UNSUPPORTED,
                 "fp_choose_paper: n=%lld needs TL > 40 (P:362: fall back to two gemv calls)", (long long)st->n);
    }
    L.variant = L.vs > p.warp_size ? FP_VAR_DENSE_CTA : FP_VAR_DENSE_VECTOR;
  }
  L.grid = L.blocks_per_sm * p.sm_count;
  // Eq. (5): C = floor(m / (NSM * NW / VS)), NW read as concurrent threads per SM
  // (the only reading that reproduces 223 at P:457).
  int64_t vectors = (int64_t)p.sm_count * L.concurrent_warps * p.warp_size / L.vs;
  L.rows_per_vector = vectors > 0 ? st->m / vectors : 0;
  *out = L;
  return FP_OK;
}

fp_status fp_choose(int is_csr, const fp_row_stats* st, fp_dtype dtype, int device, fp_launch* out) {
  FP_REQUIRE(st && out, FP_ERR_INVALID_ARG, "fp_choose: NULL argument");
  FP_REQUIRE(fp::valid_dtype(dtype), FP_ERR_INVALID_ARG, "fp_choose: bad dtype");
  fp::PatternArgs a;
  a.m = st->m;
  a.n = st->n;
  a.nnz = st->nnz;
  a.ld = st->n;
  a.dtype = dtype;
  a.X = (const void*)(uintptr_t)256;  // alignment assumed (256-byte aligned allocations)
  a.y = (const void*)(uintptr_t)256;  // plan the full pattern (HAS_Y)
  int prev = fp::current_device();
  FP_CUDA(cudaSetDevice(device));
  fp_status r = is_csr ? fp::plan_csr(a, device, out) : fp::plan_dense(a, device, out);
  cudaSetDevice(prev);
  return r;
}

}  // extern "C"

// ------------------------------------------------------------------------- device row stats
namespace {
struct DevStats {
  unsigned long long hist[64];
  long long max_len;
  long long min_len;
  unsigned long long empty;
  unsigned long long bad;  // rows with negative length
};

__global__ void k_row_stats(int64_t m, const int64_t* __restrict__ rowptr, DevStats* out) {
  __shared__ unsigned long long hist[64];
  __shared__ long long smax, smin;
  __shared__ unsigned long long sempty, sbad;
  if (threadIdx.x < 64) hist[threadIdx.x] = 0;
  if (threadIdx.x == 0) { smax = 0; smin = LLONG_MAX; sempty = 0; sbad = 0; }
  __syncthreads();
  long long lmax = 0, lmin = LLONG_MAX;
  unsigned long long lempty = 0, lbad = 0;
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    int64_t L = rowptr[r + 1] - rowptr[r];
    if (L < 0) { lbad++; continue; }
    lmax = L > lmax ? L : lmax;
    lmin = L < lmin ? L : lmin;
    lempty += (L == 0);
    int b = 0;
    if (L > 0) b = 64 - __clzll((unsigned long long)L);
    atomicAdd(&hist[b], 1ull);
  }
  atomicMax(&smax, lmax);
  atomicMin(&smin, lmin);
  atomicAdd(&sempty, lempty);
  atomicAdd(&sbad, lbad);
  __syncthreads();
  if (threadIdx.x < 64) atomicAdd(&out->hist[threadIdx.x], hist[threadIdx.x]);
  if (threadIdx.x == 0) {
    atomicMax(&out->max_len, smax);
    atomicMin(&out->min_len, smin);
    atomicAdd(&out->empty, sempty);
    atomicAdd(&out->bad, sbad);
  }
}

__global__ void k_csr_check(int64_t m, int64_t n, int64_t nnz, const int64_t* __restrict__ rowptr,
                            const int32_t* __restrict__ colidx, unsigned long long* bad) {
  unsigned long long b = 0;
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, nt = (int64_t)gridDim.x * blockDim.x;
  if (tid == 0) b += (rowptr[0] != 0) + (rowptr[m] != nnz);
  for (int64_t r = tid; r < m; r += nt) b += rowptr[r + 1] < rowptr[r];
  for (int64_t k = tid; k < nnz; k += nt) {
    int32_t c = colidx[k];
    b += (c < 0) | ((int64_t)c >= n);
  }
  if (b) atomicAdd(bad, b);
}
}  // namespace

extern "C" fp_status fp_row_stats_device(int64_t m, const int64_t* rowptr, fp_row_stats* out, fp_stream stream) {
  FP_REQUIRE(out && m >= 0 && (m == 0 || rowptr), FP_ERR_INVALID_ARG, "fp_row_stats_device: bad arguments");
  cudaStream_t s = (cudaStream_t)stream;
  memset(out, 0, sizeof(*out));
  out->m = m;
  out->n = -1;
  if (m == 0) return FP_OK;
  DevStats* d = nullptr;
  FP_CUDA(cudaMallocAsync((void**)&d, sizeof(DevStats), s));
  DevStats init{};
  init.min_len = LLONG_MAX;
  cudaMemcpyAsync(d, &init, sizeof(init), cudaMemcpyHostToDevice, s);
  int grid = (int)((m + 255) / 256);
  if (grid > 148 * 8) grid = 148 * 8;
  k_row_stats<<<grid, 256, 0, s>>>(m, rowptr, d);
  DevStats h{};
  int64_t ends[2] = {0, 0};
  cudaMemcpyAsync(&h, d, sizeof(h), cudaMemcpyDeviceToHost, s);
  cudaMemcpyAsync(&ends[0], rowptr, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
  cudaMemcpyAsync(&ends[1], rowptr + m, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(d, s);
  FP_CUDA(cudaStreamSynchronize(s));
  FP_REQUIRE(h.bad == 0, FP_ERR_INVALID_CSR, "fp_row_stats_device: rowptr decreases (%llu rows)", h.bad);
  for (int i = 0; i < 64; ++i) out->hist_log2[i] = (int64_t)h.hist[i];
  out->max_len = h.max_len;
  out->min_len = h.min_len;
  out->empty_rows = (int64_t)h.empty;
  out->nnz = ends[1] - ends[0];
  out->mean = (double)out->nnz / (double)m;
  return FP_OK;
}

extern "C" fp_status fp_csr_validate(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                                     fp_stream stream) {
  FP_REQUIRE(m >= 0 && n >= 0 && nnz >= 0 && rowptr && (nnz == 0 || colidx), FP_ERR_INVALID_ARG,
             "fp_csr_validate: bad arguments");
  cudaStream_t s = (cudaStream_t)stream;
  unsigned long long* d = nullptr;
  FP_CUDA(cudaMallocAsync((void**)&d, sizeof(*d), s));
  cudaMemsetAsync(d, 0, sizeof(*d), s);
  int64_t work = m > nnz ? m : nnz;
  int grid = (int)((work + 255) / 256);
  if (grid > 148 * 8) grid = 148 * 8;
  if (grid < 1) grid = 1;
  k_csr_check<<<grid, 256, 0, s>>>(m, n, nnz, rowptr, colidx, d);
  unsigned long long h = 0;
  cudaMemcpyAsync(&h, d, sizeof(h), cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(d, s);
  FP_CUDA(cudaStreamSynchronize(s));
  FP_REQUIRE(h == 0, FP_ERR_INVALID_CSR, "fp_csr_validate: %llu structural violations", h);
  return FP_OK;
}
