// csr_binned.cu -- variant 17 (FP_VAR_CSR_BINNED): the large-n CSR path without per-nonzero
// global reds.
//
// Why.  For n too wide for one SM (C4: n = 1e5 fp32, y and w 400 KB each) the paper sends
// every product x*q to the global w with an atomic (Alg. 2 l.17-18 at large n).  On
// sm_100a a random fp32 red costs the issuing SM ~1.7 cycles per LANE (0.60 reds/clk/SM,
// tools/microbench/l2_scatter.cu mode 1 -- the same when the 32 lanes hit consecutive words),
// so C4's 2e9 reds alone take ~12 ms whatever the layout.  Shared-memory integer atomics run
// at ~10 per clock per SM (modes 3/4), but one SM holds at most ~56K words.
//
// What.  The producer (k_csr_flat<..., MODE_BINk>, csr_flat.cuh) is variant 16's flat kernel
// -- X streamed once, the row dot from the y prefix in shared memory + L1/L2 gathers, q =
// alpha v p (Eq. 2, Alg. 2 l.9-12) -- but the scatter of Eq. (3) (Alg. 2 l.13-14) writes each
// term t = x*q as a message (16-bit column inside its column block, fp32 t) into the chunk of
// its block's bin.  Messages are plain coalesced stores: bandwidth, not per-lane atomics.
// k_bin_consume (one 1024-thread CTA per SM) owns one column block of w in shared memory as
// 32-bit fixed point and adds its bin's messages with native shared atomics; k_bin_finalize
// sums the consumers' partials exactly in int64 and writes w = beta z + quantum * sum.
//
// Fixed point (reading R22).  quantum = 2^(E-26) with 2^(E-1) <= max|t| < 2^E over
// the whole call (the producer's atomicMax of finite |t|), so every term is an int32 of
// magnitude <= 2^26 rounded to the nearest quantum (error <= 2^-27 max|t| per term, below the
// fp32 rounding of the term itself for |t| >= max|t| / 8).  The int32 accumulator wraps after
// ~32 max-size terms of one sign; the returning atomic detects the wrap and counts it in
// hi[col] (global int32, rare), so the per-column sum is exact in 64 bits: the result is the
// same for every summation order (deterministic, and bit-exact on integer inputs).  Non-finite
// terms go to an fp32 spill vector with a global red (IEEE propagation, reading R8).
#include <algorithm>

#include "csr_kernels.cuh"

namespace fp {

namespace {

constexpr int kConsBS = 1024;

struct BinCArgs {
  const uint16_t* bcol;
  const float* bval;
  const uint32_t* bdir;
  const int64_t* wbase;
  const int32_t* wcount;
  const unsigned* gmax;
  int32_t* part;   // [consumers][bw]
  int32_t* hi;     // [n] wrap counts, all-zero on entry (re-zeroed by the finalize)
  float* spill;    // [n] non-finite terms, all-zero on entry
  int bw, nbin;
  int64_t pw;      // producer warps
};

__device__ __forceinline__ uint4 ld_msg16(const uint16_t* p) {
  uint4 r;
  asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p));
  return r;
}
__device__ __forceinline__ void ld_msg32(const float* p, float (&r)[8]) {
  asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]), "=f"(r[6]), "=f"(r[7])
      : "l"(p));
}

// E with max|t| < 2^E (frexp), 0 for an all-zero call
__device__ __forceinline__ int bin_exponent(const unsigned* gmax) {
  int e = 0;
  frexpf(__uint_as_float(*gmax), &e);
  return e;
}

__global__ void __launch_bounds__(kConsBS, 1) k_bin_consume(const BinCArgs a) {
  extern __shared__ __align__(16) int32_t sw[];
  for (int j = threadIdx.x; j < a.bw; j += kConsBS) sw[j] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int b = (int)(blockIdx.x % (unsigned)a.nbin);
  const int cid = (int)(blockIdx.x / (unsigned)a.nbin);
  const int ncons = ((int)gridDim.x - b + a.nbin - 1) / a.nbin;
  const int64_t pw0 = a.pw * cid / ncons, pw1 = a.pw * (cid + 1) / ncons;
  const int ex = 26 - bin_exponent(a.gmax);
  const bool fscale = ex >= -125 && ex <= 127;  // 2^ex representable as float (the usual case)
  const float sf = fscale ? ldexpf(1.f, ex) : 0.f;
  const double sd = ldexp(1.0, ex);
  const int64_t col0 = (int64_t)b * a.bw;
  auto ADD = [&](int cl, float t) {
    if (!(fabsf(t) <= 3.402823466e38f)) {  // Inf / NaN: IEEE propagation through the spill
      atomicAdd(a.spill + col0 + cl, t);
      return;
    }
    const int qi = fscale ? __float2int_rn(t * sf) : __double2int_rn((double)t * sd);
    const int old = atomicAdd(sw + cl, qi);  // native ATOMS.ADD (with return)
    const unsigned nw = (unsigned)old + (unsigned)qi;
    if ((int)(((unsigned)old ^ nw) & ((unsigned)qi ^ nw)) < 0)  // signed wrap: carry into hi
      atomicAdd(a.hi + col0 + cl, qi > 0 ? 1 : -1);
  };
  for (int64_t p = pw0 + warp; p < pw1; p += kConsBS / 32) {
    const int64_t base = a.wbase[p];
    const int cnt = a.wcount[p];
    for (int j0 = 0; j0 < cnt; j0 += 32) {
      const uint32_t d = j0 + lane < cnt ? __ldg(a.bdir + base + j0 + lane) : 0u;
      unsigned mine = __ballot_sync(0xffffffffu, (int)(d >> 16) == b && (d & 0xffffu) != 0);
      while (mine) {
        const int i = __ffs(mine) - 1;
        mine &= mine - 1;
        const int count = (int)(__shfl_sync(0xffffffffu, d, i) & 0xffffu);
        const int64_t e0 = (base + j0 + i) * kBinCH + lane * 8;
        if (lane * 8 < count) {
          const uint4 cv = ld_msg16(a.bcol + e0);
          float tv[8];
          ld_msg32(a.bval + e0, tv);
          const uint32_t cw[4] = {cv.x, cv.y, cv.z, cv.w};
#pragma unroll
          for (int e = 0; e < 8; ++e)
            if (lane * 8 + e < count) ADD((int)((cw[e >> 1] >> (16 * (e & 1))) & 0xffffu), tv[e]);
        }
      }
    }
  }
  __syncthreads();
  int32_t* dst = a.part + (int64_t)blockIdx.x * a.bw;
  for (int j = threadIdx.x; j < a.bw; j += kConsBS) dst[j] = sw[j];
}

template <typename T>
__global__ void k_bin_finalize(int64_t n, int bw, int nbin, int ncons, const int32_t* __restrict__ part,
                               int32_t* __restrict__ hi, float* __restrict__ spill, const unsigned* __restrict__ gmax,
                               const T* __restrict__ z, double beta, int add_beta_z, int accumulate, T* w) {
  const double quantum = ldexp(1.0, bin_exponent(gmax) - 26);
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    const int b = (int)(j / bw);
    const int c = (int)(j - (int64_t)b * bw);
    int64_t s = 0;
    for (int k = b; k < ncons; k += nbin) s += part[(int64_t)k * bw + c];
    s += (int64_t)hi[j] * 4294967296ll;
    double r = (double)s * quantum + (double)spill[j];
    if (add_beta_z && beta != 0.0) r += beta * (double)z[j];
    if (accumulate) r += (double)w[j];
    w[j] = (T)r;
    hi[j] = 0;
    spill[j] = 0.f;
  }
}

}  // namespace

// columns one consumer CTA can hold (int32 partial in 227 KB of shared memory)
int binned_max_bw() { return (227 * 1024 - 1024) / 4 / 16 * 16; }

// bins for n columns (1, 2 or 4), 0 if n is too wide for this variant
int binned_nbin(int64_t n) {
  const int64_t mb = binned_max_bw();
  for (int nb = 1; nb <= 4; nb *= 2)
    if ((n + nb - 1) / nb <= mb) return nb;
  return 0;
}

size_t binned_ws_bytes(int64_t n, int64_t nnz, int nbin, int producer_grid, int consumers) {
  const int64_t pw = (int64_t)producer_grid * (kWideBS / 32);
  const int64_t chunks = nnz / kBinCH + pw * (nbin + 1) + 1;
  const int64_t bw = (n + nbin - 1) / nbin;
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  return al((size_t)chunks * kBinCH * 2) + al((size_t)chunks * kBinCH * 4) + al((size_t)chunks * 4) +
         al((size_t)pw * 8) + al((size_t)pw * 4) + al((size_t)consumers * bw * 4) + 256;
}

fp_status launch_binned(const PatternArgs& a, const fp_launch& L, int64_t y_prefix, cudaStream_t s) {
  FP_REQUIRE(a.dtype == FP_F32, FP_ERR_UNSUPPORTED, "fp_csr: variant %d (binned) is fp32 only", L.variant);
  const int nbin = L.cluster > 0 ? L.cluster : binned_nbin(a.n);
  FP_REQUIRE(nbin == 1 || nbin == 2 || nbin == 4, FP_ERR_UNSUPPORTED, "fp_csr: binned variant needs 1, 2 or 4 bins");
  const int bw = (int)((a.n + nbin - 1) / nbin);
  FP_REQUIRE(bw <= binned_max_bw(), FP_ERR_UNSUPPORTED, "fp_csr: n = %lld too wide for %d bins", (long long)a.n,
             nbin);
  const int ym = !a.y ? 0 : ((a.epi_kind == 0 && !a.row_out) ? 1 : 2);
  const int mode = nbin == 1 ? DMODE_BIN1 : (nbin == 2 ? DMODE_BIN2 : DMODE_BIN4);
  CsrKFn f = csr_pick_f32(ym, mode, 32, 8);
  FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_csr: no binned producer for y mode %d", ym);
  const int sms = device_info(current_device()).sm_count;
  const int grid = L.grid > 0 ? L.grid : sms;
  const int ncons = std::max(sms, nbin);
  const int64_t pw = (int64_t)grid * (kWideBS / 32);
  const int64_t chunks = a.nnz / kBinCH + pw * (nbin + 1) + 1;
  // workspace: [bcol][bval][bdir][wbase][wcount][part][gmax]; hi and spill live in a second
  // buffer that is all-zero between calls (zeroed when allocated, re-zeroed by the finalize)
  const size_t bytes = binned_ws_bytes(a.n, a.nnz, nbin, grid, ncons);
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  unsigned char* base = (unsigned char*)workspace_buffer(s, kWsBins, bytes, false);
  unsigned char* zbase = (unsigned char*)workspace_buffer(s, kWsBinsZero, 2 * al((size_t)a.n * 4), true);
  if (!base || !zbase) return FP_ERR_NOMEM;
  size_t off = 0;
  auto take = [&](size_t b) {
    unsigned char* p = base + off;
    off += al(b);
    return p;
  };
  CsrKArgs k{a.m, a.n, a.nnz, a.rowptr, a.colidx, a.val, a.y, a.v, a.z, a.alpha, a.beta, a.w,
             nullptr, nullptr, a.add_beta_z ? 1 : 0, a.accumulate ? 1 : 0, (int)y_prefix,
             {a.epi_kind, a.epi_c, a.row_out, a.scalar_out}, 0, nullptr, 1};
  k.bcol = (uint16_t*)take((size_t)chunks * kBinCH * 2);
  k.bval = (float*)take((size_t)chunks * kBinCH * 4);
  k.bdir = (uint32_t*)take((size_t)chunks * 4);
  k.wbase = (int64_t*)take((size_t)pw * 8);
  k.wcount = (int32_t*)take((size_t)pw * 4);
  int32_t* part = (int32_t*)take((size_t)ncons * bw * 4);
  int32_t* hi = (int32_t*)zbase;
  float* spill = (float*)(zbase + al((size_t)a.n * 4));
  k.gmax = (unsigned*)take(16);
  k.bw = bw;
  k.inv_bw = 1.0f / (float)bw;
  FP_CUDA(cudaMemsetAsync(k.gmax, 0, 16, s));
  const size_t psmem = (size_t)y_prefix * 4;
  set_max_dynamic_smem((const void*)f);
  f<<<grid, kWideBS, psmem, s>>>(k);
  FP_CUDA(cudaGetLastError());
  BinCArgs c{k.bcol, k.bval, k.bdir, k.wbase, k.wcount, k.gmax, part, hi, spill, bw, nbin, pw};
  set_max_dynamic_smem((const void*)k_bin_consume);
  k_bin_consume<<<ncons, kConsBS, (size_t)bw * 4, s>>>(c);
  FP_CUDA(cudaGetLastError());
  const int fb = 256;
  const int fg = (int)std::min<int64_t>((a.n + fb - 1) / fb, 8 * sms);
  k_bin_finalize<float><<<fg, fb, 0, s>>>(a.n, bw, nbin, ncons, part, hi, spill, k.gmax, (const float*)a.z, a.beta,
                                          a.add_beta_z ? 1 : 0, a.accumulate ? 1 : 0, (float*)a.w);
  FP_CUDA(cudaGetLastError());
  return FP_OK;
}

}  // namespace fp
