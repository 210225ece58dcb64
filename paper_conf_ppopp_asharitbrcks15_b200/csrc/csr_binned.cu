// csr_binned.cu -- variant 17 (FP_VAR_CSR_BINNED): the large-n CSR path without per-nonzero
// global reds.
//
// Why.  For n too wide for one SM (C4: n = 1e5 fp32, y and w 400 KB each) the paper sends
// every product x*q to the global w with an atomic (Alg. 2 l.17-18 at large n).  On
// sm_100a a random fp32 red costs the issuing SM ~1.7 cycles per LANE (0.60 reds/clk/SM,
// tools/microbench/l2_scatter.cu mode 1 -- the same when the 32 lanes hit consecutive words),
// so C4's 2e9 reds alone take ~12 ms.  Shared-memory integer atomics run at ~10 per clock per
// SM (modes 3/4), but one SM holds at most ~56K words.
//
// What.  Three kernels per evaluation:
//  k_bin_produce -- X streamed once (Eq. 2 / Alg. 2 l.9-12): the row dot from a y prefix in
//    shared memory + L1/L2 gathers for the rest, q = alpha v p; then the scatter of Eq. (3)
//    (Alg. 2 l.13-14) as MESSAGES: each term t = x q is stored with its column inside its
//    column block (16 bits).  Two column blocks: warp gw owns the message slots of its own
//    nonzero range [nz0, nz1); block-0 messages fill it upward from nz0, block-1 messages
//    downward from nz1 -- plain coalesced stores, no allocation, no atomics.  Rows up to
//    kLT nonzeros go in "flat" batches (lanes on consecutive nonzeros, a segmented reduction
//    steered by a per-tile head bitmask); longer rows go warp-per-row in kNB-tile segments
//    (every load of a segment in flight at once).
//  k_bin_consume -- one 1024-thread CTA per SM holds one column block of w in shared memory
//    as 32-bit fixed point and adds its block's messages with native shared atomics.
//  k_bin_finalize -- sums the consumers' partials exactly in int64 and writes
//    w = beta z + quantum * sum (+ the non-finite spill).
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

constexpr int kProdBS = 1024;
constexpr int kConsBS = 1024;
constexpr int kNB = 8;            // register tiles of 32 nonzeros per batch / segment
constexpr int kCAP = 32 * kNB;    // nonzeros per flat batch
constexpr int kLT = 128;          // rows longer than this go warp-per-row

struct BinPArgs {
  int64_t m, nnz;
  const int64_t* rowptr;
  const int32_t* colidx;
  const float* val;
  const float* y;
  const float* v;
  float alpha;
  int ny_s;          // leading y entries staged in shared memory
  int bw;            // block-0 width (columns >= bw are block 1; bw >= n: one block)
  uint16_t* bcol;    // [nnz] message column within its block
  float* bval;       // [nnz] message value
  int64_t* wsplit;   // [warps][3]: nz0, split (first block-1 slot), nz1
  unsigned* gmax;    // largest finite |term| (float bits)
};

struct BinCArgs {
  const uint16_t* bcol;
  const float* bval;
  const int64_t* wsplit;
  const unsigned* gmax;
  int32_t* part;   // [consumers][bw]
  int32_t* hi;     // [n] wrap counts, all-zero on entry (re-zeroed by the finalize)
  float* spill;    // [n] non-finite terms, all-zero on entry
  int bw, nbin;
  int64_t pw;      // producer warps
};

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned r;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned lanemask_le() {
  unsigned r;
  asm("mov.u32 %0, %%lanemask_le;" : "=r"(r));
  return r;
}

// E with max|t| < 2^E (frexp), 0 for an all-zero call
__device__ __forceinline__ int bin_exponent(const unsigned* gmax) {
  int e = 0;
  frexpf(__uint_as_float(*gmax), &e);
  return e;
}

template <int YM>
__global__ void __launch_bounds__(kProdBS, 1) k_bin_produce(const BinPArgs a) {
  constexpr int NW = kProdBS / 32;
  extern __shared__ __align__(16) float y_s[];
  __shared__ float rs[NW][32];          // per-warp row sums, compressed (non-empty) row order
  __shared__ unsigned hmw[NW][kNB];     // per-warp head masks of the batch's tiles
  __shared__ unsigned char cmap[NW][32];  // compressed row -> lane of the batch
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t* __restrict__ rowptr = a.rowptr;
  const int32_t* __restrict__ colidx = a.colidx;
  const float* __restrict__ val = a.val;
  const float* __restrict__ y = a.y;
  const int ny_s = YM ? a.ny_s : 0;
  for (int j = threadIdx.x; j < ny_s; j += kProdBS) y_s[j] = y[j];
  __syncthreads();
  auto Y = [&](int c) -> float { return c < ny_s ? y_s[c] : fpd::ld_keep(y + c); };

  const int64_t m = a.m;
  const int64_t gw = (int64_t)blockIdx.x * NW + warp, tw = (int64_t)gridDim.x * NW;
  const int64_t total = a.nnz + kRowCost * m;
  const int64_t r0 = warp_search_rows(rowptr, m, (total * gw) / tw, lane);
  const int64_t r1 = warp_search_rows(rowptr, m, (total * (gw + 1)) / tw, lane);
  const int64_t base0 = __ldg(rowptr);
  const int64_t nz0 = __ldg(rowptr + r0) - base0, nz1 = __ldg(rowptr + r1) - base0;
  int64_t up = nz0, dn = nz1;  // next block-0 slot (upward), one past the last free block-1 slot
  float tmax = 0.f;
  const unsigned lt = lanemask_lt(), le = lanemask_le();
  const int bw = a.bw;
  const float alpha = a.alpha;

  // one tile of terms (lane: column c, term t, active) -> message slots of the warp
  auto EMIT = [&](int c, float t, bool act) {
    const float at = fabsf(t);
    tmax = fmaxf(tmax, at <= 3.402823466e38f ? at : 0.f);
    const bool b1 = act && c >= bw;
    const unsigned m1 = __ballot_sync(0xffffffffu, b1);
    const unsigned m0 = __ballot_sync(0xffffffffu, act) & ~m1;
    if (act) {
      const int64_t idx = b1 ? dn - 1 - __popc(m1 & lt) : up + __popc(m0 & lt);
      a.bcol[idx] = (uint16_t)(b1 ? c - bw : c);
      a.bval[idx] = t;
    }
    up += __popc(m0);
    dn -= __popc(m1);
  };

  auto RP = [&](int64_t b) -> int64_t { return __ldg(rowptr + (b + lane < r1 ? b + lane : r1)); };
  auto RP_END = [&](int64_t b) -> int64_t { return __ldg(rowptr + (b + 32 < r1 ? b + 32 : r1)); };
  int64_t rp_cur = RP(r0), rp_end_cur = RP_END(r0);
  for (int64_t rb = r0; rb < r1;) {
    const int64_t rp = rp_cur, rp_end = rp_end_cur;
    const int64_t a0 = __shfl_sync(0xffffffffu, rp, 0);
    int64_t nxt = __shfl_down_sync(0xffffffffu, rp, 1);
    if (lane == 31) nxt = rp_end;
    const bool inr = rb + lane < r1;
    const int64_t len = inr ? nxt - rp : 0;
    // a flat batch: the leading run of rows with <= kLT nonzeros whose total fits kCAP
    const bool ok = inr && len <= kLT && nxt - a0 <= kCAP;
    const int nrows = __ffs(~__ballot_sync(0xffffffffu, ok)) - 1;  // leading ones (-1 if all 32 ok)
    const int nr = nrows < 0 ? 32 : nrows;
    const float vpre = (a.v && inr) ? fpd::ld_once(a.v + rb + lane) : 1.f;
    const int64_t rb_next = rb + (nr == 0 ? 1 : nr);
    rp_cur = RP(rb_next);
    rp_end_cur = RP_END(rb_next);

    if (nr == 0) {
      // ---- row rb is long: warp-per-row in segments of kNB tiles, loads of a segment in flight
      // together; the first segment stays in registers for the scatter, the rest is re-read
      // (L2-resident after the dot pass; the paper's "likely a cache hit")
      const int64_t s0 = a0;
      const int64_t L = __shfl_sync(0xffffffffu, len, 0);
      int cc[kNB];
      float xv[kNB];
      float acc = 0.f;
#pragma unroll
      for (int j = 0; j < kNB; ++j) {
        const int64_t k = j * 32 + lane;
        cc[j] = k < L ? fpd::ld_once(colidx + s0 + k) : 0;
        xv[j] = k < L ? fpd::ld_once(val + s0 + k) : 0.f;
      }
      if constexpr (YM != 0) {
        float yv[kNB];
#pragma unroll
        for (int j = 0; j < kNB; ++j) yv[j] = Y(cc[j]);
#pragma unroll
        for (int j = 0; j < kNB; ++j) acc = fmaf(xv[j], yv[j], acc);
        for (int64_t seg = kCAP; seg < L; seg += kCAP) {
          int c2[kNB];
          float x2[kNB], y2[kNB];
#pragma unroll
          for (int j = 0; j < kNB; ++j) {
            const int64_t k = seg + j * 32 + lane;
            c2[j] = k < L ? __ldg(colidx + s0 + k) : 0;
            x2[j] = k < L ? __ldg(val + s0 + k) : 0.f;
          }
#pragma unroll
          for (int j = 0; j < kNB; ++j) y2[j] = Y(c2[j]);
#pragma unroll
          for (int j = 0; j < kNB; ++j) acc = fmaf(x2[j], y2[j], acc);
        }
        acc = fpd::vector_allreduce<32>(acc);
      }
      const float vr = __shfl_sync(0xffffffffu, vpre, 0);
      const float q = (YM != 0 ? acc * vr : vr) * alpha;
#pragma unroll
      for (int j = 0; j < kNB; ++j) EMIT(cc[j], xv[j] * q, j * 32 + lane < L);
      for (int64_t seg = kCAP; seg < L; seg += 32) {
        const int64_t k = seg + lane;
        const bool act = k < L;
        const int c = act ? __ldg(colidx + s0 + k) : 0;
        const float x = act ? __ldg(val + s0 + k) : 0.f;
        EMIT(c, x * q, act);
      }
      rb = rb_next;
      continue;
    }

    // ---- flat batch of rows [rb, rb + nr): lanes on consecutive nonzeros
    const int cnt = (int)(__shfl_sync(0xffffffffu, nxt, nr - 1) - a0);
    const bool ne = lane < nr && len > 0;
    const unsigned nem = __ballot_sync(0xffffffffu, ne);
    const int rel = (int)(rp - a0);
    if (lane < kNB) hmw[warp][lane] = 0u;
    __syncwarp();
    if (ne) {
      atomicOr(&hmw[warp][rel >> 5], 1u << (rel & 31));
      cmap[warp][__popc(nem & lt)] = (unsigned char)lane;
    }
    int cc[kNB];
    float xv[kNB];
#pragma unroll
    for (int j = 0; j < kNB; ++j) {
      const int pos = j * 32 + lane;
      cc[j] = pos < cnt ? fpd::ld_once(colidx + a0 + pos) : 0;
      xv[j] = pos < cnt ? fpd::ld_once(val + a0 + pos) : 0.f;
    }
    rs[warp][lane] = 0.f;
    __syncwarp();
    unsigned hm[kNB];
#pragma unroll
    for (int j = 0; j < kNB; ++j) hm[j] = hmw[warp][j];
    // compressed row index of every nonzero: heads at or before it, minus one
    int rid[kNB];
    {
      int base = 0;
#pragma unroll
      for (int j = 0; j < kNB; ++j) {
        rid[j] = base - 1 + __popc(hm[j] & le);
        base += __popc(hm[j]);
      }
    }
    if constexpr (YM != 0) {
      float yv[kNB];
#pragma unroll
      for (int j = 0; j < kNB; ++j) yv[j] = Y(cc[j]);
#pragma unroll
      for (int j = 0; j < kNB; ++j) {
        if (j * 32 >= cnt) break;
        float s = xv[j] * yv[j];  // Eq. (2) products (0 on inactive lanes)
        // segmented suffix sums toward each segment's first lane: lane l adds lane l+d while
        // l+d is in its segment (no head in (l, l+d], and inside the tile)
        const unsigned after = (hm[j] >> lane) >> 1;
        const int dist = after ? __ffs(after) : 32 - lane;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const float t = __shfl_down_sync(0xffffffffu, s, d);
          if (d < dist) s += t;
        }
        const bool head = j * 32 + lane < cnt && (lane == 0 || ((hm[j] >> lane) & 1u));
        if (head) rs[warp][rid[j]] += s;  // heads of one tile hold distinct rows
      }
      __syncwarp();
    }
    // lane k owns the k-th non-empty row of the batch: q = alpha v p
    float q = 0.f;
    {
      const int nne = __popc(nem);
      const int src = lane < nne ? cmap[warp][lane] : 0;
      const float vr = __shfl_sync(0xffffffffu, vpre, src);
      if (lane < nne) q = (YM != 0 ? rs[warp][lane] * vr : vr) * alpha;
    }
#pragma unroll
    for (int j = 0; j < kNB; ++j) {
      if (j * 32 >= cnt) break;
      const float qj = __shfl_sync(0xffffffffu, q, rid[j] & 31);
      EMIT(cc[j], xv[j] * qj, j * 32 + lane < cnt);
    }
    rb = rb_next;
  }
  if (lane == 0) {
    a.wsplit[3 * gw] = nz0;
    a.wsplit[3 * gw + 1] = up;  // == dn: every slot of [nz0, nz1) written
    a.wsplit[3 * gw + 2] = nz1;
  }
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) tmax = fmaxf(tmax, __shfl_xor_sync(0xffffffffu, tmax, d));
  if (lane == 0 && tmax > 0.f) atomicMax(a.gmax, __float_as_uint(tmax));
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
  constexpr int U = 4;  // loads in flight per lane
  for (int64_t p = pw0 + warp; p < pw1; p += kConsBS / 32) {
    const int64_t lo = a.wsplit[3 * p + b], hi = a.wsplit[3 * p + b + 1];
    for (int64_t i0 = lo; i0 < hi; i0 += 32 * U) {
      int c[U];
      float t[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int64_t i = i0 + u * 32 + lane;
        c[u] = i < hi ? (int)__ldcs(a.bcol + i) : 0;
        t[u] = i < hi ? __ldcs(a.bval + i) : 0.f;
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (i0 + u * 32 + lane < hi) ADD(c[u], t[u]);
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

// columns one consumer CTA can hold (int32 partial in the opt-in shared memory)
int binned_max_bw() { return (227 * 1024 - 1024) / 4 / 16 * 16; }

// column blocks for n columns (1 or 2), 0 if n is too wide for this variant
int binned_nbin(int64_t n) {
  const int64_t mb = binned_max_bw();
  if (n <= mb) return 1;
  if ((n + 1) / 2 <= mb) return 2;
  return 0;
}

size_t binned_ws_bytes(int64_t n, int64_t nnz, int nbin, int producer_grid, int consumers) {
  const int64_t pw = (int64_t)producer_grid * (kProdBS / 32);
  const int64_t bw = (n + nbin - 1) / nbin;
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  return al((size_t)nnz * 2) + al((size_t)nnz * 4) + al((size_t)pw * 24) + al((size_t)consumers * bw * 4) + 256;
}

fp_status launch_binned(const PatternArgs& a, const fp_launch& L, int64_t y_prefix, cudaStream_t s) {
  FP_REQUIRE(a.dtype == FP_F32, FP_ERR_UNSUPPORTED, "fp_csr: variant %d (binned) is fp32 only", L.variant);
  FP_REQUIRE(a.epi_kind == 0 && !a.row_out, FP_ERR_UNSUPPORTED, "fp_csr: variant %d has no row epilogue",
             L.variant);
  const int nbin = L.cluster > 0 ? L.cluster : binned_nbin(a.n);
  FP_REQUIRE(nbin == 1 || nbin == 2, FP_ERR_UNSUPPORTED, "fp_csr: binned variant needs 1 or 2 column blocks");
  const int bw = (int)((a.n + nbin - 1) / nbin);
  FP_REQUIRE(bw <= binned_max_bw(), FP_ERR_UNSUPPORTED, "fp_csr: n = %lld too wide for %d column blocks",
             (long long)a.n, nbin);
  const int sms = device_info(current_device()).sm_count;
  const int grid = L.grid > 0 ? L.grid : sms;
  const int ncons = std::max(sms, nbin);
  const int64_t pw = (int64_t)grid * (kProdBS / 32);
  // workspace: [bcol][bval][wsplit][part][gmax]; hi and spill live in a second buffer that is
  // all-zero between calls (zeroed when allocated, re-zeroed by the finalize)
  auto al = [](size_t x) { return (x + 255) / 256 * 256; };
  const size_t bytes = binned_ws_bytes(a.n, a.nnz, nbin, grid, ncons);
  unsigned char* base = (unsigned char*)workspace_buffer(s, kWsBins, bytes, false);
  unsigned char* zbase = (unsigned char*)workspace_buffer(s, kWsBinsZero, 2 * al((size_t)a.n * 4), true);
  if (!base || !zbase) return FP_ERR_NOMEM;
  size_t off = 0;
  auto take = [&](size_t b) {
    unsigned char* p = base + off;
    off += al(b);
    return p;
  };
  BinPArgs k{};
  k.m = a.m;
  k.nnz = a.nnz;
  k.rowptr = a.rowptr;
  k.colidx = a.colidx;
  k.val = (const float*)a.val;
  k.y = (const float*)a.y;
  k.v = (const float*)a.v;
  k.alpha = (float)a.alpha;
  k.ny_s = a.y ? (int)y_prefix : 0;
  k.bw = nbin == 2 ? bw : INT32_MAX;
  k.bcol = (uint16_t*)take((size_t)a.nnz * 2);
  k.bval = (float*)take((size_t)a.nnz * 4);
  k.wsplit = (int64_t*)take((size_t)pw * 24);
  int32_t* part = (int32_t*)take((size_t)ncons * bw * 4);
  k.gmax = (unsigned*)take(16);
  int32_t* hi = (int32_t*)zbase;
  float* spill = (float*)(zbase + al((size_t)a.n * 4));
  FP_CUDA(cudaMemsetAsync(k.gmax, 0, 16, s));
  const void* f = a.y ? (const void*)k_bin_produce<1> : (const void*)k_bin_produce<0>;
  set_max_dynamic_smem(f);
  const size_t psmem = (size_t)k.ny_s * 4;
  if (a.y) k_bin_produce<1><<<grid, kProdBS, psmem, s>>>(k);
  else k_bin_produce<0><<<grid, kProdBS, psmem, s>>>(k);
  FP_CUDA(cudaGetLastError());
  BinCArgs c{k.bcol, k.bval, k.wsplit, k.gmax, part, hi, spill, bw, nbin, pw};
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

// register count of the producer (plan reports)
int binned_producer_regs(bool has_y) {
  cudaFuncAttributes fa{};
  if (cudaFuncGetAttributes(&fa, has_y ? (const void*)k_bin_produce<1> : (const void*)k_bin_produce<0>) !=
      cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return fa.numRegs;
}

}  // namespace fp
