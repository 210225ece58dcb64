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
//    kLT nonzeros go in "flat" batches (4 consecutive nonzeros per lane from 128-bit loads, a
//    two-level segmented reduction steered by a head bitmask); longer rows go warp-per-row in
//    steps of 256 nonzeros (every load of a step in flight at once).
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
#include <cstdlib>
#include <type_traits>

#include "csr_kernels.cuh"

namespace fp {

namespace {

constexpr int kProdBS = 1024;
constexpr int kConsBS = 1024;
constexpr int kNT = 2;            // super-tiles of 128 nonzeros (4 per lane) per batch
constexpr int kLT = 128;          // rows longer than this go warp-per-row

struct BinPArgs {
  int64_t m, nnz;
  const int64_t* rowptr;
  const int32_t* colidx;
  const void* val;   // T
  const void* y;     // T
  const void* v;     // T
  double alpha;
  int ny_s;          // leading y entries staged in shared memory
  int bw;            // block-0 width (columns >= bw are block 1; bw >= n: one block)
  int mis;           // (address of colidx / 4) mod 4 -- the same for val (checked on launch)
  int pf;            // nonzeros of colidx / val prefetched into L2 ahead of the next batch
  uint16_t* bcol;    // [nnz] message column within its block
  float* bval;       // [nnz] message value
  int64_t* wsplit;   // [warps][3]: nz0, split (first block-1 slot), nz1
  unsigned* gmax;    // largest finite |term| (float bits)
  // SINK_FIX (variant 18): the CTA partial w in shared memory + the grid finalize
  int64_t n;
  double* acc;
  unsigned long long* counter;
  const void* z;
  double beta;
  void* w;
  int add_beta_z, accumulate;
};

enum { SINK_BINS = 0, SINK_FIX = 1 };

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

// E with max|t| < 2^E (frexp), 0 for an all-zero call
__device__ __forceinline__ int bin_exponent(const unsigned* gmax) {
  int e = 0;
  frexpf(__uint_as_float(*gmax), &e);
  return e;
}

// read-once loads of 4 consecutive colidx (16 B) / val (16 or 32 B) entries, index aligned to 4
__device__ __forceinline__ void ld4(const int32_t* pc, const float* pv, int (&c)[4], float (&x)[4]) {
  asm("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
      : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3])
      : "l"(pc));
  asm("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
      : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3])
      : "l"(pv));
}
__device__ __forceinline__ void ld4(const int32_t* pc, const double* pv, int (&c)[4], double (&x)[4]) {
  asm("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
      : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3])
      : "l"(pc));
  asm("ld.global.nc.L1::no_allocate.L2::evict_first.v4.f64 {%0,%1,%2,%3}, [%4];"
      : "=d"(x[0]), "=d"(x[1]), "=d"(x[2]), "=d"(x[3])
      : "l"(pv));
}

// The producer.  Nonzeros are handled 4 per lane: a "super-tile" is 128 consecutive nonzeros
// starting at a 16-byte-aligned index, lane l holding entries 4l..4l+3 (two 128-bit loads);
// a batch spans kNT super-tiles.  Row boundaries inside a batch are a 256-bit head mask in
// shared memory (bit p set where a non-empty row starts at batch position p).  The row dot is
// a two-level segmented sum: in-lane over the lane's 4 products, then across lanes over the
// lanes' leading partial sums (a shuffle reduction bounded by the next lane holding a head).
// predicated message store (no branch around it)
__device__ __forceinline__ void st_msg(uint16_t* pc, float* pv, int c, float t, bool on) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "@p st.global.u16 [%0], %2;\n\t"
      "@p st.global.f32 [%1], %3;\n\t}"
      ::"l"(pc), "l"(pv), "h"((unsigned short)c), "f"(t), "r"((int)on)
      : "memory");
}

// SINK_BINS (variant 17, T = float): the scatter writes messages (above).  SINK_FIX (variant
// 18): the scatter adds into the CTA's partial w held in shared memory as 64-bit fixed point
// (fixacc.cuh: native 32-bit shared atomics, not the fp CAS loop), y fully staged, and the
// grid finalize of aggregate.cuh writes w = beta z + sum of the CTA partials (alpha folded into q).
template <typename T, int YM, int NBIN, int SINK, int BS, int MINB = 1>
__global__ void __launch_bounds__(BS, MINB) k_flat4(const BinPArgs a) {
  static_assert(SINK == SINK_FIX || sizeof(T) == 4, "messages are fp32");
  constexpr int NW = BS / 32;
  constexpr int NT = kNT;
  constexpr int SPAN = 128 * NT;                // nonzero positions of a batch
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* y_s = reinterpret_cast<T*>(smem_raw);
  __shared__ T rs[NW][32];                      // per-warp row sums, compressed (non-empty) row order
  __shared__ unsigned hmw[NW][SPAN / 32];       // per-warp head masks
  __shared__ unsigned char cmap[NW][32];        // compressed row -> lane of the batch
  __shared__ int fix_e;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t* __restrict__ rowptr = a.rowptr;
  const int32_t* __restrict__ colidx = a.colidx;
  const T* __restrict__ val = (const T*)a.val;
  const T* __restrict__ y = (const T*)a.y;
  const int ny_s = YM ? a.ny_s : 0;
  for (int j = threadIdx.x; j < ny_s; j += BS) y_s[j] = y[j];
  // SINK_FIX: [y (16-byte padded)][sp: n f64][lo: n u32][hi: n u32] behind it
  const fpd::FixAcc FA = fix_layout(smem_raw + (SINK == SINK_FIX ? fix_y_bytes(YM ? a.n : 0, (int)sizeof(T)) : 0),
                                    SINK == SINK_FIX ? a.n : 0, &fix_e);
  fpd::FixScale FS;
  if constexpr (SINK == SINK_FIX) fpd::fix_init<BS>(FA, a.n);
  __syncthreads();
  auto Y = [&](int c) -> T {
    if constexpr (SINK == SINK_FIX) return y_s[c];
    else return c < ny_s ? y_s[c] : fpd::ld_keep(y + c);
  };
  const int mis = a.mis;

  const int64_t m = a.m;
  const int64_t gw = (int64_t)blockIdx.x * NW + warp, tw = (int64_t)gridDim.x * NW;
  const int64_t total = a.nnz + kRowCost * m;
  const int64_t r0 = warp_search_rows(rowptr, m, (total * gw) / tw, lane);
  const int64_t r1 = warp_search_rows(rowptr, m, (total * (gw + 1)) / tw, lane);
  const int64_t base0 = __ldg(rowptr);
  const int64_t nz0 = __ldg(rowptr + r0) - base0, nz1 = __ldg(rowptr + r1) - base0;
  // message slots of this warp: [nz0, nz1); offsets relative to nz0 (< 2^31, checked on launch)
  uint16_t* const bcol = SINK == SINK_BINS ? a.bcol + nz0 : nullptr;
  float* const bval = SINK == SINK_BINS ? a.bval + nz0 : nullptr;
  int up = 0, dn = (int)(nz1 - nz0);  // next block-0 slot (upward), one past the last free block-1 slot
  float tmax = 0.f;
  const unsigned lt = lanemask_lt();
  const int bw = a.bw;
  const T alpha = (T)a.alpha;

  // The scatter of one super-tile: lane l's 4 terms (columns c, values t, active bits act),
  // one entry index per step: the step's block-0 lanes take consecutive slots upward from
  // `up`, its block-1 lanes consecutive slots downward from `dn` -- every store instruction
  // covers consecutive slots.  Branch-free: predicated stores, 32-bit slot arithmetic.
  auto EMIT4 = [&](const int (&c)[4], const T (&t)[4], unsigned act) {
    if constexpr (SINK == SINK_FIX) {
      if (FS.e == fpd::kFixUnset) {  // the CTA's cap exponent from the first terms (fixacc.cuh)
        double tm = 0.0;
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          double at;
          if (((act >> e) & 1u) && fpd::fix_finite_abs((double)t[e], at)) tm = fmax(tm, at);
        }
        fpd::fix_try_set(FA, FS, tm);
      }
#pragma unroll
      for (int e = 0; e < 4; ++e)
        if ((act >> e) & 1u) fpd::fix_add(FA, FS, c[e], t[e]);
      return;
    }
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      tmax = fmaxf(tmax, fabsf((float)t[e]));  // inactive terms are 0; NaN is ignored, Inf kept
      const bool on = (act >> e) & 1u;
      unsigned idx;
      int cl = c[e];
      if constexpr (NBIN == 2) {
        const bool b1 = on && c[e] >= bw;
        const unsigned m1 = __ballot_sync(0xffffffffu, b1);
        const unsigned m0 = __ballot_sync(0xffffffffu, on) & ~m1;
        const unsigned i0 = (unsigned)up + __popc(m0 & lt), i1 = (unsigned)dn - 1u - __popc(m1 & lt);
        idx = b1 ? i1 : i0;
        cl = b1 ? c[e] - bw : c[e];
        up += __popc(m0);
        dn -= __popc(m1);
      } else {
        const unsigned m0 = __ballot_sync(0xffffffffu, on);
        idx = (unsigned)up + __popc(m0 & lt);
        up += __popc(m0);
      }
      st_msg(bcol + idx, bval + idx, cl, (float)t[e], on);
    }
  };

  auto RP = [&](int64_t b) -> int64_t { return __ldg(rowptr + (b + lane < r1 ? b + lane : r1)); };
  auto RP_END = [&](int64_t b) -> int64_t { return __ldg(rowptr + (b + 32 < r1 ? b + 32 : r1)); };
  // 4 entries at aligned index g = A + o (o = 4 * lane + 128 * t): loaded when any is before
  // `hi`; active = inside [lo, hi) (positions relative to A, 32-bit)
  auto LOAD4 = [&](int64_t A, int o, int lo, int hi, int (&c)[4], T (&x)[4]) -> unsigned {
    unsigned act = 0;
    if (o < hi) {
      ld4(colidx + A + o, val + A + o, c, x);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const bool in = o + e >= lo && o + e < hi;
        act |= (unsigned)in << e;
        if (!in) c[e] = 0, x[e] = T(0);
      }
    } else {
#pragma unroll
      for (int e = 0; e < 4; ++e) c[e] = 0, x[e] = T(0);
    }
    return act;
  };
  int64_t rp_cur = RP(r0), rp_end_cur = RP_END(r0);
  for (int64_t rb = r0; rb < r1;) {
    const int64_t rp = rp_cur, rp_end = rp_end_cur;
    const int64_t a0 = __shfl_sync(0xffffffffu, rp, 0);
    int64_t nxt = __shfl_down_sync(0xffffffffu, rp, 1);
    if (lane == 31) nxt = rp_end;
    const bool inr = rb + lane < r1;
    const int64_t len = inr ? nxt - rp : 0;
    const int64_t A = a0 - ((a0 + mis) & 3);  // aligned start (colidx + A is 16-byte aligned)
    // a flat batch: the leading run of rows with <= kLT nonzeros within SPAN positions of A
    const bool ok = inr && len <= kLT && nxt - A <= SPAN;
    const int nrows = __ffs(~__ballot_sync(0xffffffffu, ok)) - 1;  // leading ones (-1 if all 32 ok)
    const int nr = nrows < 0 ? 32 : nrows;
    const T vpre = (a.v && inr) ? fpd::ld_once((const T*)a.v + rb + lane) : T(1);
    const int64_t rb_next = rb + (nr == 0 ? 1 : nr);
    rp_cur = RP(rb_next);
    rp_end_cur = RP_END(rb_next);
    const int lo = (int)(a0 - A);  // 0..3
    // the next flat batch's colidx / val (at most SPAN entries from where this one ends) on
    // their way into L2 while this batch is processed
    {
      const int64_t nstart = __shfl_sync(0xffffffffu, nxt, (nr == 0 ? 1 : nr) - 1);
      const int64_t rem = base0 + a.nnz - nstart;  // never past the arrays' end
      if (lane == 0 && rem > 0) {
        const size_t bytes = (size_t)(rem < a.pf ? rem : a.pf) * 4;
        fpd::prefetch_l2(colidx + nstart, bytes);
        fpd::prefetch_l2(val + nstart, bytes * (sizeof(T) / 4));
      }
    }

    if (nr == 0) {
      // ---- row rb is long: warp-per-row, SPAN positions per step with every load of a step in
      // flight together; the first step stays in registers for the scatter, the rest is re-read
      // (just read, so L2-resident: the paper's "likely a cache hit")
      const int64_t L = __shfl_sync(0xffffffffu, len, 0);
      const int64_t endA = L + lo;  // end relative to A (may exceed 2^31 only for n > 2^31)
      const int hi0 = (int)(endA < SPAN ? endA : SPAN);
      int cc[NT][4];
      T xv[NT][4];
      unsigned act[NT];
#pragma unroll
      for (int t = 0; t < NT; ++t) act[t] = LOAD4(A, 128 * t + 4 * lane, lo, hi0, cc[t], xv[t]);
      T acc = T(0);
      if constexpr (YM != 0) {
#pragma unroll
        for (int t = 0; t < NT; ++t)
#pragma unroll
          for (int e = 0; e < 4; ++e) acc = fmaf(xv[t][e], Y(cc[t][e]), acc);
        for (int64_t s0 = SPAN; s0 < endA; s0 += SPAN) {
          const int64_t As = A + s0;
          const int his = (int)(endA - s0 < SPAN ? endA - s0 : SPAN);
#pragma unroll
          for (int t = 0; t < NT; ++t) {
            int c2[4];
            T x2[4];
            LOAD4(As, 128 * t + 4 * lane, 0, his, c2, x2);
#pragma unroll
            for (int e = 0; e < 4; ++e) acc = fmaf(x2[e], Y(c2[e]), acc);
          }
        }
        acc = fpd::vector_allreduce<32>(acc);
      }
      const T vr = __shfl_sync(0xffffffffu, vpre, 0);
      const T q = (YM != 0 ? acc * vr : vr) * alpha;
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        T tv[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) tv[e] = xv[t][e] * q;
        EMIT4(cc[t], tv, act[t]);
      }
      // the tail beyond the first SPAN positions is re-read for the scatter: a long row's dot
      // takes longer than L2 keeps it, so the whole tail is first requested into L2 at once
      // (its DRAM latency overlapped), then streamed two super-tiles per step
      if (endA > SPAN) {
        for (int64_t o = SPAN + (int64_t)lane * 1024; o < endA; o += 32 * 1024) {
          const int64_t cnt = endA - o < 1024 ? endA - o : 1024;
          fpd::prefetch_l2(colidx + A + o, (size_t)cnt * 4);
          fpd::prefetch_l2(val + A + o, (size_t)cnt * sizeof(T));
        }
      }
      for (int64_t s0 = SPAN; s0 < endA; s0 += 256) {
        int c2[2][4];
        T x2[2][4];
        unsigned a2[2];
#pragma unroll
        for (int t = 0; t < 2; ++t) {
          const int64_t st = s0 + 128 * t;
          const int his = st < endA ? (int)(endA - st < 128 ? endA - st : 128) : 0;
          a2[t] = LOAD4(A + st, 4 * lane, 0, his, c2[t], x2[t]);
        }
#pragma unroll
        for (int t = 0; t < 2; ++t) {
          T tv[4];
#pragma unroll
          for (int e = 0; e < 4; ++e) tv[e] = x2[t][e] * q;
          EMIT4(c2[t], tv, a2[t]);
        }
      }
      rb = rb_next;
      continue;
    }

    // ---- flat batch of rows [rb, rb + nr) within positions [A, A + SPAN)
    const int hi = (int)(__shfl_sync(0xffffffffu, nxt, nr - 1) - A);
    const bool ne = lane < nr && len > 0;
    const unsigned nem = __ballot_sync(0xffffffffu, ne);
    const int rel = (int)(rp - A);
    if (lane < SPAN / 32) hmw[warp][lane] = 0u;
    __syncwarp();
    if (ne) {
      atomicOr(&hmw[warp][rel >> 5], 1u << (rel & 31));
      cmap[warp][__popc(nem & lt)] = (unsigned char)lane;
    }
    int cc[NT][4];
    T xv[NT][4];
    unsigned act[NT];
#pragma unroll
    for (int t = 0; t < NT; ++t) act[t] = LOAD4(A, 128 * t + 4 * lane, lo, hi, cc[t], xv[t]);
    rs[warp][lane] = T(0);
    __syncwarp();
    // head bits of this lane's 4 positions per super-tile, and the compressed row index of the
    // lane's first position (heads strictly before it, minus one)
    const unsigned hword = lane < SPAN / 32 ? hmw[warp][lane] : 0u;
    int pre = __popc(hword);
#pragma unroll
    for (int d = 1; d < SPAN / 32; d <<= 1) {
      const int t2 = __shfl_up_sync(0xffffffffu, pre, d);
      if (lane >= d) pre += t2;
    }
    pre -= __popc(hword);  // exclusive prefix of head counts over the mask words
    unsigned hb[NT];
    int rbase[NT];
#pragma unroll
    for (int t = 0; t < NT; ++t) {
      const int wi = 4 * t + (lane >> 3);
      const unsigned hw = __shfl_sync(0xffffffffu, hword, wi);
      const int sh = (lane & 7) * 4;
      hb[t] = (hw >> sh) & 0xFu;
      rbase[t] = __shfl_sync(0xffffffffu, pre, wi) + __popc(hw & ((1u << sh) - 1u)) - 1;
    }
    if constexpr (YM != 0) {
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        T sv[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) sv[e] = xv[t][e] * Y(cc[t][e]);  // Eq. (2) products
        // in-lane: P = sum before the first head, complete segments flushed, the last one kept
        T sum = T(0), P = T(0);
        int rid = rbase[t];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          if ((hb[t] >> e) & 1u) {
            if (rid == rbase[t]) P = sum;
            else rs[warp][rid] += sum;  // a row entirely inside this lane
            sum = T(0);
            ++rid;
          }
          sum += sv[e];
        }
        if (!hb[t]) P = sum;
        // across lanes: R_l = P_l + ... + P_h, h = the first lane >= l holding a head
        const unsigned H = __ballot_sync(0xffffffffu, hb[t] != 0u);
        const unsigned hl = H >> lane;
        const int dist = hl ? __ffs(hl) : 32 - lane;
        T r = P;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const T t2 = __shfl_down_sync(0xffffffffu, r, d);
          if (d < dist) r += t2;
        }
        T rn = __shfl_down_sync(0xffffffffu, r, 1);
        if (lane == 31) rn = T(0);  // continues in the next super-tile: its lane 0 adds it
        if (hb[t]) rs[warp][rid] += sum + rn;           // the lane's last row: its suffix + what follows
        if (lane == 0 && !(hb[t] & 1u) && rbase[t] >= 0)  // the row running in from the previous tile
          rs[warp][rbase[t]] += r;
        __syncwarp();
      }
    }
    // lane k owns the k-th non-empty row of the batch: q = alpha v p
    T q = T(0);
    {
      const int nne = __popc(nem);
      const int src = lane < nne ? cmap[warp][lane] : 0;
      const T vr = __shfl_sync(0xffffffffu, vpre, src);
      if (lane < nne) q = (YM != 0 ? rs[warp][lane] * vr : vr) * alpha;
    }
#pragma unroll
    for (int t = 0; t < NT; ++t) {
      if (128 * t >= hi) break;
      int rid = rbase[t];
      T tv[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        rid += (hb[t] >> e) & 1u;
        tv[e] = xv[t][e] * __shfl_sync(0xffffffffu, q, rid & 31);
      }
      EMIT4(cc[t], tv, act[t]);
    }
    rb = rb_next;
  }
  if constexpr (SINK == SINK_BINS) {
    if (lane == 0) {
      a.wsplit[3 * gw] = nz0;
      a.wsplit[3 * gw + 1] = nz0 + up;  // == nz0 + dn: every slot of [nz0, nz1) written
      a.wsplit[3 * gw + 2] = nz1;
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) tmax = fmaxf(tmax, __shfl_xor_sync(0xffffffffu, tmax, d));
    if (lane == 0 && tmax > 0.f) atomicMax(a.gmax, __float_as_uint(tmax));
  } else {
    (void)tmax;
    (void)up;
    (void)dn;
    __syncthreads();
    fpd::fix_to_double<BS>(FA, a.n);
    __syncthreads();
    fpd::grid_finalize<T, double>(FA.sp, a.n, a.acc, a.counter, 1.0, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z,
                                  a.accumulate);
  }
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
  // an infinite term (gmax = +Inf) leaves no finite scale: then every term goes to the spill
  const bool allspill = *a.gmax == 0x7f800000u;
  const int ex = allspill ? 0 : 26 - bin_exponent(a.gmax);
  const bool fscale = ex >= -125 && ex <= 127;  // 2^ex representable as float (the usual case)
  const float sf = fscale ? ldexpf(1.f, ex) : 0.f;
  const double sd = ldexp(1.0, ex);
  const int64_t col0 = (int64_t)b * a.bw;
  // one message: fixed point, native returning shared atomic, wrap carried into hi[]; FS =
  // the float scale is usable (decided once per call, so the two paths are separate loops)
  auto ADD = [&](int cl, float t, auto fs) {
    if (!(fabsf(t) <= 3.402823466e38f)) {  // Inf / NaN: IEEE propagation through the spill
      atomicAdd(a.spill + col0 + cl, t);
      return;
    }
    int qi;
    if constexpr (decltype(fs)::value) qi = __float2int_rn(t * sf);
    else qi = __double2int_rn((double)t * sd);
    const int old = atomicAdd(sw + cl, qi);  // native ATOMS.ADD (with return)
    const unsigned nw = (unsigned)old + (unsigned)qi;
    if ((int)(((unsigned)old ^ nw) & ((unsigned)qi ^ nw)) < 0)  // signed wrap: carry into hi
      atomicAdd(a.hi + col0 + cl, qi > 0 ? 1 : -1);
  };
  // each lane takes 8 consecutive messages per step (a 16-byte column load and a 32-byte value
  // load at 8-aligned indices), two steps in flight; which of the 8 are inside the warp's
  // block-b range is one 8-bit mask per step
  auto RUN = [&](auto fs) {
    for (int64_t p = pw0 + warp; p < pw1; p += kConsBS / 32) {
      const int64_t lo = a.wsplit[3 * p + b], hi = a.wsplit[3 * p + b + 1];
      const int64_t gs = lo & ~int64_t(7);
      const int nmsg = (int)(hi - gs);  // < 2^31 (a producer warp's range)
      const int skip = (int)(lo - gs);  // 0..7
      for (int o0 = 8 * lane; o0 < nmsg; o0 += 2 * 256) {
        uint4 cv[2];
        float tv[2][8];
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int o = o0 + u * 256;
          if (o < nmsg) {
            asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                : "=r"(cv[u].x), "=r"(cv[u].y), "=r"(cv[u].z), "=r"(cv[u].w)
                : "l"(a.bcol + gs + o));
            asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                : "=f"(tv[u][0]), "=f"(tv[u][1]), "=f"(tv[u][2]), "=f"(tv[u][3]), "=f"(tv[u][4]),
                  "=f"(tv[u][5]), "=f"(tv[u][6]), "=f"(tv[u][7])
                : "l"(a.bval + gs + o));
          }
        }
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int o = o0 + u * 256;
          if (o >= nmsg) continue;
          // entries e with skip <= o + e < nmsg
          const int lo_e = skip - o, hi_e = nmsg - o;
          const unsigned msk = (0xFFu << (lo_e > 0 ? lo_e : 0)) & (hi_e >= 8 ? 0xFFu : ((1u << hi_e) - 1u));
          const uint32_t cw[4] = {cv[u].x, cv[u].y, cv[u].z, cv[u].w};
#pragma unroll
          for (int e = 0; e < 8; ++e)
            if ((msk >> e) & 1u) ADD((int)((cw[e >> 1] >> (16 * (e & 1))) & 0xffffu), tv[u][e], fs);
        }
      }
    }
  };
  if (allspill) {
    // an infinite term: no finite scale, every message through the spill (IEEE semantics)
    for (int64_t p = pw0 + warp; p < pw1; p += kConsBS / 32) {
      const int64_t lo = a.wsplit[3 * p + b], hi = a.wsplit[3 * p + b + 1];
      for (int64_t g = lo + lane; g < hi; g += 32) atomicAdd(a.spill + col0 + a.bcol[g], a.bval[g]);
    }
  } else if (fscale) {
    RUN(std::true_type{});
  } else {
    RUN(std::false_type{});
  }
  __syncthreads();
  int32_t* dst = a.part + (int64_t)blockIdx.x * a.bw;
  for (int j = threadIdx.x; j < a.bw; j += kConsBS) dst[j] = sw[j];
}

template <typename T>
__global__ void k_bin_finalize(int64_t n, int bw, int nbin, int ncons, const int32_t* __restrict__ part,
                               int32_t* __restrict__ hi, float* __restrict__ spill, const unsigned* __restrict__ gmax,
                               const T* __restrict__ z, double beta, int add_beta_z, int accumulate, T* w) {
  const double quantum = *gmax == 0x7f800000u ? 0.0 : ldexp(1.0, bin_exponent(gmax) - 26);
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

// L2 prefetch distance of the flat-4 kernels (nonzeros); FP_BIN_PF overrides (measurement)
int prefetch_span() {
  static const int pf = [] {
    const char* e = std::getenv("FP_BIN_PF");
    const int v = e ? std::atoi(e) : 0;
    return v > 0 ? v : 128 * kNT;
  }();
  return pf;
}

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
  const int mis = (int)(((uintptr_t)a.colidx >> 2) & 3);
  FP_REQUIRE(((uintptr_t)a.colidx & 3) == 0 && ((uintptr_t)a.val & 3) == 0 &&
                 (int)(((uintptr_t)a.val >> 2) & 3) == mis,
             FP_ERR_UNSUPPORTED, "fp_csr: variant %d needs colidx and val with the same 16-byte misalignment",
             L.variant);
  const int sms = device_info(current_device()).sm_count;
  const int grid = L.grid > 0 ? L.grid : sms;
  FP_REQUIRE(a.nnz / ((int64_t)grid * (kProdBS / 32)) + a.n < INT32_MAX, FP_ERR_UNSUPPORTED,
             "fp_csr: variant %d: too many nonzeros per producer warp (grid %d)", L.variant, grid);
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
  k.val = a.val;
  k.y = a.y;
  k.v = a.v;
  k.alpha = a.alpha;
  // y prefix: what the opt-in shared memory leaves beside the producer's static arrays
  (void)y_prefix;
  const void* f = a.y ? (nbin == 2 ? (const void*)k_flat4<float, 1, 2, SINK_BINS, kProdBS>
                                   : (const void*)k_flat4<float, 1, 1, SINK_BINS, kProdBS>)
                      : (nbin == 2 ? (const void*)k_flat4<float, 0, 2, SINK_BINS, kProdBS>
                                   : (const void*)k_flat4<float, 0, 1, SINK_BINS, kProdBS>);
  {
    cudaFuncAttributes fa{};
    FP_CUDA(cudaFuncGetAttributes(&fa, f));
    const int64_t room = ((int64_t)device_info(current_device()).smem_optin_per_block - (int64_t)fa.sharedSizeBytes -
                          256) / 4 / 4 * 4;
    k.ny_s = a.y ? (int)std::min<int64_t>(a.n, room) : 0;
  }
  k.bw = nbin == 2 ? bw : INT32_MAX;
  k.mis = mis;
  k.pf = prefetch_span();
  k.bcol = (uint16_t*)take((size_t)a.nnz * 2);
  k.bval = (float*)take((size_t)a.nnz * 4);
  k.wsplit = (int64_t*)take((size_t)pw * 24);
  int32_t* part = (int32_t*)take((size_t)ncons * bw * 4);
  k.gmax = (unsigned*)take(16);
  int32_t* hi = (int32_t*)zbase;
  float* spill = (float*)(zbase + al((size_t)a.n * 4));
  FP_CUDA(cudaMemsetAsync(k.gmax, 0, 16, s));
  set_max_dynamic_smem(f);
  const size_t psmem = (size_t)k.ny_s * 4;
  void* args[] = {&k};
  FP_CUDA(cudaLaunchKernel(f, dim3(grid), dim3(kProdBS), args, psmem, s));
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

// ---- variant 18: the flat-4 kernel with the fixed-point CTA partial (n fits shared memory)
constexpr int kFixBS = 256;

template <typename T, int YM>
const void* flat4_fixed_fn() {  // fp64 keeps ~80 registers (3 CTAs of 256 per SM), fp32 64 (4)
  return (const void*)k_flat4<T, YM, 1, SINK_FIX, kFixBS, sizeof(T) == 8 ? 3 : 4>;
}
const void* flat4_fixed_pick(fp_dtype dt, bool has_y) {
  if (dt == FP_F64) return has_y ? flat4_fixed_fn<double, 1>() : flat4_fixed_fn<double, 0>();
  return has_y ? flat4_fixed_fn<float, 1>() : flat4_fixed_fn<float, 0>();
}

size_t flat4_fixed_smem(int64_t n, fp_dtype dt, bool has_y) {
  return (size_t)(has_y ? fix_y_bytes(n, (int)dtype_size(dt)) : 0) + (size_t)n * 16;
}

int flat4_fixed_blocks_per_sm(int64_t n, fp_dtype dt, bool has_y) {
  const void* f = flat4_fixed_pick(dt, has_y);
  set_max_dynamic_smem(f);
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, f, kFixBS, flat4_fixed_smem(n, dt, has_y));
  return occ;
}

fp_status launch_flat4_fixed(const PatternArgs& a, const fp_launch& L, cudaStream_t s) {
  FP_REQUIRE(a.epi_kind == 0 && !a.row_out, FP_ERR_UNSUPPORTED, "fp_csr: variant %d has no row epilogue",
             L.variant);
  const bool has_y = a.y != nullptr;
  const size_t smem = flat4_fixed_smem(a.n, a.dtype, has_y);
  const void* f = flat4_fixed_pick(a.dtype, has_y);
  cudaFuncAttributes fa{};
  FP_CUDA(cudaFuncGetAttributes(&fa, f));
  FP_REQUIRE(smem + fa.sharedSizeBytes <= (size_t)device_info(current_device()).smem_optin_per_block,
             FP_ERR_UNSUPPORTED, "fp_csr: variant %d needs n small enough for y + partial w in shared memory",
             L.variant);
  const size_t es = dtype_size(a.dtype);
  const int mis = (int)(((uintptr_t)a.colidx >> 2) & 3);
  FP_REQUIRE(((uintptr_t)a.colidx & 3) == 0 && ((uintptr_t)a.val % es) == 0 &&
                 (int)(((uintptr_t)a.val / es) & 3) == mis,
             FP_ERR_UNSUPPORTED, "fp_csr: variant %d needs colidx and val aligned alike (4-entry groups)",
             L.variant);
  const int sms = device_info(current_device()).sm_count;
  int grid = L.grid;
  if (grid <= 0) {
    const int occ = flat4_fixed_blocks_per_sm(a.n, a.dtype, has_y);
    grid = sms * (occ > 0 ? occ : 1);
  }
  FP_REQUIRE(a.nnz / ((int64_t)grid * (kFixBS / 32)) + a.n < INT32_MAX, FP_ERR_UNSUPPORTED,
             "fp_csr: variant %d: too many nonzeros per warp (grid %d)", L.variant, grid);
  Workspace* ws = workspace(s, (size_t)a.n, 0);
  if (!ws) return FP_ERR_NOMEM;
  BinPArgs k{};
  k.m = a.m;
  k.nnz = a.nnz;
  k.rowptr = a.rowptr;
  k.colidx = a.colidx;
  k.val = a.val;
  k.y = a.y;
  k.v = a.v;
  k.alpha = a.alpha;
  k.ny_s = has_y ? (int)a.n : 0;
  k.bw = INT32_MAX;
  k.mis = mis;
  k.pf = prefetch_span();
  k.n = a.n;
  k.acc = ws->acc;
  k.counter = ws->counters;
  k.z = a.z;
  k.beta = a.beta;
  k.w = a.w;
  k.add_beta_z = a.add_beta_z ? 1 : 0;
  k.accumulate = a.accumulate ? 1 : 0;
  set_max_dynamic_smem(f);
  void* args[] = {&k};
  FP_CUDA(cudaLaunchKernel(f, dim3(grid), dim3(kFixBS), args, smem, s));
  return FP_OK;
}

// register count of the producer (plan reports)
int binned_producer_regs(bool has_y) {
  cudaFuncAttributes fa{};
  if (cudaFuncGetAttributes(&fa, has_y ? (const void*)k_flat4<float, 1, 2, SINK_BINS, kProdBS>
                                      : (const void*)k_flat4<float, 0, 2, SINK_BINS, kProdBS>) !=
      cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return fa.numRegs;
}

}  // namespace fp
