// csr_flat.cuh -- "flat" CSR kernel for short rows (included by csr_kernels.cuh).
//
// The CSR-vector layout of Algorithm 2 (VS lanes per row) leaves lanes idle when rows
// are short and ragged (C3: Binomial(1000, 0.01) rows -> ~60 % of the lanes of a VS = 8 warp
// instruction carry a nonzero).  On sm_100a the scatter into the on-chip partial w costs per
// instruction, not per useful lane, so idle lanes are paid for.  This kernel keeps the paper's
// fusion (row dot -> v[r] scale -> scatter of the same row from registers) but maps the warp's
// lanes onto CONSECUTIVE NONZEROS instead of onto rows:
//   - a batch = up to 32 consecutive rows whose nonzeros fit in NB tiles of 32 (one coalesced
//     load per tile, every lane busy); longer rows take a warp-per-row path;
//   - each lane finds its nonzero's row by a 5-step shuffle binary search of the batch's
//     rowptr (held one row per lane);
//   - row dots: y gathered from shared memory, segmented shuffle reduction inside each tile,
//     segment heads add into a per-warp 32-entry row-sum scratch (heads of one tile have
//     distinct rows, so plain load-add-store suffices);
//   - lane i then owns row i: q_i = v_i p_i (or the row epilogue), and every nonzero fetches
//     its row's q by shuffle and scatters x q into the partial w (shared-memory atomicAdd in
//     MODE_SHARED, red.global in MODE_L2) -- again with every lane busy.
#pragma once

namespace fp {

template <typename T, int NB, int YM, int MODE, int BS>
__global__ void __launch_bounds__(BS) k_csr_flat(const CsrKArgs a) {
  static_assert(MODE == MODE_SHARED || MODE == MODE_L2 || MODE == MODE_PRIVATE || MODE == MODE_FIXED,
                "flat kernel aggregation mode");
  constexpr int NW = BS / 32;
  constexpr int CAP = 32 * NB;  // nonzeros per batch
  const int64_t* __restrict__ rowptr = a.rowptr;
  const int32_t* __restrict__ colidx = a.colidx;
  const T* __restrict__ val = (const T*)a.val;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t m = a.m, n = a.n;
  constexpr bool HAS_Y = YM != 0;

  // shared memory: [y_s: n (if staged)] [w_s: n (SHARED)] ; static: per-warp row sums
  extern __shared__ __align__(16) unsigned char smem_raw[];
  __shared__ T rsum[NW][32];
  T* y_s = reinterpret_cast<T*>(smem_raw);
  // y entries staged in shared memory: all of y on the smem-partial paths; on the L2 path the
  // leading a.y_in_smem columns (all of y when it fits, a prefix for the 1024-thread variant 16)
  // (a partial prefix only in the 1024-thread instantiation: the extra branch costs registers)
  constexpr bool PARTIAL_Y = BS == 1024 && MODE == MODE_L2;
  const int64_t ny_s = !HAS_Y ? 0
                              : (MODE != MODE_L2 ? n
                                                 : (a.y_in_smem >= n ? n : (PARTIAL_Y ? (int64_t)a.y_in_smem : 0)));
  const bool ysm = ny_s == n && HAS_Y;
  T* w_s = y_s + (ysm ? n : 0);
  T* w_mine = MODE == MODE_PRIVATE ? w_s + (int64_t)warp * n : w_s;
  __shared__ int fix_e;
  const fpd::FixAcc FA = fix_layout(smem_raw + (ysm ? fix_y_bytes(n, sizeof(T)) : 0), n, &fix_e);
  fpd::FixScale FS;
  {
    const int64_t nw_copies = MODE == MODE_PRIVATE ? NW : (MODE == MODE_SHARED ? 1 : 0);
    for (int64_t j = threadIdx.x; j < nw_copies * n; j += BS) w_s[j] = T(0);
    if constexpr (MODE == MODE_FIXED) fpd::fix_init<BS>(FA, n);
    for (int64_t j = threadIdx.x; j < ny_s; j += BS) y_s[j] = y[j];
    __syncthreads();
  }
  const T qscale = MODE == MODE_L2 ? (T)a.alpha : T(1);
  auto Y = [&](int c) -> T {
    if constexpr (PARTIAL_Y) return ysm ? y_s[c] : (c < ny_s ? y_s[c] : fpd::ld_keep(y + c));
    else return ysm ? y_s[c] : fpd::ld_keep(y + c);
  };
  T* const wl2 = l2_target<T>(a);
  auto W_ADD = [&](int c, T val_) {
    if constexpr (MODE == MODE_SHARED) atomicAdd(w_s + c, val_);
    else if constexpr (MODE == MODE_FIXED) fpd::fix_add(FA, FS, c, val_);
    else fpd::red_add(wl2 + c, val_);
  };
  // MODE_FIXED: until the CTA's scale is set, every warp offers its batch's largest |term|
  auto FIX_SET = [&](T term, bool act) {
    if constexpr (MODE == MODE_FIXED) {
      if (FS.e == fpd::kFixUnset) {
        double at, tm = 0.0;
        if (act && fpd::fix_finite_abs((double)term, at)) tm = at;
        fpd::fix_try_set(FA, FS, tm);
      }
    }
  };
  // one row's entries spread over the active lanes (long-row path): distinct columns when the
  // row is canonical; duplicates (R7) are serialised lane by lane
  auto ROW_ADD = [&](int c, T val_, bool act) {
    if constexpr (MODE == MODE_PRIVATE) {
      const int cn = __shfl_down_sync(0xffffffffu, c, 1);
      const bool nact = __shfl_down_sync(0xffffffffu, (int)act, 1) != 0;
      if (!__any_sync(0xffffffffu, act && nact && lane < 31 && cn <= c)) {
        if (act) w_mine[c] += val_;
      } else {
        for (int l = 0; l < 32; ++l) {
          if (act && lane == l) w_mine[c] += val_;
          __syncwarp();
        }
      }
      __syncwarp();
    } else {
      if (act) W_ADD(c, val_);
    }
  };

  const int64_t gw = (int64_t)blockIdx.x * NW + warp, tw = (int64_t)gridDim.x * NW;
  const int64_t total = a.nnz + kRowCost * m;
  const int64_t r0 = warp_search_rows(rowptr, m, (total * gw) / tw, lane);
  const int64_t r1 = warp_search_rows(rowptr, m, (total * (gw + 1)) / tw, lane);
  double loss_acc = 0.0;

  // rowptr of the batch starting at row b: lane i holds rowptr[b + i], clamped at r1
  auto RP = [&](int64_t b) -> int64_t { return __ldg(rowptr + (b + lane < r1 ? b + lane : r1)); };
  auto RP_END = [&](int64_t b) -> int64_t { return __ldg(rowptr + (b + 32 < r1 ? b + 32 : r1)); };
  int64_t rp_cur = RP(r0), rp_end_cur = RP_END(r0);
  for (int64_t rb = r0; rb < r1;) {
    // ---- batch rows [rb, rb + nrows): lane i holds rowptr[rb + i] (clamped at r1)
    const int64_t rp = rp_cur;
    const int64_t rp_end = rp_end_cur;
    const int64_t a0 = __shfl_sync(0xffffffffu, rp, 0);
    int64_t nxt = __shfl_down_sync(0xffffffffu, rp, 1);
    if (lane == 31) nxt = rp_end;
    const bool fits = (rb + lane < r1) && (nxt - a0 <= CAP);
    const int nrows = __popc(__ballot_sync(0xffffffffu, fits));  // rowptr monotone: a prefix
    // v of this lane's row, loaded now so its latency overlaps the (col, val) and y loads
    const T vpre = (v && rb + lane < r1) ? fpd::ld_once(v + rb + lane) : T(1);
    // the next batch's rowptr, loaded now: its latency overlaps this batch's work
    const int64_t rb_next = rb + (nrows == 0 ? 1 : nrows);
    rp_cur = RP(rb_next);
    rp_end_cur = RP_END(rb_next);

    if (nrows == 0) {
      // ---- a row longer than CAP: warp-per-row, dot pass then scatter pass (tail re-read)
      const int64_t s0 = a0, L = __shfl_sync(0xffffffffu, nxt, 0) - a0;
      T p = T(0);
      if constexpr (HAS_Y) {
        for (int64_t k = lane; k < L; k += 32) p = fma(__ldg(val + s0 + k), Y(__ldg(colidx + s0 + k)), p);
        p = fpd::vector_allreduce<32>(p);
      }
      const T vr = v ? v[rb] : T(1);
      T q;
      if constexpr (YM == 2) q = fpd::row_epilogue<T>(p, vr, true, rb, lane == 0, a.epi, loss_acc) * qscale;
      else if constexpr (HAS_Y) q = p * vr * qscale;
      else q = vr * qscale;
      for (int64_t kb = 0; kb < L; kb += 32) {  // warp-uniform trip count
        const int64_t k = kb + lane;
        const bool act = k < L;
        const T term = act ? __ldg(val + s0 + k) * q : T(0);
        FIX_SET(term, act);
        ROW_ADD(act ? __ldg(colidx + s0 + k) : 0, term, act);
      }
      rb = rb_next;
      continue;
    }
    const int64_t cnt = __shfl_sync(0xffffffffu, nxt, nrows - 1) - a0;   // nonzeros in the batch
    const int rel = lane < nrows ? (int)(rp - a0) : 0x7fffffff;          // row start, batch-relative

    // ---- first touch: NB coalesced tiles of (col, val), every lane busy
    int cc[NB], rid[NB];
    T xv[NB];
#pragma unroll
    for (int j = 0; j < NB; ++j) {
      const int pos = j * 32 + lane;
      const bool act = pos < cnt;
      cc[j] = act ? fpd::ld_once(colidx + a0 + pos) : 0;
      xv[j] = act ? fpd::ld_once(val + a0 + pos) : T(0);
      // row of this nonzero: largest i < nrows with rel_i <= pos (5-step shuffle search)
      int lo = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const int cand = lo + step;
        const int rc = __shfl_sync(0xffffffffu, rel, cand & 31);
        if (cand < nrows && rc <= pos) lo = cand;
      }
      rid[j] = lo;
    }

    T q = T(0);  // lane i: q of row rb + i
    if constexpr (HAS_Y) {
      // fp32: all NB gathers of y issued before the first use (their latencies overlap; 8 more
      // registers, still 64).  fp64: gathered inside the reduction loop -- hoisting costs 16
      // registers there (64 -> 91, half the resident CTAs) and made K1 slower (45.7 -> 59 ms).
      constexpr bool HOIST = sizeof(T) == 4;
      T yv[HOIST ? NB : 1];
      if constexpr (HOIST) {
        if (ysm) {
#pragma unroll
          for (int j = 0; j < NB; ++j) yv[j] = y_s[cc[j]];
        } else if (PARTIAL_Y && ny_s > 0) {
#pragma unroll
          for (int j = 0; j < NB; ++j) yv[j] = cc[j] < ny_s ? y_s[cc[j]] : fpd::ld_keep(y + cc[j]);
        } else {
#pragma unroll
          for (int j = 0; j < NB; ++j) yv[j] = fpd::ld_keep(y + cc[j]);
        }
      }
      rsum[warp][lane] = T(0);
      __syncwarp();
#pragma unroll
      for (int j = 0; j < NB; ++j) {
        const int pos = j * 32 + lane;
        T s;  // Eq. (2) products
        if constexpr (HOIST) s = pos < cnt ? xv[j] * yv[j] : T(0);
        else s = pos < cnt ? xv[j] * Y(cc[j]) : T(0);
        // segmented reduction toward the segment head (lanes of a row are contiguous)
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const T t = __shfl_down_sync(0xffffffffu, s, d);
          const int r2 = __shfl_down_sync(0xffffffffu, rid[j], d);
          if (lane + d < 32 && r2 == rid[j]) s += t;
        }
        const int rprev = __shfl_up_sync(0xffffffffu, rid[j], 1);
        const bool head = pos < cnt && (lane == 0 || rprev != rid[j]);
        if (head) rsum[warp][rid[j]] += s;  // heads of one tile hold distinct rows
        __syncwarp();
      }
      const T p = rsum[warp][lane];
      const int64_t row = rb + lane;
      (void)row;
      const bool ok = lane < nrows;
      const T vr = ok ? vpre : T(0);
      if constexpr (YM == 2) q = fpd::row_epilogue<T>(p, vr, ok, row, ok, a.epi, loss_acc) * qscale;
      else q = ok ? p * vr * qscale : T(0);
    } else {
      q = lane < nrows ? vpre * qscale : T(0);
    }

    // ---- second touch from registers: Eq. (3), every lane busy
    if constexpr (MODE == MODE_FIXED) {
      if (FS.e == fpd::kFixUnset) {
        double tm = 0.0;
#pragma unroll
        for (int j = 0; j < NB; ++j) {
          double at;
          const T qj = __shfl_sync(0xffffffffu, q, rid[j]);
          if (j * 32 + lane < cnt && fpd::fix_finite_abs((double)(xv[j] * qj), at)) tm = fmax(tm, at);
        }
        fpd::fix_try_set(FA, FS, tm);
      }
    }
#pragma unroll
    for (int j = 0; j < NB; ++j) {
      const T qj = __shfl_sync(0xffffffffu, q, rid[j]);
      const bool act = j * 32 + lane < cnt;
      if constexpr (MODE == MODE_PRIVATE) {
        // per-warp private partial, plain load-add-store: one round per row present in the
        // tile (columns of one canonical row are distinct; different rows may collide)
        if (j * 32 >= cnt) break;
        const int last = (int)(cnt - 1 - j * 32) < 31 ? (int)(cnt - 1 - j * 32) : 31;
        const int rf = __shfl_sync(0xffffffffu, rid[j], 0), rl = __shfl_sync(0xffffffffu, rid[j], last);
        const int cn = __shfl_down_sync(0xffffffffu, cc[j], 1);
        const int rn = __shfl_down_sync(0xffffffffu, rid[j], 1);
        const bool dup = act && lane < last && rn == rid[j] && cn <= cc[j];  // non-canonical row (R7)
        const T contrib = xv[j] * qj;
        if (!__any_sync(0xffffffffu, dup)) {
          for (int r = rf; r <= rl; ++r) {
            if (act && rid[j] == r) w_mine[cc[j]] += contrib;
            __syncwarp();
          }
        } else {
          for (int l = 0; l <= last; ++l) {
            if (lane == l) w_mine[cc[j]] += contrib;
            __syncwarp();
          }
        }
      } else {
        if (act) W_ADD(cc[j], xv[j] * qj);
      }
    }
    rb = rb_next;
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
  }
  if constexpr (MODE == MODE_SHARED || MODE == MODE_PRIVATE) {
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

}  // namespace fp
