// csr_stream.cuh -- CSR-vector kernel with the row stream prefetched into shared memory
// (included by csr_kernels.cuh).  Variants 14 (CTA-shared partial w) and 15 (fixed-point
// partial).
//
// Why: k_csr_vector with y and w on chip (C3) stalls on its (col, val) loads -- ncu of the
// chooser's plan: 24 % of all stall samples on the first use of the freshly loaded column
// index, DRAM at 31 % of peak.  A warp issues its row group's loads and consumes them at once,
// so at most one group's bytes are in flight per warp.  Here each warp streams its contiguous
// nonzero range through a two-stage buffer in shared memory with cp.async (LDGSTS, 16-byte
// chunks, no registers held): while the warp works on batch b (RB = 16 rows) from one stage,
// the copies of batch b+1 land in the other; the rowptr and v of batch b+2 / b+1 are loaded
// into registers one batch ahead.  The arithmetic is the paper's Alg. 2 exactly as
// in k_csr_vector: VS lanes per row, the row dot reduced inside the vector and multiplied by
// v[r] (l.10-12), the same entries -- now from registers filled out of the stage -- scattered
// into the partial w (l.13-14), CTA partials aggregated by grid_finalize (l.16-18).
#pragma once

namespace fp {

constexpr int kStreamRB = 16;    // rows per batch
constexpr int kStreamCap = 192;  // nonzeros per stage (entries beyond it are read from global)

__device__ __forceinline__ void cp_async16(void* dst, const void* src, unsigned src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(fpd::smem_u32(dst)), "l"(src),
               "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// bytes of one warp's two stages: per stage kStreamCap int32 + kStreamCap T
template <typename T>
__host__ __device__ constexpr int stream_stage_bytes() {
  return kStreamCap * 4 + kStreamCap * (int)sizeof(T);
}

template <typename T, int VS, int K, int YM, int MODE, int BS>
__global__ void __launch_bounds__(BS) k_csr_stream(const CsrKArgs a) {
  static_assert(MODE == MODE_SHARED || MODE == MODE_FIXED, "stream kernel aggregation mode");
  static_assert(YM != 2, "row epilogues run on k_csr_vector");
  static_assert(kStreamCap % 4 == 0, "stage holds whole 16-byte column chunks");
  constexpr int VPW = 32 / VS;
  constexpr int NW = BS / 32;
  constexpr int RB = kStreamRB;
  constexpr int NG = RB / VPW;  // row groups per batch
  static_assert(RB % VPW == 0 && RB < 32, "batch = whole row groups, rowptr of RB+1 rows in one warp");
  constexpr int CAP = kStreamCap;
  const int64_t* __restrict__ rowptr = a.rowptr;
  const int32_t* __restrict__ colidx = a.colidx;
  const T* __restrict__ val = (const T*)a.val;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int lid = lane & (VS - 1), vid = lane / VS;
  const int64_t m = a.m, n = a.n, nnz = a.nnz;
  constexpr bool HAS_Y = YM != 0;

  // shared memory: [y_s: n (16-byte padded)] [partial: n T (SHARED) | fixed layout] [stages]
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* y_s = reinterpret_cast<T*>(smem_raw);
  const int64_t yb = HAS_Y ? fix_y_bytes(n, sizeof(T)) : 0;
  T* w_s = reinterpret_cast<T*>(smem_raw + yb);
  __shared__ int fix_e;
  const fpd::FixAcc FA = fix_layout(smem_raw + yb, n, &fix_e);
  fpd::FixScale FS;
  const int64_t pb = MODE == MODE_FIXED ? n * 16 : (n * (int64_t)sizeof(T) + 15) / 16 * 16;
  unsigned char* stages = smem_raw + yb + pb + (int64_t)warp * 2 * stream_stage_bytes<T>();
  {
    if constexpr (MODE == MODE_SHARED)
      for (int64_t j = threadIdx.x; j < n; j += BS) w_s[j] = T(0);
    else
      fpd::fix_init<BS>(FA, n);
    if constexpr (HAS_Y)
      for (int64_t j = threadIdx.x; j < n; j += BS) y_s[j] = y[j];
    __syncthreads();
  }
  auto W_ADD = [&](int c, T val_, bool act) {
    if constexpr (MODE == MODE_SHARED) {
      if (act) atomicAdd(w_s + c, val_);
    } else {
      if (act) fpd::fix_add(FA, FS, c, val_);
    }
  };

  const int64_t gw = (int64_t)blockIdx.x * NW + warp, tw = (int64_t)gridDim.x * NW;
  const int64_t total = nnz + kRowCost * m;
  const int64_t r0 = warp_search_rows(rowptr, m, (total * gw) / tw, lane);
  const int64_t r1 = warp_search_rows(rowptr, m, (total * (gw + 1)) / tw, lane);

  // lane i <= RB: rowptr[b + i] (clamped at r1); lane i < RB: v[b + i]
  auto RPL = [&](int64_t b) -> int64_t {
    const int64_t r = b + lane < r1 ? b + lane : r1;
    return lane <= RB ? __ldg(rowptr + r) : 0;
  };
  auto VL = [&](int64_t b) -> T { return (v && lane < RB && b + lane < r1) ? fpd::ld_once(v + b + lane) : T(1); };
  // issue the copies of the batch whose rowptr is rp into stage st; returns (base, end) of the
  // entries that are in the stage: [base, cend) with base = rowptr[b] rounded down to 4
  auto ISSUE = [&](int64_t rp, int64_t b, int st, int64_t& base, int64_t& cend) {
    const int nr = (int)((r1 - b) < RB ? (r1 - b) : RB);
    const int64_t s0 = __shfl_sync(0xffffffffu, rp, 0), s1 = __shfl_sync(0xffffffffu, rp, nr);
    base = s0 & ~(int64_t)3;
    cend = s1 < base + CAP ? s1 : base + CAP;
    unsigned char* sc = stages + st * stream_stage_bytes<T>();
    unsigned char* sv = sc + CAP * 4;
    const int ncc = (int)((cend - base + 3) >> 2);                               // 16-byte column chunks
    constexpr int EPC = 16 / (int)sizeof(T);                                     // values per chunk
    const int ncv = (int)((cend - base + EPC - 1) / EPC);
    for (int c = lane; c < ncc; c += 32) {
      const int64_t e = base + 4 * c;
      const int64_t rem = (nnz - e) * 4;
      cp_async16(sc + 16 * c, rem > 0 ? colidx + e : colidx, rem >= 16 ? 16u : (rem > 0 ? (unsigned)rem : 0u));
    }
    for (int c = lane; c < ncv; c += 32) {
      const int64_t e = base + (int64_t)EPC * c;
      const int64_t rem = (nnz - e) * (int64_t)sizeof(T);
      cp_async16(sv + 16 * c, rem > 0 ? val + e : val, rem >= 16 ? 16u : (rem > 0 ? (unsigned)rem : 0u));
    }
  };

  if (r0 < r1) {
    int64_t b = r0;
    int64_t rpc = RPL(b);
    T vc = VL(b);
    int64_t base_c, cend_c, base_n = 0, cend_n = 0;
    ISSUE(rpc, b, 0, base_c, cend_c);
    cp_async_commit();
    int64_t bn = b + RB;
    int64_t rpn = bn < r1 ? RPL(bn) : 0;
    T vn = VL(bn);
    int st = 0;
    while (b < r1) {
      if (bn < r1) ISSUE(rpn, bn, st ^ 1, base_n, cend_n);
      cp_async_commit();  // possibly empty: keeps one group per batch
      const int64_t bn2 = bn + RB;
      const int64_t rpn2 = bn2 < r1 ? RPL(bn2) : 0;
      const T vn2 = VL(bn2);
      cp_async_wait1();
      __syncwarp();

      const int32_t* cst = reinterpret_cast<const int32_t*>(stages + st * stream_stage_bytes<T>());
      const T* vst = reinterpret_cast<const T*>(stages + st * stream_stage_bytes<T>() + CAP * 4);
      auto COL = [&](int64_t idx) -> int { return idx < cend_c ? cst[idx - base_c] : __ldg(colidx + idx); };
      auto VAL = [&](int64_t idx) -> T { return idx < cend_c ? vst[idx - base_c] : __ldg(val + idx); };

#pragma unroll 1
      for (int g = 0; g < NG; ++g) {
        const int o = g * VPW + vid;
        const int64_t row = b + o;
        const bool ok = row < r1;
        const int64_t s0 = __shfl_sync(0xffffffffu, rpc, o);
        const int64_t s1 = __shfl_sync(0xffffffffu, rpc, o + 1);
        const T vr0 = __shfl_sync(0xffffffffu, vc, o);
        if (!__any_sync(0xffffffffu, ok)) break;
        const int64_t start = ok ? s0 : 0, len = ok ? s1 - s0 : 0;
        const T vr = ok ? vr0 : T(0);
        const bool any_long = __any_sync(0xffffffffu, len > VS * K);

        int cc[K];
        T xv[K];
#pragma unroll
        for (int k = 0; k < K; ++k) {
          const int64_t idx = lid + k * VS;
          if (idx < len) {
            cc[k] = COL(start + idx);
            xv[k] = VAL(start + idx);
          } else {
            cc[k] = 0;
            xv[k] = T(0);
          }
        }
        int64_t lmax = 0;
        if (any_long) {
          lmax = len;
#pragma unroll
          for (int off = 16; off > 0; off >>= 1) {
            const int64_t t = __shfl_xor_sync(0xffffffffu, lmax, off);
            lmax = t > lmax ? t : lmax;
          }
        }
        T q;
        if constexpr (HAS_Y) {
          T yv[K];
#pragma unroll
          for (int k = 0; k < K; ++k) yv[k] = y_s[cc[k]];
          T p = T(0);
#pragma unroll
          for (int k = 0; k < K; ++k)
            if (lid + k * VS < len) p = fma(xv[k], yv[k], p);
          if (any_long)
            for (int64_t seg = VS * K; seg < lmax; seg += VS * K)
#pragma unroll
              for (int k = 0; k < K; ++k) {
                const int64_t idx = seg + lid + k * VS;
                if (idx < len) p = fma(VAL(start + idx), y_s[COL(start + idx)], p);
              }
          q = fpd::vector_allreduce<VS>(p) * vr;
        } else {
          q = vr;
        }
        if constexpr (MODE == MODE_FIXED) {
          if (FS.e == fpd::kFixUnset) {  // warp-uniform, until the CTA's fixed-point scale is set
            double tmax = 0.0;
#pragma unroll
            for (int k = 0; k < K; ++k) {
              double at;
              if (lid + k * VS < len && fpd::fix_finite_abs((double)(xv[k] * q), at)) tmax = fmax(tmax, at);
            }
            fpd::fix_try_set(FA, FS, tmax);
          }
        }
#pragma unroll
        for (int k = 0; k < K; ++k) W_ADD(cc[k], xv[k] * q, lid + k * VS < len);
        if (any_long)
          for (int64_t seg = VS * K; seg < lmax; seg += VS * K)
#pragma unroll
            for (int k = 0; k < K; ++k) {
              const int64_t idx = seg + lid + k * VS;
              const bool act = idx < len;
              int c = 0;
              T x = T(0);
              if (act) {
                c = COL(start + idx);
                x = VAL(start + idx);
              }
              if constexpr (MODE == MODE_FIXED) {
                if (FS.e == fpd::kFixUnset) {
                  double at, tm = 0.0;
                  if (act && fpd::fix_finite_abs((double)(x * q), at)) tm = at;
                  fpd::fix_try_set(FA, FS, tm);
                }
              }
              W_ADD(c, x * q, act);
            }
      }
      __syncwarp();  // every lane is done with stage st before it is refilled
      b = bn;
      bn = bn2;
      rpc = rpn;
      rpn = rpn2;
      vc = vn;
      vn = vn2;
      base_c = base_n;
      cend_c = cend_n;
      st ^= 1;
    }
    cp_async_wait0();
  }

  __syncthreads();
  if constexpr (MODE == MODE_SHARED) {
    fpd::grid_finalize<T, T>(w_s, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z,
                             a.accumulate);
  } else {
    fpd::fix_to_double<BS>(FA, n);
    __syncthreads();
    fpd::grid_finalize<T, double>(FA.sp, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z,
                                  a.accumulate);
  }
}

}  // namespace fp
