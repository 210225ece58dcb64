// csr_owner.cuh -- CSR-vector kernel with OWNER-COMPUTES aggregation of the partial w
// (included by csr_kernels.cuh).
//
// The paper aggregates a CTA's partial w with shared-memory atomics (SD, Alg. 2
// l.13-14).  On sm_100a a shared fp64/fp32 atomicAdd is a CAS loop (ATOMS.CAST.SPIN, ~2 shared
// wavefronts per lane measured), and that scatter bounds C3.  Here every column c has an
// OWNER thread (c mod BS) that keeps w[c] in a register; producers append (c div BS, x*q) to the
// owner's short queue in shared memory -- the slot is claimed with a native 32-bit integer
// shared atomic (ATOMS.ADD) and the queues are laid out [slot][owner] so that draining is
// conflict-free -- and every PI row-group iterations the CTA synchronises and each owner drains
// its queue into its registers.  A full queue spills to a shared fp CAS partial (rare by
// construction: the plan sizes PI so a phase fills the queues to ~half).  Everything else --
// Eq. (4) VS, the row dot, v[r], the second touch from registers -- is the vector kernel.
#pragma once

namespace fp {

constexpr int kOwnerQ = 16;  // queue slots per owner thread

template <typename T, int VS, int K, int RPV, int YM, int NPT, int BS>
__global__ void __launch_bounds__(BS) k_csr_owner(const CsrKArgs a) {
  constexpr int VPW = 32 / VS;
  constexpr int NW = BS / 32;
  constexpr int GROUP = VPW * RPV;
  static_assert(GROUP <= 32, "rowptr batch holds 32 rows");
  static_assert((BS & (BS - 1)) == 0, "owner = c mod BS");
  const int64_t* __restrict__ rowptr = a.rowptr;
  const int32_t* __restrict__ colidx = a.colidx;
  const T* __restrict__ val = (const T*)a.val;
  const T* __restrict__ y = (const T*)a.y;
  const T* __restrict__ v = (const T*)a.v;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int lid = lane & (VS - 1), vid = lane / VS;
  const int64_t m = a.m, n = a.n;
  constexpr bool HAS_Y = YM != 0;
  const int PI = a.phase_iters > 0 ? a.phase_iters : 1;

  // shared: [y_s: n] [w_over: n] [qval: kOwnerQ x BS] [qhi: kOwnerQ x BS bytes] [qcnt: BS]
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* y_s = reinterpret_cast<T*>(smem_raw);
  T* w_over = y_s + (HAS_Y ? n : 0);
  T* qval = w_over + n;
  unsigned char* qhi = reinterpret_cast<unsigned char*>(qval + kOwnerQ * BS);
  int* qcnt = reinterpret_cast<int*>(qhi + kOwnerQ * BS);
  for (int64_t j = tid; j < n; j += BS) {
    w_over[j] = T(0);
    if constexpr (HAS_Y) y_s[j] = y[j];
  }
  qcnt[tid] = 0;
  __syncthreads();
  T acc[NPT];
#pragma unroll
  for (int j = 0; j < NPT; ++j) acc[j] = T(0);

  const T qscale = T(1);  // alpha applied by the finaliser
  auto Y = [&](int c) -> T { return y_s[c]; };
  auto ENQ = [&](int c, T val_, bool act) {
    if (!act) return;
    const int owner = c & (BS - 1);
    const int k = atomicAdd(qcnt + owner, 1);  // native ATOMS.ADD
    if (k < kOwnerQ) {
      qval[k * BS + owner] = val_;
      qhi[k * BS + owner] = (unsigned char)(c / BS);
    } else {
      atomicAdd(w_over + c, val_);  // queue full (rare): shared CAS partial
    }
  };
  auto DRAIN = [&]() {
    const int cnt = qcnt[tid] < kOwnerQ ? qcnt[tid] : kOwnerQ;
    for (int k = 0; k < cnt; ++k) {
      const T x = qval[k * BS + tid];
      const int hi = qhi[k * BS + tid];
#pragma unroll
      for (int j = 0; j < NPT; ++j)
        if (hi == j) acc[j] += x;
    }
    qcnt[tid] = 0;
  };

  const int64_t gw = (int64_t)blockIdx.x * NW + warp, tw = (int64_t)gridDim.x * NW;
  const int64_t total = a.nnz + kRowCost * m;
  const int64_t r0 = warp_search_rows(rowptr, m, (total * gw) / tw, lane);
  const int64_t r1 = warp_search_rows(rowptr, m, (total * (gw + 1)) / tw, lane);
  int64_t bstart = r0;
  int64_t rp = (bstart + lane <= m) ? __ldg(rowptr + bstart + lane) : 0;
  int64_t rp32 = (bstart + 32 <= m) ? __ldg(rowptr + bstart + 32) : 0;
  double loss_acc = 0.0;

  int64_t rb = r0;
  while (true) {
    for (int it = 0; it < PI && rb < r1; ++it, rb += GROUP) {
      if (rb + GROUP > bstart + 32) {
        bstart = rb;
        rp = (bstart + lane <= m) ? __ldg(rowptr + bstart + lane) : 0;
        rp32 = (bstart + 32 <= m) ? __ldg(rowptr + bstart + 32) : 0;
      }
      int64_t start[RPV], len[RPV];
      T vr[RPV];
      bool okr[RPV];
      bool any_long = false;
#pragma unroll
      for (int i = 0; i < RPV; ++i) {
        const int64_t row = rb + i * VPW + vid;
        const int o = (int)(row - bstart);
        const int64_t s0 = __shfl_sync(0xffffffffu, rp, o & 31);
        const int64_t s1n = __shfl_sync(0xffffffffu, rp, (o + 1) & 31);
        const int64_t s1 = (o + 1 == 32) ? rp32 : s1n;
        const bool ok = row < r1;
        okr[i] = ok;
        start[i] = ok ? s0 : 0;
        len[i] = ok ? s1 - s0 : 0;
        vr[i] = ok ? (v ? v[row] : T(1)) : T(0);
        any_long |= len[i] > VS * K;
      }
      any_long = __any_sync(0xffffffffu, any_long);
      int cc[RPV][K];
      T xv[RPV][K];
#pragma unroll
      for (int i = 0; i < RPV; ++i)
#pragma unroll
        for (int k = 0; k < K; ++k) {
          const int64_t idx = lid + k * VS;
          if (idx < len[i]) {
            cc[i][k] = fpd::ld_once(colidx + start[i] + idx);
            xv[i][k] = fpd::ld_once(val + start[i] + idx);
          } else {
            cc[i][k] = 0;
            xv[i][k] = T(0);
          }
        }
      int64_t lmax = 0;
      if (any_long) {
#pragma unroll
        for (int i = 0; i < RPV; ++i) lmax = len[i] > lmax ? len[i] : lmax;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
          const int64_t o = __shfl_xor_sync(0xffffffffu, lmax, off);
          lmax = o > lmax ? o : lmax;
        }
      }
      T q[RPV];
      if constexpr (HAS_Y) {
        T p[RPV];
#pragma unroll
        for (int i = 0; i < RPV; ++i) {
          p[i] = T(0);
#pragma unroll
          for (int k = 0; k < K; ++k)
            if (lid + k * VS < len[i]) p[i] = fma(xv[i][k], Y(cc[i][k]), p[i]);
        }
        if (any_long) {
          for (int64_t seg = VS * K; seg < lmax; seg += VS * K) {
#pragma unroll
            for (int i = 0; i < RPV; ++i)
#pragma unroll
              for (int k = 0; k < K; ++k) {
                const int64_t idx = seg + lid + k * VS;
                if (idx < len[i]) {
                  const int c = __ldg(colidx + start[i] + idx);
                  p[i] = fma(__ldg(val + start[i] + idx), Y(c), p[i]);
                }
              }
          }
        }
#pragma unroll
        for (int i = 0; i < RPV; ++i)
          if constexpr (YM == 2)
            q[i] = fpd::row_epilogue<T>(fpd::vector_allreduce<VS>(p[i]), vr[i], okr[i], rb + i * VPW + vid,
                                        lid == 0, a.epi, loss_acc) *
                   qscale;
          else
            q[i] = fpd::vector_allreduce<VS>(p[i]) * vr[i] * qscale;
      } else {
#pragma unroll
        for (int i = 0; i < RPV; ++i) q[i] = vr[i] * qscale;
      }
#pragma unroll
      for (int i = 0; i < RPV; ++i)
#pragma unroll
        for (int k = 0; k < K; ++k) ENQ(cc[i][k], xv[i][k] * q[i], lid + k * VS < len[i]);
      if (any_long) {
        for (int64_t seg = VS * K; seg < lmax; seg += VS * K) {
#pragma unroll
          for (int i = 0; i < RPV; ++i)
#pragma unroll
            for (int k = 0; k < K; ++k) {
              const int64_t idx = seg + lid + k * VS;
              if (idx < len[i]) ENQ(__ldg(colidx + start[i] + idx), __ldg(val + start[i] + idx) * q[i], true);
            }
        }
      }
    }
    __syncthreads();  // the phase's queues are complete
    DRAIN();
    if (!__syncthreads_or(rb < r1 ? 1 : 0)) break;  // also orders DRAIN before the next phase
  }
  if constexpr (YM == 2) fpd::flush_loss(a.epi, loss_acc);

  // owners' registers + spilled CAS partial -> w_over (the CTA partial) -> grid finalize
#pragma unroll
  for (int j = 0; j < NPT; ++j) {
    const int64_t c = (int64_t)j * BS + tid;
    if (c < n) w_over[c] += acc[j];
  }
  __syncthreads();
  fpd::grid_finalize<T, T>(w_over, n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w, a.add_beta_z,
                           a.accumulate);
}

}  // namespace fp
