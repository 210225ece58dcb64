// csr_colsplit.cuh -- CSR fused kernel for n too wide for one SM's shared memory (C4: n = 1e5,
// y and the partial w 400 KB each in fp32), on a thread-block CLUSTER with the COLUMNS split
// across its CTAs (included by csr_kernels.cuh; FP_VAR_CSR_COLSPLIT).
//
// The paper's large-n path scatters into w in global memory with atomics.  On
// sm_100a that is the bound of C4: a random red.global.add costs ~1.6 SM cycles per lane and
// a random y gather from L2 ~0.7 (tools/microbench/l2_scatter.cu), ~19 ms for 2e9 nonzeros
// against a 2.5 ms HBM roofline, and random DSMEM word access is no better (0.35-0.64 ops /
// clk / SM, tools/microbench/dsmem_ubench.cu).  So the columns are split instead of routed:
//   - column block k = [cb[k], cb[k+1]) belongs to CTA rank k of a cluster of CS CTAs, whose
//     shared memory holds y and a partial w for that block only (random gathers and scatter
//     adds stay local: LDS and shared atomics);
//   - canonical CSR rows are sorted by column, so a row's entries of block k are one
//     contiguous segment; its start offsets (CS-1 int32 per row, soff) are computed once per
//     matrix by the plan (fp_csr_plan_create, amortised like the paper's pre-built transpose,
//     P:413) -- each CTA streams ONLY its segments, so X is still read from HBM exactly once;
//   - every CTA of the cluster works on the same 32-row batch per warp: it reduces its
//     segments' partial dots, sends them to every CTA of the cluster with st.async (credited
//     to a per-warp mbarrier, 2-deep slots), and sums the CS partials in rank order -- all
//     CTAs get the same p[r] (Eq. 2), q = v[r] p (or the row epilogue), and scatter their own
//     segments from registers into their block of w (Eq. 3);
//   - at the end each CTA adds its block of w into the fp64 grid accumulator and the last CTA
//     writes w = alpha acc + beta z (aggregate.cuh).
// Within a warp the segments of 32 rows are flattened: lanes on consecutive segment entries
// (an exclusive scan of segment lengths + a 5-step shuffle search gives each entry's row),
// NB tiles of 32 entries stay in registers; entries beyond them are re-read for the scatter
// (L2 hits, the paper's P:149 "likely a cache hit").
#pragma once
#include <cooperative_groups.h>

namespace fp {

struct SplitKArgs {
  CsrKArgs k;
  const int32_t* soff;
  int cb[kSplitMaxCS + 1];
  int width;
};

template <typename T, int CS, int NB, int YM, int BS>
__global__ void __launch_bounds__(BS, 1) k_csr_colsplit(const SplitKArgs sa) {
  namespace cg = cooperative_groups;
  cg::cluster_group cluster = cg::this_cluster();
  const CsrKArgs& a = sa.k;
  constexpr int NW = BS / 32;
  constexpr int NSLOT = 2;
  constexpr bool HAS_Y = YM != 0;
  constexpr unsigned kXBytes = CS * 32 * (unsigned)sizeof(T);  // one batch of partials, all ranks
  const int64_t* __restrict__ rowptr = a.rowptr;
  const int32_t* __restrict__ colidx = a.colidx;
  const T* __restrict__ val = (const T*)a.val;
  const T* __restrict__ v = (const T*)a.v;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int rank = (int)cluster.block_rank();
  const int c0 = sa.cb[rank], wdt = sa.cb[rank + 1] - c0;
  const int64_t m = a.m;

  extern __shared__ __align__(16) unsigned char smem_raw[];
  T* xslot = reinterpret_cast<T*>(smem_raw);  // [NW][NSLOT][CS][32]
  T* rsum = xslot + NW * NSLOT * CS * 32;     // [NW][32]
  T* y_s = rsum + NW * 32;                    // [width] (HAS_Y)
  T* w_s = y_s + (HAS_Y ? sa.width : 0);      // [width]
  __shared__ uint64_t xbar[NW][NSLOT];

  for (int j = threadIdx.x; j < wdt; j += BS) {
    w_s[j] = T(0);
    if constexpr (HAS_Y) y_s[j] = ((const T*)a.y)[c0 + j];
  }
  if constexpr (HAS_Y) {
    if (lane == 0) {
      for (int s = 0; s < NSLOT; ++s) fpd::mbar_init(&xbar[warp][s], 1);
      fpd::fence_mbar_init();
      for (int s = 0; s < NSLOT; ++s) fpd::mbar_arrive_expect_tx(&xbar[warp][s], kXBytes);
    }
  }
  cluster.sync();  // every CTA resident, windows loaded, exchange barriers armed

  // this warp's rows: the same partition in every CTA of the cluster (warp w pairs with warp w)
  const int64_t cid = blockIdx.x / CS, ncl = gridDim.x / CS;
  const int64_t gw = cid * NW + warp, tw = ncl * NW;
  const int64_t total = a.nnz + kRowCost * m;
  const int64_t r0 = warp_search_rows(rowptr, m, (total * gw) / tw, lane);
  const int64_t r1 = warp_search_rows(rowptr, m, (total * (gw + 1)) / tw, lane);
  const unsigned my_slot = fpd::smem_u32(xslot + ((warp * NSLOT) * CS + rank) * 32 + lane);
  const unsigned my_bar = fpd::smem_u32(&xbar[warp][0]);
  double loss_acc = 0.0;

  // row metadata of a batch (lane i: row rb + i): segment bounds of this block and v[row];
  // loaded one batch ahead so the next batch's rowptr / soff / v latency overlaps this one
  auto meta = [&](int64_t rb, int64_t& sa_, int64_t& sb_, T& vr_) {
    const int64_t row = rb + lane;
    sa_ = sb_ = 0;
    vr_ = T(0);
    if (row < r1) {
      const int64_t rs = __ldg(rowptr + row);
      sa_ = rank > 0 ? rs + __ldg(sa.soff + (int64_t)(rank - 1) * m + row) : rs;
      sb_ = rank < CS - 1 ? rs + __ldg(sa.soff + (int64_t)rank * m + row) : __ldg(rowptr + row + 1);
      vr_ = v ? v[row] : T(1);
    }
  };
  int64_t n_sa, n_sb;
  T n_vr;
  meta(r0, n_sa, n_sb, n_vr);

  int it = 0;
  for (int64_t rb = r0; rb < r1; rb += 32, ++it) {
    // ---- lane i: row rb + i, its segment [sa_i, sb_i) of column block `rank`
    const int64_t row = rb + lane;
    const bool ok = row < r1;
    const int64_t sa_i = n_sa, sb_i = n_sb;
    const T vr = n_vr;
    if (rb + 32 < r1) meta(rb + 32, n_sa, n_sb, n_vr);
    const int len = (int)(sb_i - sa_i);
    int inc = len;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int t = __shfl_up_sync(0xffffffffu, inc, d);
      if (lane >= d) inc += t;
    }
    const int pre = inc - len;                              // exclusive prefix: lane's first entry
    const int cnt = __shfl_sync(0xffffffffu, inc, 31);      // entries of the batch in this block

    // entry at flattened position pos: its row (largest i with pre_i <= pos) and address
    auto locate = [&](int pos, int& rid, int64_t& addr) {
      int lo = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const int cand = lo + step;
        if (__shfl_sync(0xffffffffu, pre, cand) <= pos) lo = cand;
      }
      rid = lo;
      addr = __shfl_sync(0xffffffffu, sa_i, lo) + (pos - __shfl_sync(0xffffffffu, pre, lo));
    };
    // NB tiles of 32 consecutive segment entries from position base: (col - c0, val, row)
    int cc[NB], rid[NB];
    T xv[NB];
    auto load_tiles = [&](int base) {
#pragma unroll
      for (int j = 0; j < NB; ++j) {
        const int pos = base + j * 32 + lane;
        cc[j] = 0;
        xv[j] = T(0);
        rid[j] = 0;
        if (base + j * 32 < cnt) {  // warp-uniform
          int64_t ad;
          locate(pos, rid[j], ad);
          if (pos < cnt) {
            cc[j] = fpd::ld_once(colidx + ad) - c0;
            xv[j] = fpd::ld_once(val + ad);
          }
        }
      }
    };
    // Eq. (2) partial dots of the loaded tiles into rsum[row]: products, then segmented sums
    // in groups of 4 tiles with the shuffle steps interleaved across tiles (independent chains)
    auto dot_tiles = [&](int base) {
      T sv[NB];
#pragma unroll
      for (int j = 0; j < NB; ++j) sv[j] = base + j * 32 + lane < cnt ? xv[j] * y_s[cc[j]] : T(0);
#pragma unroll
      for (int g = 0; g < NB; g += 4) {
        if (base + g * 32 >= cnt) break;  // warp-uniform
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
#pragma unroll
          for (int j = g; j < g + 4 && j < NB; ++j) {
            const T t = __shfl_down_sync(0xffffffffu, sv[j], d);
            const int r2 = __shfl_down_sync(0xffffffffu, rid[j], d);
            if (lane + d < 32 && r2 == rid[j]) sv[j] += t;
          }
        }
      }
#pragma unroll
      for (int j = 0; j < NB; ++j) {
        if (base + j * 32 >= cnt) break;
        const int rprev = __shfl_up_sync(0xffffffffu, rid[j], 1);
        if (base + j * 32 + lane < cnt && (lane == 0 || rprev != rid[j])) rsum[warp * 32 + rid[j]] += sv[j];
        __syncwarp();  // heads of one tile are distinct rows; the next tile may share its first row
      }
    };
    // Eq. (3) scatter of the loaded tiles into this CTA's block of w.  Float shared atomics are
    // CAS loops on sm_100a; issuing the CAS of all tiles before retrying any keeps them
    // independent (one round almost always: columns rarely collide in the window).
    auto scatter_tiles = [&](int base, T q) {
      T inc_[NB], old_[NB];
      unsigned pend = 0;
#pragma unroll
      for (int j = 0; j < NB; ++j) {
        inc_[j] = T(0);
        old_[j] = T(0);
        if (base + j * 32 < cnt) {
          inc_[j] = xv[j] * __shfl_sync(0xffffffffu, q, rid[j]);
          if (base + j * 32 + lane < cnt) {
            old_[j] = w_s[cc[j]];
            pend |= 1u << j;
          }
        }
      }
      while (pend) {
#pragma unroll
        for (int j = 0; j < NB; ++j)
          if (pend & (1u << j)) {
            const T prev = fpd::cas_shared(w_s + cc[j], old_[j], old_[j] + inc_[j]);
            if (fpd::same_bits(prev, old_[j])) pend &= ~(1u << j);
            else old_[j] = prev;
          }
      }
    };

    // ---- first touch: the first NB tiles stay in registers for the scatter (every lane busy);
    // segments longer than NB tiles stream through in further groups of NB tiles (loads of a
    // group in flight together) and are re-read for the scatter (L2 hits)
    constexpr int SPAN = NB * 32;
    T q = T(0);  // lane i: q of row rb + i
    if constexpr (HAS_Y) {
      rsum[warp * 32 + lane] = T(0);
      __syncwarp();
      for (int base = SPAN; base < cnt; base += SPAN) {  // long segments first (registers reused)
        load_tiles(base);
        dot_tiles(base);
      }
      load_tiles(0);
      dot_tiles(0);
      const T mine = rsum[warp * 32 + lane];
      // ---- exchange: this block's partial of row i -> slot [sl][rank][i] of every CTA
      const int sl = it & 1;
      const unsigned so = my_slot + (unsigned)(sl * CS * 32 * sizeof(T));
      const unsigned bo = my_bar + (unsigned)(sl * sizeof(uint64_t));
#pragma unroll
      for (int j = 0; j < CS; ++j) fpd::st_async(fpd::mapa_u32(so, (unsigned)j), mine, fpd::mapa_u32(bo, (unsigned)j));
      // CTA-scope wait: the slots are this CTA's own shared memory, filled by st.async whose
      // bytes the mbarrier's tx-count tracks (a cluster-scope acquire would also invalidate L1,
      // CCTL.IVALL, every batch)
      fpd::mbar_wait(&xbar[warp][sl], (unsigned)((it >> 1) & 1));
      __syncwarp();
      if (lane == 0) fpd::mbar_arrive_expect_tx(&xbar[warp][sl], kXBytes);  // re-arm for batch it + 2
      T p = T(0);
#pragma unroll
      for (int j = 0; j < CS; ++j) p += xslot[((warp * NSLOT + sl) * CS + j) * 32 + lane];  // rank order
      if constexpr (YM == 2) q = fpd::row_epilogue<T>(p, vr, ok, row, ok && rank == 0, a.epi, loss_acc);
      else q = p * vr;
    } else {
      q = vr;
      load_tiles(0);
    }
    scatter_tiles(0, q);
    for (int base = SPAN; base < cnt; base += SPAN) {
      load_tiles(base);
      scatter_tiles(base, q);
    }
  }
  if constexpr (YM == 2) fpd::flush_loss(a.epi, loss_acc);
  cluster.sync();  // no CTA leaves while a peer's st.async may still target it
  fpd::grid_finalize_window<T, T>(w_s, c0, wdt, a.n, a.acc, a.counter, a.alpha, a.beta, (const T*)a.z, (T*)a.w,
                                  a.add_beta_z, a.accumulate);
}

}  // namespace fp
