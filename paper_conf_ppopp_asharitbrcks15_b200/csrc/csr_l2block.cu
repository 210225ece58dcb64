// csr_l2block.cu -- variant 20 (FP_VAR_CSR_L2BLOCK): Eq. (1) on a packed copy of a CSR matrix
// whose y and w are too wide for the shared memory of a CTA group (variant 19): the KDD-shaped
// ultra-wide case (Table 4: KDD2010 has n = 29.9M columns).
//
// Why.  With n = 29.9M fp64, y and w are 240 MB each: every nonzero of the flat path (variant 7)
// is a random 32-byte gather of y plus a random red.global into w that mostly miss the 126 MB
// L2, so the pass is bound by random HBM sectors (K1: 42 ms, 0.022 of the copy peak).  Split
// the COLUMNS into L2-sized blocks instead (bw = 4M columns: y and w of a fp64 block are 64 MB)
// and process the blocks one after the other, so that every gather and every red of a block
// pass hits L2:
//   DOT(b)   for every block but the heaviest H: p[r] += sum over row r's block-b entries of
//            x y (Eq. 2, the row dot, accumulated over the blocks in fp64);
//   FUSED(H) the heaviest block last: its window completes p[r] of its rows, q = alpha v p
//            (Eq. 2 x v), and the same registers scatter x q into w (Eq. 3; a7) --
//            H's entries are read once;
//   Q        q[r] = alpha v[r] p[r] for every row (in place);
//   SCAT(b)  the other blocks re-read: w[c] += x q[r] (Eq. 3), reds into the L2-resident block.
// X is read once for H and twice for the other blocks (KDD-shaped Zipf columns put ~half of the
// nonzeros into block 0): the trade is ~1.5x the streaming bytes for L2 instead of HBM random
// access (reading R27).  The paper's kernels read X once at n that fits its
// GPU's shared memory; this is the B200 plan for n beyond it.
//
// The copy (fp_csr_plan_pack, once per matrix, amortised as the paper amortises its baseline's
// transpose): per block, the block's entries in row order, cut into CHUNKS of at most
// 256 entries (one 8-entry-per-lane register window) and consecutive rows (at most 64 in the
// fused block, whose q sits in shared memory; up to 1024 elsewhere, so that the sparse blocks
// fill their windows); a row with more than 256 entries in a block becomes a run of "partial"
// chunks of 256.  Entry word = column in block | hot flag | row in chunk; chunks padded to 8
// entries (32-byte aligned 256-bit loads).  Descriptor per chunk: (offset / 8, length | rows
// << 16, first row, flags).  HOT columns (more nonzeros than max(2048, nnz / 2^16): a bias
// feature, the head of a Zipf distribution) would serialise their reds on one L2 address;
// their entries are listed once more sorted by column and scattered by k_l2b_hot (one red per
// 256 entries).
#include <algorithm>
#include <cstdlib>
#include <new>
#include <vector>

#include <cub/device/device_scan.cuh>

#include "kernels.cuh"

#include <cub/device/device_radix_sort.cuh>

namespace fp {

namespace {

constexpr int kL2Win = 256;          // entries per chunk (one window, 8 per lane)
constexpr int kL2Group = 1024;       // chunks never cross a group of 1024 rows
constexpr int kL2HeavyRows = 64;     // rows per chunk of the fused block (its q in shared memory)
constexpr unsigned kL2Partial = 1u;  // desc.w: one piece of a row longer than a window
constexpr int kL2MaxBlocks = 64;
constexpr int kL2BS = 256;
constexpr int kL2NW = kL2BS / 32;
constexpr int kL2MaxHot = 1 << 16;   // hot columns (scattered by column, see k_l2b_hot)

enum { L2_DOT = 0, L2_FUSED = 1, L2_SCAT = 2, L2_SCAT_PARTIAL = 3 };

// Entry word: column in block (cb bits) | hot flag (bit cb) | row in chunk (bits cb + 1 ..).
// Padding: column 0, row 63, value 0 (never gathered: entries beyond a chunk's length are
// predicated off; a run of row 63 adds 0).
struct L2Enc {
  unsigned cb;  // column bits
  __host__ __device__ uint32_t colmask() const { return (1u << cb) - 1u; }
  __host__ __device__ uint32_t hotbit() const { return 1u << cb; }
  __host__ __device__ unsigned ridshift() const { return cb + 1; }
  __host__ __device__ uint32_t pad() const { return 63u << (cb + 1); }
};

struct L2Args {
  const uint4* desc;    // chunks (offset / 8, length | rows << 16, first row, flags | block << 8)
  int64_t nch;
  int64_t bw;           // columns per block (block b starts at column b bw)
  L2Enc enc;
  const uint32_t* cr;
  const void* val;      // T
  const void* y;        // T, the full vector
  const void* v;        // T or NULL (= 1)
  double alpha;
  double* p;            // [m]: row dots, q after k_l2b_q
  void* w;              // T
  const uint32_t* list; // chunk c of this launch = desc[list[c]] (NULL: desc[c])
};

// 8 consecutive entries (32-byte aligned): streamed, evict-first in L2 (the blocks of y and w
// are what L2 should keep)
__device__ __forceinline__ void l2_ldc(const uint32_t* p, uint32_t (&c)[8]) {
  asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]), "=r"(c[4]), "=r"(c[5]), "=r"(c[6]), "=r"(c[7])
      : "l"(p));
}
__device__ __forceinline__ void l2_ldv(const float* p, float (&x)[8]) {
  asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]), "=f"(x[4]), "=f"(x[5]), "=f"(x[6]), "=f"(x[7])
      : "l"(p));
}
__device__ __forceinline__ void l2_ldv(const double* p, double (&x)[8]) {
  asm("ld.global.nc.L1::no_allocate.L2::evict_first.v4.f64 {%0,%1,%2,%3}, [%4];"
      : "=d"(x[0]), "=d"(x[1]), "=d"(x[2]), "=d"(x[3]) : "l"(p));
  asm("ld.global.nc.L1::no_allocate.L2::evict_first.v4.f64 {%0,%1,%2,%3}, [%4];"
      : "=d"(x[4]), "=d"(x[5]), "=d"(x[6]), "=d"(x[7]) : "l"(p + 4));
}
// y of the block: kept in L2 (an evict_last cache policy) and cached in L1 -- the hot columns'
// y values are read by most rows: without L1 every such read goes to the one L2 slice that
// holds the word (K1's fused block: 3.99 ms with L1::no_allocate, ncu r02c)
__device__ __forceinline__ uint64_t l2_keep_policy() {
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ float l2_ldy(const float* p, uint64_t pol) {
  float v;
  asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ double l2_ldy(const double* p, uint64_t pol) {
  double v;
  asm("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
  return v;
}

// One pass over the chunks of one column block (a warp per chunk, grid-stride).
//   DOT / FUSED: Eq. (2) on the window -- in-lane runs of a row, one bounded segmented scan
//     across lanes; the lane that closes a row's run owns its window sum.  DOT (and the partial
//     chunks of the fused block): the owner adds it into p[row] (fp64 red).  FUSED (rows <= 64):
//     the sums go to shared memory, p[row] is completed, q = alpha v p, and the scatter runs
//     from the registers that hold the window (a7).
//   SCAT: q[row] = p[row] after k_l2b_q; SCAT_PARTIAL: the fused block's partial chunks.
// Hot entries (columns scattered by column in k_l2b_hot) take part in the dot, not the scatter.
template <typename T, int MODE>
__global__ void __launch_bounds__(kL2BS) k_l2b(const L2Args a) {
  __shared__ double s_rs[kL2NW][kL2HeavyRows];
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  double* rs = s_rs[wi];
  const T* __restrict__ yall = reinterpret_cast<const T*>(a.y);
  const T* __restrict__ vv = reinterpret_cast<const T*>(a.v);
  const T* __restrict__ val = reinterpret_cast<const T*>(a.val);
  T* wall = reinterpret_cast<T*>(a.w);
  double* p = a.p;
  const uint32_t cmask = a.enc.colmask(), hot = a.enc.hotbit();
  const unsigned rsh = a.enc.ridshift();
  const uint32_t padw = a.enc.pad();
  const uint64_t keep = l2_keep_policy();
  const int64_t nw = (int64_t)gridDim.x * kL2NW;
  for (int64_t c = (int64_t)blockIdx.x * kL2NW + wi; c < a.nch; c += nw) {
    const uint4 D = __ldg(a.desc + (a.list ? (int64_t)__ldg(a.list + c) : c));
    const bool partial = (D.w & kL2Partial) != 0;
    if (MODE == L2_SCAT_PARTIAL && !partial) continue;
    const int len = (int)(D.y & 0xFFFFu), rows = (int)(D.y >> 16);
    double* pr0 = p + D.z;
    const int64_t col0 = (int64_t)(D.w >> 8) * a.bw;  // the chunk's block (a launch may span several)
    const T* __restrict__ y = yall + col0;
    T* w = wall + col0;
    const int o = 8 * lane;
    uint32_t cw[8];
    T xv[8];
    if (o < len) {
      const int64_t e0 = (int64_t)D.x * 8 + o;
      l2_ldc(a.cr + e0, cw);
      l2_ldv(val + e0, xv);
    } else {
#pragma unroll
      for (int e = 0; e < 8; ++e) cw[e] = padw, xv[e] = T(0);
    }
    bool fused = false;
    if constexpr (MODE == L2_DOT || MODE == L2_FUSED) {
      fused = MODE == L2_FUSED && !partial;
      if (fused) {
        rs[lane] = 0.0;
        rs[lane + 32] = 0.0;
        __syncwarp();
      }
      // the owner of a row's window sum: the shared slot (fused) or a red into p
      auto put = [&](unsigned r, T sum) {
        if (fused) rs[r] = (double)sum;
        else if ((int)r < rows) atomicAdd(pr0 + r, (double)sum);
      };
      T cs_[8];
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const T pr = o + e < len ? xv[e] * l2_ldy(y + (cw[e] & cmask), keep) : T(0);
        cs_[e] = (e == 0 || (cw[e] >> rsh) != (cw[e - 1] >> rsh)) ? pr : cs_[e - 1] + pr;
      }
      const int last = (int)(cw[7] >> rsh);
      int prev = __shfl_up_sync(0xffffffffu, last, 1);
      if (lane == 0) prev = -1;
      const bool h0 = (int)(cw[0] >> rsh) != prev;
      bool seen = h0;
#pragma unroll
      for (int e = 0; e < 7; ++e) {
        const bool h = (cw[e + 1] >> rsh) != (cw[e] >> rsh);
        if (h && seen) put(cw[e] >> rsh, cs_[e]);
        seen |= h;
      }
      T P = cs_[7];
#pragma unroll
      for (int e = 7; e >= 1; --e)
        if ((cw[e] >> rsh) != (cw[e - 1] >> rsh)) P = cs_[e - 1];
      if (h0) P = T(0);
      const unsigned hl = __ballot_sync(0xffffffffu, seen) >> lane;
      const int dist = hl ? __ffs(hl) : 32 - lane;
      T r = P;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const T t2 = __shfl_down_sync(0xffffffffu, r, d);
        if (d < dist) r += t2;
      }
      T rn = __shfl_down_sync(0xffffffffu, r, 1);
      if (lane == 31) rn = T(0);
      if (seen) put((unsigned)last, cs_[7] + rn);
      if (fused) {
        // the fused block, processed last: p complete -> q = alpha v p, kept for the scatter
        __syncwarp();
        for (int k = lane; k < rows; k += 32) {
          const double pt = pr0[k] + rs[k];
          pr0[k] = pt;
          const double vr = vv ? (double)vv[D.z + k] : 1.0;
          rs[k] = a.alpha * (vr * pt);
        }
        __syncwarp();
      }
    }
    if (MODE == L2_SCAT || MODE == L2_SCAT_PARTIAL || fused) {
      // Eq. (3) from the registers that hold the window: one red per nonzero into the block of w
      const double q1 = MODE == L2_SCAT_PARTIAL ? __ldg(pr0) : 0.0;
#pragma unroll
      for (int e = 0; e < 8; ++e)
        if (o + e < len && !(cw[e] & hot)) {
          const double q = MODE == L2_SCAT_PARTIAL ? q1 : (fused ? rs[cw[e] >> rsh] : __ldg(pr0 + (cw[e] >> rsh)));
          atomicAdd(w + (cw[e] & cmask), (T)((double)xv[e] * q));
        }
    }
    __syncwarp();
  }
}

// Hot columns (a column with more nonzeros than the threshold of l2block_build, e.g. the bias
// feature every row of a KDD-like matrix has): one red per nonzero would serialise on one L2
// address (K1: ~15M reds into the first columns).  Their entries are kept a second time sorted
// by column; a warp sums 256 of them, x q[row], and adds ONE red per item (Eq. 3 by column).
template <typename T>
__global__ void __launch_bounds__(kL2BS) k_l2b_hot(const uint4* __restrict__ items, int64_t nitems,
                                                   const uint32_t* __restrict__ hrow, const T* __restrict__ hval,
                                                   const int32_t* __restrict__ hcol, const double* __restrict__ q,
                                                   T* w) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * kL2NW;
  for (int64_t it = (int64_t)blockIdx.x * kL2NW + (threadIdx.x >> 5); it < nitems; it += nw) {
    const uint4 I = __ldg(items + it);  // (first entry, count, hot slot)
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < kL2Win / 32; ++k) {
      const int e = k * 32 + lane;
      if (e < (int)I.y) s += (double)hval[I.x + e] * __ldg(q + hrow[I.x + e]);
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
    if (lane == 0) atomicAdd(w + hcol[I.z], (T)s);
  }
}

// q[r] = alpha v[r] p[r] in place (has_y = 0: q = alpha v, Table 1 row 1)
template <typename T>
__global__ void k_l2b_q(int64_t m, double* __restrict__ p, const T* __restrict__ v, double alpha, int has_y) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    const double vr = v ? (double)v[r] : 1.0;
    p[r] = has_y ? alpha * (vr * p[r]) : alpha * vr;
  }
}

// w = (accumulate ? w : 0) + (beta z when added here); the block passes then red into it
template <typename T>
__global__ void k_l2b_init(int64_t n, T* __restrict__ w, const T* __restrict__ z, double beta, int add_bz, int acc) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    double s = acc ? (double)w[j] : 0.0;
    if (add_bz && beta != 0.0) s += beta * (double)z[j];
    w[j] = (T)s;
  }
}

// ---------------------------------------------------------------- the copy (pack time)
// (1) entries of row r in block b (cnt[b m + r]) and of column c (colcnt[c]); a warp per row
// (its lanes on distinct columns of the row)
__global__ void k_l2b_count(int64_t m, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ colidx,
                            int64_t bw, uint32_t* __restrict__ cnt, uint32_t* __restrict__ colcnt) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x / 32);
  for (int64_t r = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); r < m; r += nw) {
    const int64_t e = rowptr[r + 1];
    for (int64_t i = rowptr[r] + lane; i < e; i += 32) {
      atomicAdd(cnt + (int64_t)(colidx[i] / bw) * m + r, 1u);
      atomicAdd(colcnt + colidx[i], 1u);
    }
  }
}
// entries per block: sum of cnt over the rows (one CTA per (block, slice), a red per CTA)
__global__ void k_l2b_blocktot(int64_t m, const uint32_t* __restrict__ cnt, unsigned long long* __restrict__ tot) {
  const int b = blockIdx.y;
  unsigned long long s = 0;
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x)
    s += cnt[(int64_t)b * m + r];
  for (int d = 16; d > 0; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
  if ((threadIdx.x & 31) == 0) atomicAdd(tot + b, s);
}
// hot entries of each row (their offsets: an exclusive scan)
__global__ void k_l2b_hotrows(int64_t m, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ colidx,
                              const int32_t* __restrict__ slot, int64_t* __restrict__ hr) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    int64_t k = 0;
    for (int64_t i = rowptr[r]; i < rowptr[r + 1]; ++i) k += slot[colidx[i]] >= 0;
    hr[r] = k;
  }
}

// (2) hot columns: more than `thr` nonzeros -> a slot (at most kL2MaxHot)
__global__ void k_l2b_hotsel(int64_t n, const uint32_t* __restrict__ colcnt, uint32_t thr, int32_t* __restrict__ slot,
                             int32_t* __restrict__ hcol, unsigned* __restrict__ nhot) {
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
    int32_t sl = -1;
    if (colcnt[c] > thr) {
      const unsigned k = atomicAdd(nhot, 1u);
      if (k < (unsigned)kL2MaxHot) {
        sl = (int32_t)k;
        hcol[k] = (int32_t)c;
      }
    }
    slot[c] = sl;
  }
}

// (3) the chunks of one (block, 1024-row group): a thread walks the group's rows.  COUNT:
// number of chunks and padded entries; WRITE: the descriptors, and per (block, row) the entry
// offset of the row's first block-b entry and its row in the chunk.  A chunk: <= 256 entries,
// <= rowcap rows (64 in the fused block, else as many as the entry word's row field holds).
template <bool WRITE>
__global__ void k_l2b_walk(int64_t m, int cs, int heavy, int rowcap, const uint32_t* __restrict__ cnt,
                           int64_t* __restrict__ nchunk, int64_t* __restrict__ nent, const int64_t* __restrict__ cbase,
                           const int64_t* __restrict__ ebase, uint4* __restrict__ desc, uint32_t* __restrict__ rowoff,
                           uint16_t* __restrict__ rid) {
  const int64_t ng = (m + kL2Group - 1) / kL2Group;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < (int64_t)cs * ng;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int b = (int)(t / ng);
    const int64_t g = t % ng;
    const int cap = b == heavy ? kL2HeavyRows : rowcap;
    int64_t ci = WRITE ? cbase[t] : 0, ei = WRITE ? ebase[t] : 0;
    int64_t nc = 0, ne = 0;
    int64_t r0 = -1, last_row = -1;
    int len = 0;
    auto emit = [&](int64_t first, int rows, int l, unsigned flags) {
      if (WRITE)
        desc[ci++] = make_uint4((unsigned)(ei / 8), (unsigned)l | ((unsigned)rows << 16), (unsigned)first,
                                flags | ((unsigned)b << 8));
      ++nc;
      const int64_t al = (l + 7) & ~7;
      ne += al;
      ei += al;
    };
    auto flush = [&]() {
      if (r0 >= 0) emit(r0, (int)(last_row - r0 + 1), len, 0u);
      r0 = -1;
      len = 0;
    };
    for (int i = 0; i < kL2Group && g * kL2Group + i < m; ++i) {
      const int64_t r = g * kL2Group + i;
      const uint32_t c = cnt[(int64_t)b * m + r];
      if (c == 0) continue;
      if (c > (uint32_t)kL2Win) {  // a run of partial chunks of 256 (contiguous entries)
        flush();
        if (WRITE) {
          rowoff[(int64_t)b * m + r] = (uint32_t)ei;
          rid[(int64_t)b * m + r] = 0;
        }
        for (uint32_t k = 0; k < c; k += kL2Win) emit(r, 1, (int)std::min<uint32_t>(kL2Win, c - k), kL2Partial);
        continue;
      }
      if (r0 >= 0 && (len + (int)c > kL2Win || r - r0 >= cap)) flush();
      if (r0 < 0) r0 = r;
      if (WRITE) {
        rowoff[(int64_t)b * m + r] = (uint32_t)(ei + len);
        rid[(int64_t)b * m + r] = (uint16_t)(r - r0);
      }
      len += (int)c;
      last_row = r;
    }
    flush();
    if (!WRITE) {
      nchunk[t] = nc;
      nent[t] = ne;
    }
  }
}

// (4) the entries: a thread per row, running count per block (stable order: non-canonical rows
// are packed as given, reading R7); hot entries flagged and listed once more (key: slot, row)
template <typename V>
__global__ void k_l2b_scatter(int64_t m, int cs, int64_t bw, L2Enc enc, const int64_t* __restrict__ rowptr,
                              const int32_t* __restrict__ colidx, const V* __restrict__ val,
                              const uint32_t* __restrict__ rowoff, const uint16_t* __restrict__ rid,
                              const int32_t* __restrict__ slot, uint32_t* __restrict__ cr, V* __restrict__ pval,
                              unsigned long long* __restrict__ hkey, V* __restrict__ hv, const int64_t* __restrict__ hroff) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    uint32_t k[kL2MaxBlocks];
    for (int b = 0; b < cs; ++b) k[b] = 0;
    const int64_t e = rowptr[r + 1];
    int64_t h = slot ? hroff[r] : 0;
    for (int64_t i = rowptr[r]; i < e; ++i) {
      const int col = colidx[i];
      const int b = (int)(col / bw);
      const int64_t pos = (int64_t)rowoff[(int64_t)b * m + r] + k[b]++;
      const int32_t sl = slot ? slot[col] : -1;
      cr[pos] = (uint32_t)(col - b * bw) | (sl >= 0 ? enc.hotbit() : 0u) |
                ((uint32_t)rid[(int64_t)b * m + r] << enc.ridshift());
      pval[pos] = val[i];
      if (sl >= 0) {
        hkey[h] = ((unsigned long long)sl << 32) | (unsigned long long)r;
        hv[h++] = val[i];
      }
    }
  }
}

__global__ void k_l2b_fill(int64_t n, uint32_t* __restrict__ p, uint32_t v) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}
__global__ void k_l2b_gather(int64_t n, const int32_t* __restrict__ idx, const uint32_t* __restrict__ src,
                             uint32_t* __restrict__ dst) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = src[idx[i]];
}
__global__ void k_l2b_rows(int64_t n, const unsigned long long* __restrict__ key, uint32_t* __restrict__ row) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    row[i] = (uint32_t)key[i];
}

unsigned bits_for(int64_t v) {  // bits to hold 0 .. v - 1
  unsigned b = 1;
  while (((int64_t)1 << b) < v) ++b;
  return b;
}

}  // namespace

// columns per L2 block: fp64 4M (y and w of a block: 64 MB) -- measured on K1 (per-block
// launches, hot columns by column, y cached in L1): 1M / 2M / 3M / 4M / 6M / 8M / 12M columns
// 6.43 / 5.62 / 5.30 / 5.17 / 5.33 / 6.34 / 8.65 ms; fp32 4M (32 MB, unmeasured: no fp32
// config is this wide).  FP_L2B_BW (measurement / tests) overrides; at most kL2MaxBlocks
// blocks, at most 2^24 columns a block
int64_t l2block_bw(int64_t n, fp_dtype dt) {
  int64_t bw = (int64_t)1 << 22;
  if (const char* e = std::getenv("FP_L2B_BW")) bw = std::max<int64_t>(1, std::atoll(e));
  bw = std::max<int64_t>(bw, (n + kL2MaxBlocks - 1) / kL2MaxBlocks);
  return std::min<int64_t>(std::min<int64_t>(bw, n), (int64_t)1 << 24);
}

fp_status l2block_build(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                        const void* val, fp_dtype dtype, Packed* p, cudaStream_t s) {
  const int64_t bw = l2block_bw(n, dtype);
  const int cs = (int)((n + bw - 1) / bw);
  FP_REQUIRE(cs <= kL2MaxBlocks, FP_ERR_UNSUPPORTED, "fp_csr_plan_pack: n = %lld needs more than %d L2 blocks",
             (long long)n, kL2MaxBlocks);
  const L2Enc enc{bits_for(bw)};
  const int rowcap = (int)std::min<int64_t>(kL2Group, (int64_t)1 << (31 - enc.cb));
  const DeviceInfo& di = device_info(current_device());
  const int64_t ng = (m + kL2Group - 1) / kL2Group;
  const int64_t nt = (int64_t)cs * ng;
  const size_t vs = dtype_size(dtype);
  uint32_t *cnt = nullptr, *colcnt = nullptr, *rowoff = nullptr;
  uint16_t* rid = nullptr;
  int32_t* slot = nullptr;
  unsigned long long *blocktot = nullptr, *hkey = nullptr, *hkey2 = nullptr, *hn = nullptr;
  void *hv = nullptr, *tmp = nullptr;
  unsigned* nhot = nullptr;
  int64_t *nchunk = nullptr, *nent = nullptr, *cbase = nullptr, *ebase = nullptr, *hroff = nullptr;
  auto cleanup = [&]() {
    for (void* b : {(void*)cnt, (void*)colcnt, (void*)rowoff, (void*)rid, (void*)slot, (void*)blocktot, (void*)hkey,
                    (void*)hkey2, (void*)hn, hv, tmp, (void*)nhot, (void*)nchunk, (void*)nent, (void*)cbase,
                    (void*)ebase, (void*)hroff})
      if (b) cudaFree(b);
  };
  auto fail = [&](cudaError_t e, const char* what) {
    cudaGetLastError();
    set_error("fp_csr_plan_pack (L2 blocks): %s: %s", what, cudaGetErrorString(e));
    cleanup();
    return e == cudaErrorMemoryAllocation ? FP_ERR_NOMEM : FP_ERR_CUDA;
  };
#define L2_TRY(call, what)                          \
  do {                                              \
    cudaError_t e_ = (call);                        \
    if (e_ != cudaSuccess) return fail(e_, what);   \
  } while (0)
  const int tb = 256;
  auto grid_of = [&](int64_t k) { return (int)std::max<int64_t>(1, std::min<int64_t>((k + tb - 1) / tb, (int64_t)di.sm_count * 32)); };
  L2_TRY(cudaMalloc((void**)&cnt, (size_t)cs * m * 4), "alloc");
  L2_TRY(cudaMalloc((void**)&colcnt, (size_t)n * 4), "alloc");
  L2_TRY(cudaMalloc((void**)&blocktot, (size_t)cs * 8), "alloc");
  L2_TRY(cudaMemsetAsync(cnt, 0, (size_t)cs * m * 4, s), "memset");
  L2_TRY(cudaMemsetAsync(colcnt, 0, (size_t)n * 4, s), "memset");
  L2_TRY(cudaMemsetAsync(blocktot, 0, (size_t)cs * 8, s), "memset");
  k_l2b_count<<<grid_of(m * 32), tb, 0, s>>>(m, rowptr, colidx, bw, cnt, colcnt);
  k_l2b_blocktot<<<dim3((unsigned)std::min<int64_t>((m + tb - 1) / tb, 256), (unsigned)cs), tb, 0, s>>>(m, cnt, blocktot);
  // the heaviest block runs last, fused
  std::vector<unsigned long long> hbt(cs);
  L2_TRY(cudaMemcpyAsync(hbt.data(), blocktot, (size_t)cs * 8, cudaMemcpyDeviceToHost, s), "copy");
  // hot columns: more than max(2048, nnz / 2^16) nonzeros (FP_L2B_HOT overrides; 0 = none)
  uint32_t thr = (uint32_t)std::max<int64_t>(2048, nnz >> 16);
  if (const char* e = std::getenv("FP_L2B_HOT"); e && *e) thr = (uint32_t)std::max<long long>(0, std::atoll(e));
  L2_TRY(cudaMalloc((void**)&slot, (size_t)n * 4), "alloc");
  L2_TRY(cudaMalloc((void**)&p->hcol, (size_t)kL2MaxHot * 4), "alloc");
  L2_TRY(cudaMalloc((void**)&nhot, 4), "alloc");
  L2_TRY(cudaMemsetAsync(nhot, 0, 4, s), "memset");
  const bool use_hot = thr > 0;
  if (use_hot) k_l2b_hotsel<<<grid_of(n), tb, 0, s>>>(n, colcnt, thr, slot, p->hcol, nhot);
  unsigned hnh = 0;
  L2_TRY(cudaMemcpyAsync(&hnh, nhot, 4, cudaMemcpyDeviceToHost, s), "copy");
  L2_TRY(cudaStreamSynchronize(s), "sync");
  const int nh = (int)std::min<unsigned>(hnh, (unsigned)kL2MaxHot);
  int heavy = 0;
  for (int b = 1; b < cs; ++b)
    if (hbt[b] > hbt[heavy]) heavy = b;
  // chunks
  L2_TRY(cudaMalloc((void**)&nchunk, (size_t)(nt + 1) * 8), "alloc");
  L2_TRY(cudaMalloc((void**)&nent, (size_t)(nt + 1) * 8), "alloc");
  L2_TRY(cudaMalloc((void**)&cbase, (size_t)(nt + 1) * 8), "alloc");
  L2_TRY(cudaMalloc((void**)&ebase, (size_t)(nt + 1) * 8), "alloc");
  L2_TRY(cudaMemsetAsync(nchunk + nt, 0, 8, s), "memset");
  L2_TRY(cudaMemsetAsync(nent + nt, 0, 8, s), "memset");
  k_l2b_walk<false><<<grid_of(nt), tb, 0, s>>>(m, cs, heavy, rowcap, cnt, nchunk, nent, nullptr, nullptr, nullptr,
                                               nullptr, nullptr);
  size_t tb_bytes = 0, tmp_bytes = 0;
  L2_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb_bytes, nchunk, cbase, nt + 1, s), "scan");
  tmp_bytes = tb_bytes;
  L2_TRY(cudaMalloc(&tmp, tmp_bytes), "alloc");
  L2_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb_bytes, nchunk, cbase, nt + 1, s), "scan");
  L2_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb_bytes, nent, ebase, nt + 1, s), "scan");
  std::vector<int64_t> hcb(cs + 1), heb(cs + 1);
  for (int b = 0; b <= cs; ++b) {
    L2_TRY(cudaMemcpyAsync(&hcb[b], cbase + (int64_t)b * ng, 8, cudaMemcpyDeviceToHost, s), "copy");
    L2_TRY(cudaMemcpyAsync(&heb[b], ebase + (int64_t)b * ng, 8, cudaMemcpyDeviceToHost, s), "copy");
  }
  L2_TRY(cudaStreamSynchronize(s), "sync");
  const int64_t nch = hcb[cs], total = heb[cs];
  if (total >= (int64_t)UINT32_MAX * 8) return fail(cudaErrorInvalidValue, "too many entries for 32-bit offsets");
  if (total >= (int64_t)UINT32_MAX) return fail(cudaErrorInvalidValue, "too many entries for 32-bit row offsets");
  L2_TRY(cudaMalloc((void**)&p->tile_desc, (size_t)std::max<int64_t>(nch, 1) * sizeof(uint4)), "alloc");
  L2_TRY(cudaMalloc((void**)&rowoff, (size_t)cs * m * 4), "alloc");
  L2_TRY(cudaMalloc((void**)&rid, (size_t)cs * m * 2), "alloc");
  k_l2b_walk<true><<<grid_of(nt), tb, 0, s>>>(m, cs, heavy, rowcap, cnt, nullptr, nullptr, cbase, ebase, p->tile_desc,
                                              rowoff, rid);
  const int64_t cap = total + 8;
  L2_TRY(cudaMalloc((void**)&p->cr, (size_t)cap * 4), "alloc");
  L2_TRY(cudaMalloc((void**)&p->val, (size_t)cap * vs), "alloc");
  k_l2b_fill<<<grid_of(cap), tb, 0, s>>>(cap, p->cr, enc.pad());
  L2_TRY(cudaMemsetAsync(p->val, 0, (size_t)cap * vs, s), "memset");
  // hot entries: exactly the nonzeros of the hot columns
  int64_t nhe = 0;
  if (nh > 0) {
    std::vector<uint32_t> hcnt(nh);
      L2_TRY(cudaMalloc((void**)&hkey, (size_t)nh * 4), "alloc");  // (scratch: the hot columns' counts)
    k_l2b_gather<<<grid_of(nh), tb, 0, s>>>(nh, p->hcol, colcnt, (uint32_t*)hkey);
    L2_TRY(cudaMemcpyAsync(hcnt.data(), hkey, (size_t)nh * 4, cudaMemcpyDeviceToHost, s), "copy");
    L2_TRY(cudaStreamSynchronize(s), "sync");
    cudaFree(hkey);
    hkey = nullptr;
    // work items: <= 256 entries of one hot column, in slot order (the sort below)
    std::vector<uint4> items;
    int64_t off = 0;
    for (int k = 0; k < nh; ++k) {
      for (uint32_t e = 0; e < hcnt[k]; e += kL2Win)
        items.push_back(make_uint4((unsigned)(off + e), std::min<uint32_t>(kL2Win, hcnt[k] - e), (unsigned)k, 0u));
      off += hcnt[k];
    }
    nhe = off;
    L2_TRY(cudaMalloc((void**)&hkey, (size_t)nhe * 8), "alloc");
    L2_TRY(cudaMalloc((void**)&hkey2, (size_t)nhe * 8), "alloc");
    L2_TRY(cudaMalloc(&hv, (size_t)nhe * vs), "alloc");
    L2_TRY(cudaMalloc((void**)&p->hval, (size_t)nhe * vs), "alloc");
    L2_TRY(cudaMalloc((void**)&p->hrow, (size_t)nhe * 4), "alloc");
    // each row's hot entries at an offset of its own (no shared counter)
    L2_TRY(cudaMalloc((void**)&hn, (size_t)(m + 1) * 8), "alloc");
    L2_TRY(cudaMalloc((void**)&hroff, (size_t)(m + 1) * 8), "alloc");
    L2_TRY(cudaMemsetAsync(hn + m, 0, 8, s), "memset");
    k_l2b_hotrows<<<grid_of(m), tb, 0, s>>>(m, rowptr, colidx, slot, (int64_t*)hn);
    size_t hb = 0;
    L2_TRY(cub::DeviceScan::ExclusiveSum(nullptr, hb, (int64_t*)hn, hroff, m + 1, s), "scan");
    if (hb > tmp_bytes) {
      cudaFree(tmp);
      tmp = nullptr;
      tmp_bytes = hb;
      L2_TRY(cudaMalloc(&tmp, tmp_bytes), "alloc");
    }
    L2_TRY(cub::DeviceScan::ExclusiveSum(tmp, hb, (int64_t*)hn, hroff, m + 1, s), "scan");
    L2_TRY(cudaMalloc((void**)&p->hitems, items.size() * sizeof(uint4)), "alloc");
    L2_TRY(cudaMemcpyAsync(p->hitems, items.data(), items.size() * sizeof(uint4), cudaMemcpyHostToDevice, s), "copy");
    L2_TRY(cudaStreamSynchronize(s), "sync");
    p->nhitems = (int64_t)items.size();
  }
  if (dtype == FP_F64)
    k_l2b_scatter<double><<<grid_of(m), tb, 0, s>>>(m, cs, bw, enc, rowptr, colidx, (const double*)val, rowoff, rid,
                                                    nh > 0 ? slot : nullptr, p->cr, (double*)p->val, hkey,
                                                    (double*)hv, hroff);
  else
    k_l2b_scatter<float><<<grid_of(m), tb, 0, s>>>(m, cs, bw, enc, rowptr, colidx, (const float*)val, rowoff, rid,
                                                   nh > 0 ? slot : nullptr, p->cr, (float*)p->val, hkey, (float*)hv,
                                                   hroff);
  if (nhe > 0) {  // sort the hot entries by (slot, row): each column's entries contiguous, in row order
    size_t sb = 0;
    const int end_bit = 32 + (int)bits_for(nh + 1);
    if (dtype == FP_F64)
      L2_TRY(cub::DeviceRadixSort::SortPairs(nullptr, sb, hkey, hkey2, (const double*)hv, (double*)p->hval, nhe, 0,
                                             end_bit, s), "sort");
    else
      L2_TRY(cub::DeviceRadixSort::SortPairs(nullptr, sb, hkey, hkey2, (const float*)hv, (float*)p->hval, nhe, 0,
                                             end_bit, s), "sort");
    if (sb > tmp_bytes) {
      cudaFree(tmp);
      tmp = nullptr;
      tmp_bytes = sb;
      L2_TRY(cudaMalloc(&tmp, tmp_bytes), "alloc");
    }
    if (dtype == FP_F64)
      L2_TRY(cub::DeviceRadixSort::SortPairs(tmp, sb, hkey, hkey2, (const double*)hv, (double*)p->hval, nhe, 0,
                                             end_bit, s), "sort");
    else
      L2_TRY(cub::DeviceRadixSort::SortPairs(tmp, sb, hkey, hkey2, (const float*)hv, (float*)p->hval, nhe, 0,
                                             end_bit, s), "sort");
    k_l2b_rows<<<grid_of(nhe), tb, 0, s>>>(nhe, hkey2, p->hrow);
  }
  // the dot phase of the non-fused blocks in (row panel, block) order: a panel of 2^21 rows
  // keeps its 16 MB of p in L2 while the blocks' dots red into it (one block at a time the reds
  // into the whole 120 MB p go to HBM: ~0.5 GB per block pass on K1)
  {
    const int64_t R = (int64_t)1 << 21, gpp = R / kL2Group;  // rows, 1024-row groups per panel
    std::vector<int64_t> hcbase(nt + 1);
    L2_TRY(cudaMemcpyAsync(hcbase.data(), cbase, (size_t)(nt + 1) * 8, cudaMemcpyDeviceToHost, s), "copy");
    L2_TRY(cudaStreamSynchronize(s), "sync");
    std::vector<uint32_t> list;
    list.reserve((size_t)(nch - (hcb[heavy + 1] - hcb[heavy])));
    for (int64_t g0 = 0; g0 < ng; g0 += gpp) {
      const int64_t g1 = std::min(ng, g0 + gpp);
      for (int b = 0; b < cs; ++b) {
        if (b == heavy) continue;
        for (int64_t c = hcbase[(int64_t)b * ng + g0]; c < hcbase[(int64_t)b * ng + g1]; ++c) list.push_back((uint32_t)c);
      }
    }
    p->ndot = (int64_t)list.size();
    if (!list.empty()) {
      L2_TRY(cudaMalloc((void**)&p->dotlist, list.size() * 4), "alloc");
      L2_TRY(cudaMemcpyAsync(p->dotlist, list.data(), list.size() * 4, cudaMemcpyHostToDevice, s), "copy");
    }
  }
  L2_TRY(cudaMalloc((void**)&p->rowdot, (size_t)std::max<int64_t>(m, 1) * 8), "alloc");
  L2_TRY(cudaStreamSynchronize(s), "sync");
#undef L2_TRY
  cleanup();
  p->mode = 1;
  p->cs = cs;
  p->bw = (int)bw;
  p->cbits = (int)enc.cb;
  p->ntiles = nch;
  p->entries = total;
  p->groups = 0;
  p->nhot = nh;
  p->l2cb.assign(hcb.begin(), hcb.end());
  p->heavy = heavy;
  p->hot_entries = nhe;
  p->heavy_entries = heb[heavy + 1] - heb[heavy];
  return FP_OK;
}

void packed_detail(const Packed* p, int64_t out[8]) {
  for (int i = 0; i < 8; ++i) out[i] = 0;
  if (p->mode == 1) {
    out[0] = FP_VAR_CSR_L2BLOCK;
    out[1] = p->cs;
    out[2] = p->heavy;
    out[3] = p->nhot;
    out[4] = p->hot_entries;
    out[5] = 2 * p->entries - p->heavy_entries + p->hot_entries;
    // init, the dot launch(es), fused, q, a scatter launch per other block, partial, hot
    const char* e = std::getenv("FP_L2B_PANELS");
    const bool panels = e && std::atoi(e) != 0 && p->dotlist;
    out[6] = (panels ? 1 : (p->cs - 1)) + (p->cs - 1) + 5;
  } else {
    out[0] = FP_VAR_CSR_PACKED;
    out[1] = p->cs;
    out[2] = -1;
    out[5] = p->entries;
    out[6] = 2;  // the pass + the finalize
  }
}

fp_status l2block_exec(Packed* p, const PatternArgs& a, cudaStream_t s) {
  const DeviceInfo& di = device_info(current_device());
  const bool has_y = a.y != nullptr;
  const int64_t m = p->m, n = p->n;
  const int tb = 256;
  const bool f64 = p->dtype == FP_F64;
  const int gn = (int)std::min<int64_t>((n + tb - 1) / tb, (int64_t)di.sm_count * 8);
  if (f64)
    k_l2b_init<double><<<gn, tb, 0, s>>>(n, (double*)a.w, (const double*)a.z, a.beta, a.add_beta_z ? 1 : 0,
                                         a.accumulate ? 1 : 0);
  else
    k_l2b_init<float><<<gn, tb, 0, s>>>(n, (float*)a.w, (const float*)a.z, a.beta, a.add_beta_z ? 1 : 0,
                                        a.accumulate ? 1 : 0);
  FP_CUDA(cudaGetLastError());
  if (has_y) FP_CUDA(cudaMemsetAsync(p->rowdot, 0, (size_t)m * 8, s));
  // one launch per phase over a range of chunks [c0, c1): the chunks are stored block by block
  // and a grid-stride loop walks them in order, so the SMs work on one or two blocks at a time
  // (their y / w stay in L2) without a launch per block
  auto pass = [&](int64_t c0, int64_t c1, int mode, const uint32_t* list = nullptr) -> fp_status {
    L2Args k{};  // (an empty range still launches: a fixed launch count per call)
    k.nch = std::max<int64_t>(0, c1 - c0);
    k.desc = list ? p->tile_desc : p->tile_desc + c0;
    k.list = list ? list + c0 : nullptr;
    k.bw = p->bw;
    k.enc = L2Enc{(unsigned)p->cbits};
    k.cr = p->cr;
    k.val = p->val;
    k.y = a.y;
    k.v = a.v;
    k.alpha = a.alpha;
    k.p = p->rowdot;
    k.w = a.w;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((k.nch + kL2NW - 1) / kL2NW, (int64_t)di.sm_count * 8));
#define L2_LAUNCH(M)                                                    \
  if (f64) k_l2b<double, M><<<grid, kL2BS, 0, s>>>(k);                  \
  else k_l2b<float, M><<<grid, kL2BS, 0, s>>>(k);
    switch (mode) {
      case L2_DOT: L2_LAUNCH(L2_DOT) break;
      case L2_FUSED: L2_LAUNCH(L2_FUSED) break;
      case L2_SCAT: L2_LAUNCH(L2_SCAT) break;
      default: L2_LAUNCH(L2_SCAT_PARTIAL) break;
    }
#undef L2_LAUNCH
    FP_CUDA(cudaGetLastError());
    return FP_OK;
  };
  const std::vector<int64_t>& cb = p->l2cb;
  const int H = p->heavy, cs = p->cs;
  static const bool merge = [] {  // FP_L2B_MERGE=1: one launch per phase over all blocks (measurement)
    const char* e = std::getenv("FP_L2B_MERGE");
    return e && std::atoi(e) != 0;
  }();
  auto others = [&](int mode) -> fp_status {  // every block but the fused one
    if (merge) {
      fp_status st = pass(cb[0], cb[H], mode);
      return st != FP_OK ? st : pass(cb[H + 1], cb[cs], mode);
    }
    for (int b = 0; b < cs; ++b)
      if (b != H) {
        fp_status st = pass(cb[b], cb[b + 1], mode);
        if (st != FP_OK) return st;
      }
    return FP_OK;
  };
  // FP_L2B_PANELS=1 (measurement): the dot phase as ONE launch over the (row panel, block) list;
  // measured on K1 5.66 vs 5.58 ms for one launch per block (the warps of one launch drift
  // over more blocks than L2 holds), so per-block launches stay the default
  static const bool panels = [] {
    const char* e = std::getenv("FP_L2B_PANELS");
    return e && std::atoi(e) != 0;
  }();
  fp_status st = FP_OK;
  if (has_y) {
    st = (panels && p->dotlist) ? pass(0, p->ndot, L2_DOT, p->dotlist) : others(L2_DOT);
    if (st == FP_OK) st = pass(cb[H], cb[H + 1], L2_FUSED);
    if (st != FP_OK) return st;
  }
  const int gm = (int)std::min<int64_t>((m + tb - 1) / tb, (int64_t)di.sm_count * 8);
  if (f64)
    k_l2b_q<double><<<gm, tb, 0, s>>>(m, p->rowdot, (const double*)a.v, a.alpha, has_y ? 1 : 0);
  else
    k_l2b_q<float><<<gm, tb, 0, s>>>(m, p->rowdot, (const float*)a.v, a.alpha, has_y ? 1 : 0);
  FP_CUDA(cudaGetLastError());
  st = others(L2_SCAT);
  if (st == FP_OK) st = pass(cb[H], cb[H + 1], has_y ? L2_SCAT_PARTIAL : L2_SCAT);
  if (st == FP_OK) {
    const int gh = (int)std::max<int64_t>(1, std::min<int64_t>((p->nhitems + kL2NW - 1) / kL2NW, (int64_t)di.sm_count * 8));
    if (f64)
      k_l2b_hot<double><<<gh, kL2BS, 0, s>>>(p->hitems, p->nhitems, p->hrow, (const double*)p->hval, p->hcol,
                                             p->rowdot, (double*)a.w);
    else
      k_l2b_hot<float><<<gh, kL2BS, 0, s>>>(p->hitems, p->nhitems, p->hrow, (const float*)p->hval, p->hcol,
                                            p->rowdot, (float*)a.w);
    FP_CUDA(cudaGetLastError());
  }
  return st;
}

void l2block_launch(const Packed* p, fp_launch* L) {
  *L = fp_launch{};
  L->variant = FP_VAR_CSR_L2BLOCK;
  L->vs = 32;
  L->tl = kL2Win;
  L->bs = kL2BS;
  L->grid = device_info(current_device()).sm_count * 8;
  L->cluster = p->cs;
  L->smem_bytes = kL2NW * kL2HeavyRows * 8;
  L->blocks_per_sm = 8;
  cudaFuncAttributes fa{};
  const void* f = p->dtype == FP_F64 ? (const void*)k_l2b<double, L2_FUSED> : (const void*)k_l2b<float, L2_FUSED>;
  if (cudaFuncGetAttributes(&fa, f) == cudaSuccess) L->regs_per_thread = fa.numRegs;
  else cudaGetLastError();
}

}  // namespace fp
