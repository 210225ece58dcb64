// csr_l2block.cu -- variant 20 (FP_VAR_CSR_L2BLOCK): Eq. (1) on a packed copy of a CSR matrix
// whose y and w are too wide for the shared memory of a CTA group (variant 19): the KDD-shaped
// ultra-wide case (Table 4: KDD2010 has n = 29.9M columns).
//
// Why.  With n = 29.9M fp64, y and w are 240 MB each: every nonzero of the flat path (variant 7)
// is a random 32-byte gather of y plus a random red.global into w that mostly miss the 126 MB
// L2, so the pass is bound by random HBM sectors (K1: 42 ms, 0.022 of the copy peak).  Split
// the COLUMNS into L2-sized blocks instead (bw = 2M fp64 columns: y and w of a block are 32 MB)
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
// 256 entries and 64 consecutive rows (one 8-entry-per-lane register window; a chunk never
// crosses a 64-row group); a row with more than 256 entries in a block becomes a run of
// "partial" chunks of 256.  Entry word = column in block | row in chunk << 26; chunks padded to
// 8 entries (32-byte aligned 256-bit loads).  Descriptor per chunk: (offset / 8, length | rows
// << 25, first row, flags).
#include <algorithm>
#include <cstdlib>
#include <new>
#include <vector>

#include <cub/device/device_scan.cuh>

#include "kernels.cuh"

namespace fp {

namespace {

constexpr int kL2Win = 256;                 // entries per chunk (one window, 8 per lane)
constexpr int kL2Rows = 64;                 // rows per chunk / per row group
constexpr int kL2RidShift = 26;             // entry word: column in block | row in chunk << 26
constexpr uint32_t kL2ColMask = (1u << kL2RidShift) - 1u;
constexpr uint32_t kL2PadWord = 63u << kL2RidShift;  // padding: column 0 (never read), row 63, value 0
constexpr unsigned kL2Partial = 1u;         // desc.w: one piece of a row longer than a window
constexpr int kL2MaxBlocks = 64;
constexpr int kL2BS = 256;
constexpr int kL2NW = kL2BS / 32;

enum { L2_DOT = 0, L2_FUSED = 1, L2_SCAT = 2, L2_SCAT_PARTIAL = 3 };

struct L2Args {
  const uint4* desc;    // this block's chunks
  int64_t nch;
  int64_t col0;         // first column of the block
  const uint32_t* cr;
  const void* val;      // T
  const void* y;        // T, the full vector
  const void* v;        // T or NULL (= 1)
  double alpha;
  double* p;            // [m]: row dots, q after k_l2b_q
  void* w;              // T
};

// 8 consecutive entries (32-byte aligned): streamed once, evict-first in L2 (the blocks of y
// and w are what L2 should keep)
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
// y of the block: kept in L2 (an evict_last cache policy), not in L1 (little reuse per SM)
__device__ __forceinline__ uint64_t l2_keep_policy() {
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ float l2_ldy(const float* p, uint64_t pol) {
  float v;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ double l2_ldy(const double* p, uint64_t pol) {
  double v;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
  return v;
}

// One pass over the chunks of one column block (a warp per chunk, grid-stride).
template <typename T, int MODE>
__global__ void __launch_bounds__(kL2BS) k_l2b(const L2Args a) {
  __shared__ double s_rs[kL2NW][kL2Rows];
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  double* rs = s_rs[wi];
  const T* __restrict__ y = reinterpret_cast<const T*>(a.y) + a.col0;
  const T* __restrict__ vv = reinterpret_cast<const T*>(a.v);
  const T* __restrict__ val = reinterpret_cast<const T*>(a.val);
  T* w = reinterpret_cast<T*>(a.w) + a.col0;
  double* p = a.p;
  const uint64_t keep = l2_keep_policy();
  const int64_t nw = (int64_t)gridDim.x * kL2NW;
  for (int64_t c = (int64_t)blockIdx.x * kL2NW + wi; c < a.nch; c += nw) {
    const uint4 D = __ldg(a.desc + c);
    const bool partial = (D.w & kL2Partial) != 0;
    if (MODE == L2_SCAT_PARTIAL && !partial) continue;
    const int len = (int)(D.y & 0x1FFFFFFu), rows = (int)(D.y >> 25);
    const int64_t r0 = (int64_t)D.z;
    const int o = 8 * lane;
    uint32_t cw[8];
    T xv[8];
    if (o < len) {
      const int64_t e0 = (int64_t)D.x * 8 + o;
      l2_ldc(a.cr + e0, cw);
      l2_ldv(val + e0, xv);
    } else {
#pragma unroll
      for (int e = 0; e < 8; ++e) cw[e] = kL2PadWord, xv[e] = T(0);
    }
    bool fused_scatter = false;
    if constexpr (MODE == L2_DOT || MODE == L2_FUSED) {
      // Eq. (2) on the window: in-lane runs of a row, then one bounded segmented scan across
      // lanes; each row's window sum lands in rs[row] exactly once
      rs[lane] = 0.0;
      rs[lane + 32] = 0.0;
      __syncwarp();
      T cs_[8];
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const T pr = o + e < len ? xv[e] * l2_ldy(y + (cw[e] & kL2ColMask), keep) : T(0);
        cs_[e] = (e == 0 || (cw[e] >> kL2RidShift) != (cw[e - 1] >> kL2RidShift)) ? pr : cs_[e - 1] + pr;
      }
      const int last = (int)(cw[7] >> kL2RidShift);
      int prev = __shfl_up_sync(0xffffffffu, last, 1);
      if (lane == 0) prev = -1;
      const bool h0 = (int)(cw[0] >> kL2RidShift) != prev;
      bool seen = h0;
#pragma unroll
      for (int e = 0; e < 7; ++e) {
        const bool h = (cw[e + 1] >> kL2RidShift) != (cw[e] >> kL2RidShift);
        if (h && seen) rs[cw[e] >> kL2RidShift] = (double)cs_[e];
        seen |= h;
      }
      T P = cs_[7];
#pragma unroll
      for (int e = 7; e >= 1; --e)
        if ((cw[e] >> kL2RidShift) != (cw[e - 1] >> kL2RidShift)) P = cs_[e - 1];
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
      if (seen) rs[last] = (double)(cs_[7] + rn);
      __syncwarp();
      if (MODE == L2_DOT || partial) {
        // the block's share of the row dots (a partial chunk: its piece of one long row)
        if (lane < rows) atomicAdd(p + r0 + lane, rs[lane]);
        if (lane + 32 < rows) atomicAdd(p + r0 + lane + 32, rs[lane + 32]);
      } else {
        // the heaviest block, processed last: p complete -> q = alpha v p, kept for the scatter
        for (int k = lane; k < rows; k += 32) {
          const double pt = p[r0 + k] + rs[k];
          p[r0 + k] = pt;
          const double vr = vv ? (double)vv[r0 + k] : 1.0;
          rs[k] = a.alpha * (vr * pt);
        }
        fused_scatter = true;
      }
    } else {
      // q of the chunk's rows (k_l2b_q converted p in place)
      for (int k = lane; k < rows; k += 32) rs[k] = p[r0 + k];
    }
    if (MODE == L2_SCAT || MODE == L2_SCAT_PARTIAL || fused_scatter) {
      __syncwarp();
      // Eq. (3) from the registers that hold the window: one red per nonzero into the block of w
#pragma unroll
      for (int e = 0; e < 8; ++e)
        if (o + e < len) atomicAdd(w + (cw[e] & kL2ColMask), (T)((double)xv[e] * rs[cw[e] >> kL2RidShift]));
    }
    __syncwarp();
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
// (1) entries of row r in block b: cnt[b m + r] (zeroed before)
__global__ void k_l2b_count(int64_t m, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ colidx,
                            int64_t bw, uint32_t* __restrict__ cnt) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = rowptr[r + 1];
    for (int64_t i = rowptr[r]; i < e; ++i) cnt[(int64_t)(colidx[i] / bw) * m + r] += 1u;
  }
}

// (2) the chunks of one (block, 64-row group): a thread walks the group's rows.  COUNT: number
// of chunks and padded entries; WRITE: the descriptors, and per (block, row) the entry offset
// of the row's first block-b entry and its row-in-chunk.
template <bool WRITE>
__global__ void k_l2b_walk(int64_t m, int cs, const uint32_t* __restrict__ cnt, int64_t* __restrict__ nchunk,
                           int64_t* __restrict__ nent, const int64_t* __restrict__ cbase,
                           const int64_t* __restrict__ ebase, uint4* __restrict__ desc, uint32_t* __restrict__ rowoff,
                           uint8_t* __restrict__ rid) {
  const int64_t ng = (m + kL2Rows - 1) / kL2Rows;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < (int64_t)cs * ng;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int b = (int)(t / ng);
    const int64_t g = t % ng;
    int64_t ci = WRITE ? cbase[t] : 0, ei = WRITE ? ebase[t] : 0;
    int64_t nc = 0, ne = 0;
    int64_t r0 = -1;
    int len = 0;
    auto emit = [&](int64_t first, int rows, int l, unsigned flags) {
      if (WRITE) desc[ci++] = make_uint4((unsigned)(ei / 8), (unsigned)l | ((unsigned)rows << 25), (unsigned)first, flags);
      ++nc;
      const int64_t al = (l + 7) & ~7;
      ne += al;
      ei += al;
    };
    int64_t last_row = -1;
    auto flush = [&]() {
      if (r0 >= 0) emit(r0, (int)(last_row - r0 + 1), len, 0u);
      r0 = -1;
      len = 0;
    };
    for (int i = 0; i < kL2Rows && g * kL2Rows + i < m; ++i) {
      const int64_t r = g * kL2Rows + i;
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
      if (r0 >= 0 && len + (int)c > kL2Win) flush();
      if (r0 < 0) r0 = r;
      if (WRITE) {
        rowoff[(int64_t)b * m + r] = (uint32_t)(ei + len);
        rid[(int64_t)b * m + r] = (uint8_t)(r - r0);
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

// (3) the entries: a thread per row, running count per block (stable order: non-canonical rows
// are packed as given, reading R7)
template <typename V>
__global__ void k_l2b_scatter(int64_t m, int cs, int64_t bw, const int64_t* __restrict__ rowptr,
                              const int32_t* __restrict__ colidx, const V* __restrict__ val,
                              const uint32_t* __restrict__ rowoff, const uint8_t* __restrict__ rid,
                              uint32_t* __restrict__ cr, V* __restrict__ pval) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    uint32_t k[kL2MaxBlocks];
    for (int b = 0; b < cs; ++b) k[b] = 0;
    const int64_t e = rowptr[r + 1];
    for (int64_t i = rowptr[r]; i < e; ++i) {
      const int col = colidx[i];
      const int b = (int)(col / bw);
      const int64_t pos = (int64_t)rowoff[(int64_t)b * m + r] + k[b]++;
      cr[pos] = (uint32_t)(col - b * bw) | ((uint32_t)rid[(int64_t)b * m + r] << kL2RidShift);
      pval[pos] = val[i];
    }
  }
}

__global__ void k_l2b_fill(int64_t n, uint32_t* __restrict__ p, uint32_t v) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}

}  // namespace

// columns per L2 block: y and w of a block take 32 MB (fp64: 2M columns, fp32: 4M); FP_L2B_BW
// (measurement / tests) overrides; at most kL2MaxBlocks blocks
int64_t l2block_bw(int64_t n, fp_dtype dt) {
  int64_t bw = dt == FP_F64 ? (int64_t)1 << 21 : (int64_t)1 << 22;
  if (const char* e = std::getenv("FP_L2B_BW")) bw = std::max<int64_t>(1, std::atoll(e));
  bw = std::max<int64_t>(bw, (n + kL2MaxBlocks - 1) / kL2MaxBlocks);
  return std::min<int64_t>(bw, (int64_t)kL2ColMask + 1);
}

fp_status l2block_build(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                        const void* val, fp_dtype dtype, Packed* p, cudaStream_t s) {
  const int64_t bw = l2block_bw(n, dtype);
  const int cs = (int)((n + bw - 1) / bw);
  FP_REQUIRE(cs <= kL2MaxBlocks, FP_ERR_UNSUPPORTED, "fp_csr_plan_pack: n = %lld needs more than %d L2 blocks",
             (long long)n, kL2MaxBlocks);
  const DeviceInfo& di = device_info(current_device());
  const int64_t ng = (m + kL2Rows - 1) / kL2Rows;
  const int64_t nt = (int64_t)cs * ng;
  uint32_t* cnt = nullptr;
  uint32_t* rowoff = nullptr;
  uint8_t* rid = nullptr;
  int64_t *nchunk = nullptr, *nent = nullptr, *cbase = nullptr, *ebase = nullptr;
  void* tmp = nullptr;
  auto cleanup = [&]() {
    for (void* b : {(void*)cnt, (void*)rowoff, (void*)rid, (void*)nchunk, (void*)nent, (void*)cbase, (void*)ebase, tmp})
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
  const int grid_r = (int)std::min<int64_t>((m + tb - 1) / tb, (int64_t)di.sm_count * 32);
  const int grid_t = (int)std::min<int64_t>((nt + tb - 1) / tb, (int64_t)di.sm_count * 32);
  L2_TRY(cudaMalloc((void**)&cnt, (size_t)cs * m * 4), "alloc");
  L2_TRY(cudaMemsetAsync(cnt, 0, (size_t)cs * m * 4, s), "memset");
  k_l2b_count<<<grid_r, tb, 0, s>>>(m, rowptr, colidx, bw, cnt);
  L2_TRY(cudaMalloc((void**)&nchunk, (size_t)(nt + 1) * 8), "alloc");
  L2_TRY(cudaMalloc((void**)&nent, (size_t)(nt + 1) * 8), "alloc");
  L2_TRY(cudaMalloc((void**)&cbase, (size_t)(nt + 1) * 8), "alloc");
  L2_TRY(cudaMalloc((void**)&ebase, (size_t)(nt + 1) * 8), "alloc");
  L2_TRY(cudaMemsetAsync(nchunk + nt, 0, 8, s), "memset");
  L2_TRY(cudaMemsetAsync(nent + nt, 0, 8, s), "memset");
  k_l2b_walk<false><<<grid_t, tb, 0, s>>>(m, cs, cnt, nchunk, nent, nullptr, nullptr, nullptr, nullptr, nullptr);
  size_t tb_bytes = 0;
  L2_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb_bytes, nchunk, cbase, nt + 1, s), "scan");
  L2_TRY(cudaMalloc(&tmp, tb_bytes), "alloc");
  L2_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb_bytes, nchunk, cbase, nt + 1, s), "scan");
  L2_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb_bytes, nent, ebase, nt + 1, s), "scan");
  // chunk ranges of the blocks (block b's chunks are [cbase[b ng], cbase[(b + 1) ng])) and the
  // entries of every block (the heaviest is processed last, fused)
  std::vector<int64_t> hcb(cs + 1), heb(cs + 1);
  for (int b = 0; b <= cs; ++b) {
    L2_TRY(cudaMemcpyAsync(&hcb[b], cbase + (int64_t)b * ng, 8, cudaMemcpyDeviceToHost, s), "copy");
    L2_TRY(cudaMemcpyAsync(&heb[b], ebase + (int64_t)b * ng, 8, cudaMemcpyDeviceToHost, s), "copy");
  }
  L2_TRY(cudaStreamSynchronize(s), "sync");
  const int64_t nch = hcb[cs], total = heb[cs];
  if (total >= (int64_t)UINT32_MAX) return fail(cudaErrorInvalidValue, "too many entries for 32-bit offsets");
  L2_TRY(cudaMalloc((void**)&p->tile_desc, (size_t)std::max<int64_t>(nch, 1) * sizeof(uint4)), "alloc");
  L2_TRY(cudaMalloc((void**)&rowoff, (size_t)cs * m * 4), "alloc");
  L2_TRY(cudaMalloc((void**)&rid, (size_t)cs * m), "alloc");
  k_l2b_walk<true><<<grid_t, tb, 0, s>>>(m, cs, cnt, nullptr, nullptr, cbase, ebase, p->tile_desc, rowoff, rid);
  const int64_t cap = total + 8;
  const size_t vs = dtype_size(dtype);
  L2_TRY(cudaMalloc((void**)&p->cr, (size_t)cap * 4), "alloc");
  L2_TRY(cudaMalloc((void**)&p->val, (size_t)cap * vs), "alloc");
  k_l2b_fill<<<(int)std::min<int64_t>((cap + tb - 1) / tb, (int64_t)di.sm_count * 32), tb, 0, s>>>(cap, p->cr,
                                                                                                   kL2PadWord);
  L2_TRY(cudaMemsetAsync(p->val, 0, (size_t)cap * vs, s), "memset");
  if (dtype == FP_F64)
    k_l2b_scatter<double><<<grid_r, tb, 0, s>>>(m, cs, bw, rowptr, colidx, (const double*)val, rowoff, rid, p->cr,
                                                (double*)p->val);
  else
    k_l2b_scatter<float><<<grid_r, tb, 0, s>>>(m, cs, bw, rowptr, colidx, (const float*)val, rowoff, rid, p->cr,
                                               (float*)p->val);
  L2_TRY(cudaMalloc((void**)&p->rowdot, (size_t)std::max<int64_t>(m, 1) * 8), "alloc");
  L2_TRY(cudaStreamSynchronize(s), "sync");
#undef L2_TRY
  cleanup();
  p->mode = 1;
  p->cs = cs;
  p->bw = (int)bw;
  p->ntiles = nch;
  p->entries = total;
  p->groups = 0;
  p->l2cb.assign(hcb.begin(), hcb.end());
  int heavy = 0;
  for (int b = 1; b < cs; ++b)
    if (heb[b + 1] - heb[b] > heb[heavy + 1] - heb[heavy]) heavy = b;
  p->heavy = heavy;
  (void)nnz;
  return FP_OK;
}

fp_status l2block_exec(Packed* p, const PatternArgs& a, cudaStream_t s) {
  const DeviceInfo& di = device_info(current_device());
  const bool has_y = a.y != nullptr;
  const int64_t m = p->m, n = p->n;
  const int tb = 256;
  const int gn = (int)std::min<int64_t>((n + tb - 1) / tb, (int64_t)di.sm_count * 8);
  if (p->dtype == FP_F64)
    k_l2b_init<double><<<gn, tb, 0, s>>>(n, (double*)a.w, (const double*)a.z, a.beta, a.add_beta_z ? 1 : 0,
                                         a.accumulate ? 1 : 0);
  else
    k_l2b_init<float><<<gn, tb, 0, s>>>(n, (float*)a.w, (const float*)a.z, a.beta, a.add_beta_z ? 1 : 0,
                                        a.accumulate ? 1 : 0);
  FP_CUDA(cudaGetLastError());
  if (has_y) FP_CUDA(cudaMemsetAsync(p->rowdot, 0, (size_t)m * 8, s));
  auto pass = [&](int b, int mode) -> fp_status {
    L2Args k{};
    k.nch = p->l2cb[b + 1] - p->l2cb[b];
    if (k.nch == 0) return FP_OK;
    k.desc = p->tile_desc + p->l2cb[b];
    k.col0 = (int64_t)b * p->bw;
    k.cr = p->cr;
    k.val = p->val;
    k.y = a.y;
    k.v = a.v;
    k.alpha = a.alpha;
    k.p = p->rowdot;
    k.w = a.w;
    const int grid = (int)std::min<int64_t>((k.nch + kL2NW - 1) / kL2NW, (int64_t)di.sm_count * 8);
    const bool f64 = p->dtype == FP_F64;
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
  fp_status st = FP_OK;
  if (has_y) {
    for (int b = 0; b < p->cs && st == FP_OK; ++b)
      if (b != p->heavy) st = pass(b, L2_DOT);
    if (st == FP_OK) st = pass(p->heavy, L2_FUSED);
    if (st != FP_OK) return st;
  }
  const int gm = (int)std::min<int64_t>((m + tb - 1) / tb, (int64_t)di.sm_count * 8);
  if (p->dtype == FP_F64)
    k_l2b_q<double><<<gm, tb, 0, s>>>(m, p->rowdot, (const double*)a.v, a.alpha, has_y ? 1 : 0);
  else
    k_l2b_q<float><<<gm, tb, 0, s>>>(m, p->rowdot, (const float*)a.v, a.alpha, has_y ? 1 : 0);
  FP_CUDA(cudaGetLastError());
  for (int b = 0; b < p->cs && st == FP_OK; ++b)
    if (b != p->heavy) st = pass(b, L2_SCAT);
  if (st == FP_OK) st = pass(p->heavy, has_y ? L2_SCAT_PARTIAL : L2_SCAT);
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
  L->smem_bytes = kL2NW * kL2Rows * 8;
  L->blocks_per_sm = 8;
  cudaFuncAttributes fa{};
  const void* f = p->dtype == FP_F64 ? (const void*)k_l2b<double, L2_FUSED> : (const void*)k_l2b<float, L2_FUSED>;
  if (cudaFuncGetAttributes(&fa, f) == cudaSuccess) L->regs_per_thread = fa.numRegs;
  else cudaGetLastError();
}

}  // namespace fp
