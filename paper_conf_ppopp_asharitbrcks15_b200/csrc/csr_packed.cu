// csr_packed.cu -- variant 19 (FP_VAR_CSR_PACKED): Eq. (1) on a column-blocked copy of a CSR
// matrix whose y and partial w do not fit one SM (C4: n = 1e5 fp32), X read once per call.
//
// Why.  For n beyond one SM's shared memory every nonzero costs a random access to the
// L2-resident y and w (variants 7/16: 2e9 reds + 2e9 gathers, ~11 ms of issuing cost on
// sm_100a) or a message round trip through HBM (variant 17: 12 GB written + read).  Split the
// COLUMNS instead: a group of CS CTAs (one per SM) holds y and the partial w of column block k
// (CTA k) in shared memory, so every gather and every scatter is a shared-memory access (y as
// fp32, w as 32-bit fixed point with native integer atomics).  Each CTA streams only the
// nonzeros of its block; the row dots of Eq. (2) are completed by summing the CS block partials
// of each row (a 32-row exchange per tile through L2), then Eq. (3) scatters the terms from
// the registers that still hold the row (a7: scale-back from the same registers).
//
// The copy (fp_csr_plan_pack, once per matrix, amortised over calls as the paper amortises
// its baseline's transpose): for each column block k the block-k segments of every row
// stored contiguously; rows grouped into TILES (<= 64 rows, every block segment <= 1024
// entries, or one long row); each entry one 32-bit word (byte offset of the column inside the
// block | row inside the tile << 26) + its value; every segment padded to 8 entries (32 bytes).  The row structure of a
// tile is therefore in the entries themselves: no rowptr search and no head masks per call.
//
// One call: k_pk (the whole Eq. 1 pass, cooperative launch: the CTAs of a group wait on each
// other) + k_pk_finalize (sums the groups' partials in a fixed order, adds beta z).
//
// Fixed point (reading R25): CTA c adds every term t = x q as round(t / quantum_c)
// into a 32-bit shared accumulator, quantum_c = 2^(E_c - 26), E_c = (exponent of the largest
// finite |t| of the CTA's first tile round) + H (H = 3 headroom bits), so the first round's
// terms are int32s of magnitude < 2^26 (error <= quantum_c / 2 per term) and terms up to
// 2^(E_c + 5) (power-law rows: |q| grows like sqrt(row length)) still fit an int32 exactly;
// an add that wraps the int32 sum is detected from the returned old value and carries 2^32
// quanta into an fp64 spill vector; larger or non-finite terms go to the spill themselves.  The partials are
// converted exactly to fp64 and summed in group order: deterministic except for spills.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include <cub/device/device_scan.cuh>

#include "kernels.cuh"

namespace fp {

namespace {

constexpr int kPkBS = 1024;
constexpr int kPkNW = kPkBS / 32;
constexpr int kPkRows = 64;           // rows per tile (at most)
constexpr int kPkLong = 1024;         // a block segment longer than this makes its row a tile of its own
constexpr int kPkRowCost = 4;         // work of a row in entries (warp partition)
constexpr int kPkStatic = 27 * 1024;  // static shared memory reserve of k_pk
constexpr int kPkRing = 4;            // tile descriptors a warp keeps between DOT and SCATTER (>= D + 1)
constexpr unsigned kPkOffMask = 0x3FFFFu;  // entry word: byte offset of the column in the block (18 bits)
constexpr int kPkRidShift = 26;            //             | row in tile << 26 (rid * 4 = word >> 24)
constexpr float kPkCap = 2147483520.f;     // 2^31 - 128: |term / quantum| below this is an exact-range int32
                                           // (one int32 wrap at most per add: detected, carried)

template <int D>
struct PkSlots {
  static constexpr int NS = 2 * D + 2;  // exchange slots per warp: a slot is rewritten only after
};                                      // every CTA of the group consumed its tile

struct PkArgs {
  int64_t n;
  int bw;                        // columns per block (block k = [k bw, min(n, (k+1) bw)))
  int groups;
  int64_t ntiles;
  int64_t padidx;                // 8 padding entries (the inactive lanes' loads)
  const uint4* tile_desc;        // [cs][ntiles]: (offset / 8, length | rows << 25, first row, max |x| bits)
  const int32_t* wtile;          // [groups * 32 + 1]: first tile of each warp-quad
  const uint32_t* cr;            // packed entry words
  const float* val;
  const float* y;
  const float* v;
  float alpha;
  int hbits;                     // headroom bits of the fixed-point cap
  unsigned long long* xch;       // exchange slots [groups][32 warps][NS][cs + 1][64 rows]
  const unsigned* epoch;         // call counter (advanced by k_pk_finalize)
  double* part;                  // [groups][n]
  double* spill;                 // [cs][bw + 1], all-zero between calls
  int nap;                       // ns a warp sleeps between polls of the exchange (0: spin)
  int pf;                        // L2 prefetch of the next tile: 0 none, 1 per-lane lines, 2 bulk (FP_PK_PF)
  unsigned long long* trace;     // FP_PK_TRACE: per warp (start, end of the pass, tiles, prologue end)
};

// 8 consecutive entries (32 bytes).  KEEP: the dot's read asks L2 to keep the segment
// (evict_last) for the scatter's re-read, which releases it (evict_first)
#define PK_LD8(Q)                                                                                      \
  asm("ld.global.nc.L1::no_allocate" Q ".v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"                      \
      : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]), "=r"(c[4]), "=r"(c[5]), "=r"(c[6]), "=r"(c[7])  \
      : "l"(pc));                                                                                      \
  asm("ld.global.nc.L1::no_allocate" Q ".v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"                      \
      : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]), "=f"(x[4]), "=f"(x[5]), "=f"(x[6]), "=f"(x[7])  \
      : "l"(pv))
template <bool KEEP>
__device__ __forceinline__ void pk_ld8(const uint32_t* pc, const float* pv, uint32_t (&c)[8], float (&x)[8]) {
  if constexpr (KEEP) {
    PK_LD8(".L2::evict_last");
  } else {
    PK_LD8(".L2::evict_first");
  }
}
#undef PK_LD8
__device__ __forceinline__ void st_relaxed_gpu(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_gpu2(unsigned long long* p, unsigned long long a, unsigned long long b) {
  asm volatile("st.relaxed.gpu.global.v2.b64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}
// two 8-byte words; each is single-copy atomic on its own (its value and tag consistent)
__device__ __forceinline__ void ld_relaxed_gpu2(const unsigned long long* p, unsigned long long& a,
                                                unsigned long long& b) {
  asm volatile("ld.relaxed.gpu.global.v2.b64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed_gpu(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned pk_lanemask_lt() {
  unsigned r;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
  return r;
}
// shared memory through 32-bit addresses (y and q are read-only while read).  No "memory"
// clobbers: they would pin the next step's global loads behind this step's atomics; the
// volatile ones keep their order among themselves, __syncwarp orders them across lanes.
__device__ __forceinline__ float pk_lds(unsigned addr) {
  float v;
  asm("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ float pk_lds_v(unsigned addr) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ void pk_sts(unsigned addr, float v) {
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(addr), "f"(v));
}
__device__ __forceinline__ int pk_atom_add(unsigned addr, int v) {
  int old;
  asm volatile("atom.shared.add.s32 %0, [%1], %2;" : "=r"(old) : "r"(addr), "r"(v));
  return old;
}
__device__ __forceinline__ void pk_prefetch_l2(const void* p) {
  asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(p));
}
// (acc << 1) | (x >> 31): collect one sign bit per entry
__device__ __forceinline__ unsigned pk_push_sign(unsigned acc, unsigned x) { return __funnelshift_l(x, acc, 1); }

// typed shared-memory accesses (the single-block pass, fp32 / fp64)
__device__ __forceinline__ double pk_lds(unsigned addr, double) {
  double v;
  asm("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ float pk_lds(unsigned addr, float) { return pk_lds(addr); }
__device__ __forceinline__ double pk_lds_v(unsigned addr, double) {
  double v;
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ float pk_lds_v(unsigned addr, float) { return pk_lds_v(addr); }
__device__ __forceinline__ void pk_sts(unsigned addr, double v) {
  asm volatile("st.shared.f64 [%0], %1;" ::"r"(addr), "d"(v));
}
__device__ __forceinline__ unsigned pk_atom_addu(unsigned addr, unsigned v) {
  unsigned old;
  asm volatile("atom.shared.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(addr), "r"(v));
  return old;
}
// 8 values of a window: fp32 one 32-byte load, fp64 two
template <bool KEEP>
__device__ __forceinline__ void pk_ldv(const float* pv, float* x) {
  if constexpr (KEEP)
    asm("ld.global.nc.L1::no_allocate.L2::evict_last.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]), "=f"(x[4]), "=f"(x[5]), "=f"(x[6]), "=f"(x[7])
        : "l"(pv));
  else
    asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]), "=f"(x[4]), "=f"(x[5]), "=f"(x[6]), "=f"(x[7])
        : "l"(pv));
}
template <bool KEEP>
__device__ __forceinline__ void pk_ldv(const double* pv, double* x) {
  if constexpr (KEEP) {
    asm("ld.global.nc.L1::no_allocate.L2::evict_last.v4.f64 {%0,%1,%2,%3}, [%4];"
        : "=d"(x[0]), "=d"(x[1]), "=d"(x[2]), "=d"(x[3]) : "l"(pv));
    asm("ld.global.nc.L1::no_allocate.L2::evict_last.v4.f64 {%0,%1,%2,%3}, [%4];"
        : "=d"(x[4]), "=d"(x[5]), "=d"(x[6]), "=d"(x[7]) : "l"(pv + 4));
  } else {
    asm("ld.global.nc.L1::no_allocate.L2::evict_first.v4.f64 {%0,%1,%2,%3}, [%4];"
        : "=d"(x[0]), "=d"(x[1]), "=d"(x[2]), "=d"(x[3]) : "l"(pv));
    asm("ld.global.nc.L1::no_allocate.L2::evict_first.v4.f64 {%0,%1,%2,%3}, [%4];"
        : "=d"(x[4]), "=d"(x[5]), "=d"(x[6]), "=d"(x[7]) : "l"(pv + 4));
  }
}
template <bool KEEP>
__device__ __forceinline__ void pk_ldc(const uint32_t* pc, uint32_t* c) {
  if constexpr (KEEP)
    asm("ld.global.nc.L1::no_allocate.L2::evict_last.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]), "=r"(c[4]), "=r"(c[5]), "=r"(c[6]), "=r"(c[7])
        : "l"(pc));
  else
    asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=r"(c[0]), "=r"(c[1]), "=r"(c[2]), "=r"(c[3]), "=r"(c[4]), "=r"(c[5]), "=r"(c[6]), "=r"(c[7])
        : "l"(pc));
}


struct Pk1Args {
  int64_t m;
  int64_t n;
  int64_t ntiles;
  int ns;                        // tile slots per warp in the shared-memory ring (0: no ring)
  const uint4* tile_desc;        // [ntiles]
  const int32_t* wtile;          // [ctas * 32 + 1]
  const uint32_t* cr;
  const void* val;               // T
  const void* y;                 // T
  const void* v;                 // T
  double alpha;
  int hbits;
  double* part;                  // [ctas][n]
  double* spill;                 // [n + 1]
};

constexpr int kPk1MaxNS = 4;
#ifndef FP_PK1_FG
#define FP_PK1_FG 8
#endif
constexpr int kPk1FG = FP_PK1_FG;  // fp64 scatter: terms whose low limbs are added before their high limbs
constexpr uint32_t pk1_pad_word(int n) { return ((uint32_t)n * 4u) | ((uint32_t)(kPkRows - 1) << kPkRidShift); }

__device__ __forceinline__ uint4 pk_lds128(unsigned addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}
__device__ __forceinline__ uint4 pk_ldg128(const void* p) {
  uint4 v;
  asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
// 16 bytes -> 4 fp32 / 2 fp64 values of a window
__device__ __forceinline__ void pk_put(float* x, const uint4& u) {
  x[0] = __uint_as_float(u.x), x[1] = __uint_as_float(u.y), x[2] = __uint_as_float(u.z), x[3] = __uint_as_float(u.w);
}
__device__ __forceinline__ void pk_put(double* x, const uint4& u) {
  x[0] = __hiloint2double((int)u.y, (int)u.x), x[1] = __hiloint2double((int)u.w, (int)u.z);
}

// The single-block pass (one column block, CS = 1: y and the whole partial w in each CTA's
// shared memory, no exchange).  Every tile (<= 256 entries) is loaded ONCE: the dot, q and the
// scatter all run from the registers that hold it (a7) -- X is read from HBM once.
//
// Staging (round 2c; fp64 -- fp32's 32 warps hide the load themselves): each warp keeps a
// ring of NS tile slots in shared memory, filled by TMA bulk copies (cp.async.bulk of the
// tile's column words, values and the v of its rows, completion on the slot's mbarrier) NS
// tiles ahead of the tile being processed, so the HBM latency of the stream is off the warp's
// critical path (the round-2b pass loaded every tile into registers itself: 20 % of its stall
// samples waited on that load, ncu r02c).  Descriptors arrive in batches of 16 by cp.async.  The window of a tile is stored lane-interleaved (pack
// time, k_pk_interleave): the 16-byte piece k of lane l's 8 entries at (k G + l) 16 bytes, G =
// the tile's groups of 8 -- a warp's 16-byte shared loads then touch 8 distinct bank quads per
// phase (conflict-free), and lane l still holds the logical entries 8l..8l+7.  A longer segment
// (one long row) is streamed from global memory by the dot and re-read by the scatter.  fp32:
// the partial w is one int32 per column (reading R25); fp64: a 64-bit fixed point in two
// native int32 limbs, quantum 2^(E - 50) (the low limb's returned value gives the carry; a
// wrap of the high limb carries 2^64 quanta into the spill).
template <typename T, int YM, int BS1>
__global__ void __launch_bounds__(BS1, 1) k_pk1(const Pk1Args a) {
  constexpr int NW1 = BS1 / 32;
  constexpr bool F64 = sizeof(T) == 8;
  constexpr int QB = F64 ? 50 : 26;  // bits of the first round's largest term
  constexpr int TS = (int)sizeof(T);
  // a slot: cw (256 words) | values (256) | v of the tile's rows (a 16-byte aligned superset)
  constexpr int SLOT_CW = 256 * 4, SLOT_V = 256 * (4 + TS), SLOT = SLOT_V + kPkRows * TS + 16;
  constexpr int NV = 8 * TS / 16;    // 16-byte pieces of a lane's 8 values
  extern __shared__ __align__(128) unsigned char pk_smem[];
  __shared__ unsigned s_tmax;
  __shared__ uint64_t s_bar[NW1][kPk1MaxNS];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int n = (int)a.n;
  const int NS = a.ns;
  // dynamic: [ring: NW1 x NS slots of (cw: 256 words | val: 256 values)][descriptors: NW1 x 2
  // batches x 16][rs | q / quantum | q: 3 x NW1 warps x 64 rows][y: n + 1 (y[n] = 0: padding
  // entries)][lo: n + 33][hi (fp64): n + 33]
  unsigned char* ring = pk_smem + (size_t)warp * NS * SLOT;
  uint4* sdesc = reinterpret_cast<uint4*>(pk_smem + (size_t)NW1 * NS * SLOT) + warp * 32;
  T (*rs)[kPkRows] = reinterpret_cast<T (*)[kPkRows]>(pk_smem + (size_t)NW1 * NS * SLOT + (size_t)NW1 * 32 * 16);
  T (*qsm)[kPkRows] = rs + NW1;
  T (*qus)[kPkRows] = rs + 2 * NW1;
  T* y_s = reinterpret_cast<T*>(reinterpret_cast<unsigned char*>(rs) + (size_t)3 * NW1 * kPkRows * sizeof(T));
  const int ystride = YM ? (n + 4) & ~3 : 0;
  unsigned* lo = reinterpret_cast<unsigned*>(reinterpret_cast<unsigned char*>(y_s) + (size_t)ystride * sizeof(T));
  int* hi = reinterpret_cast<int*>(lo + ((n + 36) & ~3));
  for (int j = threadIdx.x; j <= n + 32; j += BS1) {
    if (YM && j <= n) y_s[j] = j < n ? reinterpret_cast<const T*>(a.y)[j] : T(0);
    lo[j] = 0u;
    if (F64) hi[j] = 0;
  }
  if (threadIdx.x == 0) s_tmax = 0u;
  if (lane == 0) {
    for (int s = 0; s < NS; ++s) fpd::mbar_init(&s_bar[warp][s], 1);
    fpd::fence_mbar_init();
  }
  __syncthreads();
  const unsigned ys_base = fpd::smem_u32(y_s), lo_base = fpd::smem_u32(lo), hi_base = fpd::smem_u32(hi);
  const unsigned rs_base = fpd::smem_u32(&rs[warp][0]), qs_base = fpd::smem_u32(&qsm[warp][0]),
                 qu_base = fpd::smem_u32(&qus[warp][0]), ring_base = fpd::smem_u32(ring);
  const int gq = (int)blockIdx.x * NW1 + warp;
  const int64_t t0 = a.wtile[gq];
  const int nt = a.wtile[gq + 1] - a.wtile[gq];
  const uint4* __restrict__ desc = a.tile_desc + t0;
  const uint32_t* __restrict__ crp = a.cr;
  const T* __restrict__ val = reinterpret_cast<const T*>(a.val);
  const T* __restrict__ vv = reinterpret_cast<const T*>(a.v);
  const T alpha = (T)a.alpha;
  double* const spill = a.spill;
  const uint32_t padw = pk1_pad_word(n);
  // v rides with the tile's copy when 16-byte aligned: rows whose v lies below vlim (the last
  // 16-byte boundary of v) come from the slot, the few beyond it from global memory
  const bool vring = vv != nullptr && NS > 0 && ((uintptr_t)vv & 15u) == 0;
  const int64_t vlim = ((int64_t)a.m * TS) & ~(int64_t)15;
  auto seg_len = [](const uint4& D) { return (int)(D.y & 0x1FFFFFFu); };
  auto seg_rows = [](const uint4& D) { return (int)(D.y >> 25); };

  // tile descriptors in shared memory (no registers held), batches of 16 (batch b in half b & 1),
  // one batch ahead: batch b + 1 is requested (cp.async, zero-filled beyond the warp's tiles)
  // when tile 16 b starts and waited for at tile 16 b + 8; tiles j .. j + NS (NS <= 8) resident
  const unsigned sdesc_base = fpd::smem_u32(sdesc);
  auto desc_req = [&](int b) {
    const int i = 16 * b + (lane & 15);
    if (lane < 16)
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(sdesc_base + 16u * ((b & 1) * 16 + lane)),
                   "l"(desc + (i < nt ? i : 0)), "r"(i < nt ? 16u : 0u)
                   : "memory");
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  auto desc_wait = [&]() {
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncwarp();
  };
  auto desc_of = [&](int i) { return pk_lds128(sdesc_base + 16u * (unsigned)(i & 31)); };
  desc_req(0);
  desc_wait();
  // fill slot s with tile i (a tile beyond the ring's window size, or none, only arrives)
  auto issue = [&](int i, int s) {
    if (i >= nt) return;
    const uint4 Di = desc_of(i);
    if (lane == 0) {
      const unsigned len = Di.y & 0x1FFFFFFu, len8 = (len + 7u) & ~7u;
      const unsigned cwb = len <= 256 ? len8 * 4u : 0u;
      int64_t v0b = (int64_t)Di.z * TS & ~(int64_t)15;
      const int64_t v1b = std::min<int64_t>(((int64_t)(Di.z + (Di.y >> 25)) * TS + 15) & ~(int64_t)15, vlim);
      const unsigned vb = (vring && cwb && v1b > v0b) ? (unsigned)(v1b - v0b) : 0u;
      uint64_t* b = &s_bar[warp][s];
      fpd::fence_proxy_async_smem();  // this warp's reads of the slot precede the copy's writes
      fpd::mbar_arrive_expect_tx(b, cwb + cwb / 4u * TS + vb);
      if (cwb) {
        unsigned char* slot = ring + (size_t)s * SLOT;
        const int64_t e0 = (int64_t)Di.x * 8;
        fpd::bulk_g2s(slot, crp + e0, cwb, b);
        fpd::bulk_g2s(slot + SLOT_CW, val + e0, cwb / 4u * TS, b);
        if (vb) fpd::bulk_g2s(slot + SLOT_V, reinterpret_cast<const unsigned char*>(vv) + v0b, vb, b);
      }
    }
  };
  // the lane's 8 entries of a window with G groups: 16-byte pieces at (k G + lane) 16 bytes
  auto win_smem = [&](int s, int G, uint32_t (&cw)[8], T (&xv)[8]) {
    const unsigned sb = ring_base + (unsigned)s * SLOT;
    if (lane < G) {
      const uint4 c0 = pk_lds128(sb + 16u * lane), c1 = pk_lds128(sb + 16u * (G + lane));
      cw[0] = c0.x, cw[1] = c0.y, cw[2] = c0.z, cw[3] = c0.w, cw[4] = c1.x, cw[5] = c1.y, cw[6] = c1.z, cw[7] = c1.w;
#pragma unroll
      for (int k = 0; k < NV; ++k) pk_put(xv + k * (16 / TS), pk_lds128(sb + SLOT_CW + 16u * (k * G + lane)));
    } else {
#pragma unroll
      for (int e = 0; e < 8; ++e) cw[e] = padw, xv[e] = T(0);
    }
  };
  auto win_glob = [&](const uint4& D, int s0, uint32_t (&cw)[8], T (&xv)[8]) {
    const int len8 = (seg_len(D) + 7) & ~7;
    const int G = min(32, (len8 - s0) >> 3);
    const int64_t e0 = (int64_t)D.x * 8 + s0;
    if (lane < G) {
      const uint4 c0 = pk_ldg128(crp + e0 + 4 * lane), c1 = pk_ldg128(crp + e0 + 4 * (G + lane));
      cw[0] = c0.x, cw[1] = c0.y, cw[2] = c0.z, cw[3] = c0.w, cw[4] = c1.x, cw[5] = c1.y, cw[6] = c1.z, cw[7] = c1.w;
#pragma unroll
      for (int k = 0; k < NV; ++k) pk_put(xv + k * (16 / TS), pk_ldg128(val + e0 + (16 / TS) * (k * G + lane)));
    } else {
#pragma unroll
      for (int e = 0; e < 8; ++e) cw[e] = padw, xv[e] = T(0);
    }
  };
  // y[col]: the entry word holds col * 4
  auto yaddr = [&](uint32_t w) { return ys_base + (F64 ? 2u : 1u) * (w & kPkOffMask); };
  auto qaddr = [&](unsigned base, uint32_t w) { return base + (F64 ? 2u : 1u) * (w >> 24); };

  // one window of the dot into rs: in-lane runs, then one bounded segmented scan across lanes
  auto dot_win = [&](const uint32_t (&cw)[8], const T (&xv)[8], int& carry) {
    T c[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      const T pr = xv[e] * pk_lds(yaddr(cw[e]), T(0));
      c[e] = (e == 0 || (cw[e] >> 24) != (cw[e - 1] >> 24)) ? pr : c[e - 1] + pr;
    }
    const int last = (int)(cw[7] >> 24);
    int prev = __shfl_up_sync(0xffffffffu, last, 1);
    if (lane == 0) prev = carry;
    const bool h0 = (int)(cw[0] >> 24) != prev;
    bool seen = h0;
#pragma unroll
    for (int e = 0; e < 7; ++e) {
      const bool h = (cw[e + 1] >> 24) != (cw[e] >> 24);
      if (h && seen) pk_sts(qaddr(rs_base, cw[e]), c[e]);
      seen |= h;
    }
    T P = c[7];
#pragma unroll
    for (int e = 7; e >= 1; --e)
      if ((cw[e] >> 24) != (cw[e - 1] >> 24)) P = c[e - 1];
    if (h0) P = T(0);
    const unsigned H = __ballot_sync(0xffffffffu, seen);
    const unsigned hl = H >> lane;
    const int dist = hl ? __ffs(hl) : 32 - lane;
    T r = P;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const T t2 = __shfl_down_sync(0xffffffffu, r, d);
      if (d < dist) r += t2;
    }
    T rn = __shfl_down_sync(0xffffffffu, r, 1);
    if (lane == 31) rn = T(0);
    if (seen) pk_sts(qaddr(rs_base, cw[7]), c[7] + rn);
    if (lane == 0 && !h0 && prev >= 0) {
      const unsigned ad = rs_base + (F64 ? 2 : 1) * (unsigned)prev;
      pk_sts(ad, pk_lds_v(ad, T(0)) + r);
    }
    carry = __shfl_sync(0xffffffffu, last, 31);
    __syncwarp();
  };

  double sc = 1.0;     // 2^(QB - E)
  double quantum = 0;  // 2^(E - QB)
  auto set_scale = [&](int e) {
    e = min(max(e, F64 ? -900 : -95), F64 ? 900 : 100);
    sc = ldexp(1.0, QB - e);
    quantum = ldexp(1.0, e - QB);
  };
  set_scale(0);

  // one window of the scatter: every x q into the fixed-point partial; terms beyond the
  // int32 / int64 range, non-finite terms and wraps spill (rare)
  // SAFE (the tile's max |x| times every |q / quantum| of its rows below the limb range, from the
  // plan's per-tile max |x|): no per-entry range checks -- only wraps can be rare
  auto scat_win = [&](const uint32_t (&cw)[8], const T (&xv)[8], int s0, int len, bool safe) {
    const unsigned dm = (s0 + 8 * lane < len) ? 0u : 4u * (lane + 1);  // lane's dummy beyond the segment
    unsigned rare = 0;
    auto body = [&](auto SAFE) {
      constexpr bool S = decltype(SAFE)::value;
      if constexpr (!F64) {
#pragma unroll
        for (int e = 0; e < 8; ++e) {
          const T ts = xv[e] * pk_lds(qaddr(qs_base, cw[e]), T(0));
          const unsigned off = dm + (cw[e] & kPkOffMask);
          const bool big = S ? false : !(fabsf(ts) < kPkCap);
          const int qi = big ? 0 : __float2int_rn(ts);
          const int old = pk_atom_add(lo_base + off, qi);
          const unsigned nw = (unsigned)old + (unsigned)qi;
          rare = (rare << 1) | (unsigned)(big | ((int)(((unsigned)old ^ nw) & ((unsigned)qi ^ nw)) < 0));
        }
      } else {
        // |term| < 2^62 quanta: both limbs always added (no branch); the high limb's wrap is
        // detected from its returned old value.  The low limbs of a group of PG terms go first:
        // a high limb's operand waits for its low limb's returned value (the carry) and the
        // volatile atomics keep program order, so alternating lo / hi per term would chain 16
        // shared-memory round trips per window
#pragma unroll
        for (int g0 = 0; g0 < 8; g0 += kPk1FG) {
          unsigned l[kPk1FG], ol[kPk1FG], off[kPk1FG];
          int hh[kPk1FG];
          bool big[kPk1FG];
#pragma unroll
          for (int k = 0; k < kPk1FG; ++k) {
            const int e = g0 + k;
            const T ts = xv[e] * pk_lds(qaddr(qs_base, cw[e]), T(0));
            off[k] = dm + (cw[e] & kPkOffMask);
            big[k] = S ? false : !(fabs(ts) < 4.6e18);
            const long long I = big[k] ? 0ll : __double2ll_rn(ts);
            l[k] = (unsigned)I;
            hh[k] = (int)(I >> 32);
          }
#pragma unroll
          for (int k = 0; k < kPk1FG; ++k) ol[k] = pk_atom_addu(lo_base + off[k], l[k]);
#pragma unroll
          for (int k = 0; k < kPk1FG; ++k) {
            const int h = hh[k] + ((ol[k] + l[k] < ol[k]) ? 1 : 0);
            const int oh = pk_atom_add(hi_base + off[k], h);
            const unsigned nw = (unsigned)oh + (unsigned)h;
            const bool ovf = (int)(((unsigned)oh ^ nw) & ((unsigned)h ^ nw)) < 0;
            rare = (rare << 1) | (unsigned)(big[k] | ovf);
          }
        }
      }
    };
    if (safe) body(std::true_type{});
    else body(std::false_type{});
    if (rare) {  // bit 7 - e flags entry e
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        if ((rare >> (7 - e)) & 1u) {
          const T ts = xv[e] * pk_lds_v(qaddr(qs_base, cw[e]), T(0));
          const int col = (int)((cw[e] & kPkOffMask) >> 2);
          const bool big = F64 ? !(fabs((double)ts) < 4.6e18) : !(fabsf((float)ts) < kPkCap);
          if (big)
            atomicAdd(spill + col, (double)(xv[e] * pk_lds_v(qaddr(qu_base, cw[e]), T(0))));
          else  // the int32 (fp32: the sum; fp64: the high limb) wrapped
            atomicAdd(spill + col, (ts > T(0) ? 1.0 : -1.0) * (F64 ? 18446744073709551616.0 : 4294967296.0) * quantum);
        }
      }
    }
  };

  // prologue: the first NS tiles in flight
  for (int i = 0; i < NS; ++i) issue(i, i);
  // v of row D.z + k of a tile (k < rows): from the slot when it came with the copy
  auto v_of = [&](const uint4& D, int k, bool from_slot, int s) {
    if (!vv) return T(1);
    const int64_t row = (int64_t)D.z + k;
    if (from_slot && (row + 1) * TS <= vlim) {
      const int64_t v0b = (int64_t)D.z * TS & ~(int64_t)15;
      return pk_lds_v(ring_base + (unsigned)s * SLOT + SLOT_V + (unsigned)(row * TS - v0b), T(0));
    }
    return __ldg(vv + row);
  };
  int slot = 0;
  unsigned par = 0;

  // FRONT of tile j: descriptor, window (ring or global), the dot, q = alpha v p into qu;
  // `first`: the tile's largest |term| into the CTA's cap
  auto front = [&](int j, bool first, uint4& D, bool& one, uint32_t (&cw)[8], T (&xv)[8]) {
    if ((j & 15) == 0) desc_req((j >> 4) + 1);
    if ((j & 15) == 8) desc_wait();
    D = desc_of(j);
    const int len = seg_len(D);
    one = NS > 0 && len <= 256;
    if (one) {
      fpd::mbar_wait(&s_bar[warp][slot], par);
      win_smem(slot, ((len + 7) & ~7) >> 3, cw, xv);
    } else if (len <= 256) {
      win_glob(D, 0, cw, xv);
    }
    const int nr = seg_rows(D);
    const T v0 = lane < nr ? v_of(D, lane, one && vring, slot) : T(0);
    const T v1 = lane + 32 < nr ? v_of(D, lane + 32, one && vring, slot) : T(0);
    const bool reg = len <= 256;  // the window is in registers (else streamed)
    T q0, q1;
    if constexpr (YM != 0) {
      pk_sts(rs_base + TS * lane, T(0));
      pk_sts(rs_base + TS * (lane + 32), T(0));
      __syncwarp();
      int carry = -4;
      if (reg) {
        if (len > 0) dot_win(cw, xv, carry);
      } else {
        for (int s0 = 0; s0 < len; s0 += 256) {
          uint32_t c2[8];
          T x2[8];
          win_glob(D, s0, c2, x2);
          dot_win(c2, x2, carry);
        }
      }
      q0 = alpha * (v0 * pk_lds_v(rs_base + TS * lane, T(0)));
      q1 = alpha * (v1 * pk_lds_v(rs_base + TS * (lane + 32), T(0)));
    } else {
      q0 = alpha * v0;
      q1 = alpha * v1;
    }
    pk_sts(qu_base + TS * lane, q0);
    pk_sts(qu_base + TS * (lane + 32), q1);
    if (first) {  // the CTA's cap from every warp's first tile (one barrier per round)
      __syncwarp();
      float tm = 0.f;
      for (int s0 = 0; s0 < len; s0 += 256) {
        uint32_t c2[8];
        T x2[8];
        if (!reg) win_glob(D, s0, c2, x2);
#pragma unroll
        for (int e = 0; e < 8; ++e) {
          const double t = fabs((double)((reg ? xv[e] : x2[e]) * pk_lds_v(qaddr(qu_base, reg ? cw[e] : c2[e]), T(0))));
          if (t <= 1.7976931348623157e308) tm = fmaxf(tm, (float)fmin(t, 3.0e38));
        }
      }
#pragma unroll
      for (int d = 16; d > 0; d >>= 1) tm = fmaxf(tm, __shfl_xor_sync(0xffffffffu, tm, d));
      if (lane == 0 && tm > 0.f) atomicMax(&s_tmax, __float_as_uint(tm));
    }
  };
  // BACK of tile j: q / quantum, the scatter (registers, or the long segment re-streamed), then
  // the freed slot takes tile j + NS
  auto back = [&](int j, const uint4& D, bool one, const uint32_t (&cw)[8], const T (&xv)[8]) {
    __syncwarp();
    const T s = (T)sc;
    pk_sts(qs_base + TS * lane, pk_lds_v(qu_base + TS * lane, T(0)) * s);
    pk_sts(qs_base + TS * (lane + 32), pk_lds_v(qu_base + TS * (lane + 32), T(0)) * s);
    __syncwarp();
    const int len = seg_len(D);
    // fp64 only (C3 0.821 -> 0.785 ms); the fp32 pass at 64 registers spills with both paths
    // (S3 0.487 -> 0.501 ms), so it keeps the checked one
    bool safe = false;
    if constexpr (F64) {
      const double xm = (double)__uint_as_float(D.w);  // the tile's max |x| (+Inf if not finite)
      safe = __all_sync(0xffffffffu, fabs(pk_lds_v(qs_base + TS * lane, T(0))) * xm < 4.0e18 &&
                                         fabs(pk_lds_v(qs_base + TS * (lane + 32), T(0))) * xm < 4.0e18);
    }
    if (len <= 256) {
      if (len > 0) scat_win(cw, xv, 0, len, safe);
    } else {
      for (int s0 = 0; s0 < len; s0 += 256) {
        uint32_t c2[8];
        T x2[8];
        win_glob(D, s0, c2, x2);
        scat_win(c2, x2, s0, len, safe);
      }
    }
    if (NS > 0) {
      __syncwarp();
      issue(j + NS, slot);
      if (++slot == NS) slot = 0, par ^= 1u;
    }
    (void)one;
  };

  int j = 0;
  for (;;) {  // first rounds (CTA-uniform loop): calibrate the fixed-point scale
    const bool have = j < nt;
    uint32_t cw[8];
    T xv[8];
    uint4 D = make_uint4(0, 0, 0, 0);
    bool one = false;
    if (have) front(j, true, D, one, cw, xv);
    const int any = __syncthreads_or(have);
    const float mx = __uint_as_float(*(volatile unsigned*)&s_tmax);
    if (mx > 0.f) {
      int e0;
      frexpf(mx, &e0);
      set_scale(e0 + a.hbits);
    }
    if (have) {
      back(j, D, one, cw, xv);
      ++j;
    }
    if (mx > 0.f || !any) break;
  }
  for (; j < nt; ++j) {  // steady state
    uint32_t cw[8];
    T xv[8];
    uint4 D;
    bool one;
    front(j, false, D, one, cw, xv);
    back(j, D, one, cw, xv);
  }

  __syncthreads();
  double* dst = a.part + (int64_t)blockIdx.x * a.n;
  for (int i = threadIdx.x; i < n; i += BS1) {
    const long long I = F64 ? (long long)(((unsigned long long)(long long)hi[i] << 32) | (unsigned long long)lo[i])
                            : (long long)(int)lo[i];
    dst[i] = (double)I * quantum;
  }
}

template <typename T>
__global__ void k_pk1_finalize(int64_t n, int ctas, const double* __restrict__ part, double* __restrict__ spill,
                               const T* __restrict__ z, double beta, int add_beta_z, int accumulate, T* w) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int gi = 0; gi < ctas; ++gi) s += part[(int64_t)gi * n + j];  // fixed order
    s += spill[j];
    if (add_beta_z && beta != 0.0) s += beta * (double)z[j];
    if (accumulate) s += (double)w[j];
    w[j] = (T)s;
    spill[j] = 0.0;
  }
}

// The pass.  Warp `warp` of CTA k (block k) in group g walks the tile list of warp-quad
// (g, warp) -- the same list in every CTA of the group -- as a pipeline:
//   DOT(i):  stream tile i's segment (256 entries per step, lane l holding entries 8l..8l+7
//            from two 32-byte loads), Eq. (2) products y[col] x, segmented sums by row ->
//            the block partials of the row dots, published as one tagged word per row (CTA 0
//            also publishes v of the rows);
//   Q(j):    j = i - D: wait for the CS (+ v) words of rows `lane` and `lane + 32` of tile j,
//            sum them in block order (identical in every CTA), q = alpha v p;
//   SCAT(j): stream tile j's segment again (read D tiles ago: an L2 hit) and add every
//            term x q into the block's fixed-point partial.
// The dot runs D tiles ahead of the scatter, so the exchange latency hides behind the warp's
// own work.  Padding entries (column = the block's zero / dummy slot, row 63, value 0) fill the
// segments to 8 entries and the lanes beyond a segment load a padding block: no per-entry
// predicates.
template <int CS, int YM, int BS>
__global__ void __launch_bounds__(BS, 1) k_pk(const PkArgs a) {
  constexpr int NW = BS / 32;
  // BS <= 768: 85 registers -- the scatter's first window is loaded before the exchange poll
  constexpr bool PFS = BS <= 768;
  // pipeline depth: measured on C4, D = 1 6.22 ms, D = 2 7.05 ms (the segments of 3 tiles per warp
  // in flight between dot and scatter overflow L2: the re-reads miss), D = 0 13.5 ms (exchange latency)
  constexpr int D = (CS > 1 && YM != 0) ? 1 : 0;
  constexpr int NS = PkSlots<D>::NS;
  static_assert(kPkRing >= D + 1, "descriptor ring");
  extern __shared__ __align__(16) unsigned char pk_smem[];
  __shared__ float rs[NW][kPkRows];   // the tile's block partials of the row dots (by row in tile)
  __shared__ float qsm[NW][kPkRows];  // q / quantum of the tile's rows
  __shared__ float qus[NW][kPkRows];  // q of the tile's rows (spill path, first rounds)
  __shared__ uint4 ring[NW][kPkRing]; // descriptors of the tiles between DOT and SCATTER
  __shared__ unsigned s_tmax;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int k = CS == 1 ? 0 : (int)(blockIdx.x % CS);
  const int g = CS == 1 ? (int)blockIdx.x : (int)(blockIdx.x / CS);
  const int bw = a.bw;
  const int64_t c0 = (int64_t)k * bw;
  const int bwk = (int)max((int64_t)0, min((int64_t)bw, a.n - c0));  // columns of this block
  // [y: bw + 1 floats, y[bw] = 0 (padding entries)][acc: bw + 1 + 32 ints: acc[bw] = the padding
  // entries' dummy, acc[bw + 1 + l] = lane l's dummy when it is beyond the segment (the
  // padding block: 32 lanes on one word would serialise the atomic 32 ways)]
  const int ystride = YM ? (bw + 4) & ~3 : 0;
  float* y_s = reinterpret_cast<float*>(pk_smem);
  int* acc = reinterpret_cast<int*>(pk_smem) + ystride;
  for (int j = threadIdx.x; j <= bw + 32; j += BS) {
    if (YM && j <= bw) y_s[j] = j < bwk ? a.y[c0 + j] : 0.f;
    acc[j] = 0;
  }
  if (threadIdx.x == 0) s_tmax = 0u;
  __syncthreads();
  const unsigned ys_base = fpd::smem_u32(y_s), acc_base = fpd::smem_u32(acc);
  const unsigned rs_base = fpd::smem_u32(&rs[warp][0]), qs_base = fpd::smem_u32(&qsm[warp][0]),
                 qu_base = fpd::smem_u32(&qus[warp][0]);

  unsigned long long tr0 = 0, tr1 = 0;
  if (a.trace) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tr0));
  const int gq = g * NW + warp;
  const int64_t t0 = a.wtile[gq];
  const int nt = a.wtile[gq + 1] - a.wtile[gq];
  const uint4* __restrict__ desc = a.tile_desc + (int64_t)k * a.ntiles + t0;
  const unsigned tag0 = *a.epoch << 20;
  constexpr int SW = (CS + 1) * kPkRows;  // words of one slot
  unsigned long long* const xslot = a.xch + (int64_t)gq * NS * SW;
  const float alpha = a.alpha;
  double* const spill = a.spill + (int64_t)k * (bw + 1);
  const int64_t padidx = a.padidx;

  auto seg_len = [](const uint4& T) { return (int)(T.y & 0x1FFFFFFu); };
  auto seg_rows = [](const uint4& T) { return (int)(T.y >> 25); };
  // the lane's 8 entries of step s0 (the padding block beyond the segment)
  auto ld_step = [&](const uint4& T, int s0, auto keep, uint32_t (&cw)[8], float (&xv)[8]) {
    const int o = s0 + 8 * lane;
    const int64_t idx = o < seg_len(T) ? (int64_t)T.x * 8 + o : padidx;
    pk_ld8<decltype(keep)::value>(a.cr + idx, a.val + idx, cw, xv);
  };

  // ---- DOT(i): tile i's block partials of the row dots, published (YM), descriptor -> ring
  uint4 cd = make_uint4(0, 0, 0, 0);  // lane l: descriptor of tile (i & ~31) + l
  float pown0 = 0.f, pown1 = 0.f, vown0 = 0.f, vown1 = 0.f;  // D == 0: partials / v of rows lane, lane + 32
  auto dot = [&](int i) {
    if ((i & 31) == 0 && i + lane < nt) cd = __ldg(desc + i + lane);
    uint4 T;
    T.x = __shfl_sync(0xffffffffu, cd.x, i & 31);
    T.y = __shfl_sync(0xffffffffu, cd.y, i & 31);
    T.z = __shfl_sync(0xffffffffu, cd.z, i & 31);
    T.w = __shfl_sync(0xffffffffu, cd.w, i & 31);
    if (lane == 0) ring[warp][i % kPkRing] = T;
    // the next tile's segment on its way into L2 (lanes 0-15: 128-byte lines of cr, 16-31: val)
    {
      const int i1 = i + 1;
      const unsigned off1 = __shfl_sync(0xffffffffu, cd.x, i1 & 31), len1 = __shfl_sync(0xffffffffu, cd.y, i1 & 31);
      if ((i1 & 31) != 0 && i1 < nt) {
        if (a.pf == 1) {
          const int l = lane & 15;
          if (32 * l < (int)min(len1 & 0x1FFFFFFu, 512u)) {
            const int64_t e = (int64_t)off1 * 8 + 32 * l;
            pk_prefetch_l2(lane < 16 ? (const void*)(a.cr + e) : (const void*)(a.val + e));
          }
        } else if (a.pf == 2 && lane == 0) {  // bulk prefetch (TMA unit, not the LSU pipe)
          const int64_t e = (int64_t)off1 * 8;
          const unsigned nb = min(len1 & 0x1FFFFFFu, 2048u) * 4u;
          fpd::prefetch_l2(a.cr + e, nb);
          fpd::prefetch_l2(a.val + e, nb);
        }
      }
    }
    __syncwarp();
    if constexpr (YM == 0) return;
    const int nr = seg_rows(T), len = seg_len(T);
    float v0 = 0.f, v1 = 0.f;
    if (CS == 1 || k == 0) {
      const float* vp = a.v + (int)T.z;
      if (lane < nr) v0 = a.v ? __ldg(vp + lane) : 1.f;
      if (lane + 32 < nr) v1 = a.v ? __ldg(vp + lane + 32) : 1.f;
    }
    pk_sts(rs_base + 4 * lane, 0.f);
    pk_sts(rs_base + 128 + 4 * lane, 0.f);
    __syncwarp();
    int carry = -4;  // rid * 4 of the previous step's last entry
    for (int s0 = 0; s0 < len; s0 += 256) {
      uint32_t cw[8];
      float xv[8];
      ld_step(T, s0, std::true_type{}, cw, xv);
      int r4[8];
      float c[8];  // in-lane inclusive segmented sums of the Eq. (2) products
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        r4[e] = (int)(cw[e] >> 24);
        const float pr = xv[e] * pk_lds(ys_base + (cw[e] & kPkOffMask));
        c[e] = (e == 0 || r4[e] != r4[e - 1]) ? pr : c[e - 1] + pr;
      }
      int prev = __shfl_up_sync(0xffffffffu, r4[7], 1);
      if (lane == 0) prev = carry;
      const bool h0 = r4[0] != prev;
      bool seen = h0;
      // rows that start and end inside the lane
#pragma unroll
      for (int e = 0; e < 7; ++e) {
        const bool h = r4[e + 1] != r4[e];
        if (h && seen) pk_sts(rs_base + r4[e], c[e]);
        seen |= h;
      }
      // P = the entries before the lane's first row start (continuing a row from before)
      float P = c[7];
#pragma unroll
      for (int e = 7; e >= 1; --e)
        if (r4[e] != r4[e - 1]) P = c[e - 1];
      if (h0) P = 0.f;
      // across lanes: R_l = P_l + ... + P_h, h = the first lane >= l holding a row start
      const unsigned H = __ballot_sync(0xffffffffu, seen);
      const unsigned hl = H >> lane;
      const int dist = hl ? __ffs(hl) : 32 - lane;
      float r = P;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const float t2 = __shfl_down_sync(0xffffffffu, r, d);
        if (d < dist) r += t2;
      }
      float rn = __shfl_down_sync(0xffffffffu, r, 1);
      if (lane == 31) rn = 0.f;
      if (seen) pk_sts(rs_base + r4[7], c[7] + rn);                                  // the lane's last row
      if (lane == 0 && !h0 && prev >= 0) pk_sts(rs_base + prev, pk_lds_v(rs_base + prev) + r);  // running in
      carry = __shfl_sync(0xffffffffu, r4[7], 31);
      __syncwarp();
    }
    const float p0 = pk_lds_v(rs_base + 4 * lane), p1 = pk_lds_v(rs_base + 128 + 4 * lane);
    if constexpr (CS > 1) {
      // lane l's two rows (l, l + 32) side by side: one 16-byte store / load per block, each
      // 8-byte half its own (value, tag) word
      const unsigned long long tg = (unsigned long long)(tag0 + (unsigned)i) << 32;
      unsigned long long* slot = xslot + (int64_t)(i % NS) * SW + 2 * lane;
      st_relaxed_gpu2(slot + k * kPkRows, tg | __float_as_uint(p0), tg | __float_as_uint(p1));
      if (k == 0) st_relaxed_gpu2(slot + CS * kPkRows, tg | __float_as_uint(v0), tg | __float_as_uint(v1));
    } else {
      pown0 = p0;
      pown1 = p1;
      vown0 = v0;
      vown1 = v1;
    }
  };

  // ---- Q(j): q of rows lane and lane + 32 of tile j (descriptor T) -> qus
  auto qcalc = [&](const uint4& T, int j) {
    const int nr = seg_rows(T);
    float q0, q1;
    if constexpr (YM == 0) {
      (void)j;
      const float* vp = a.v + (int)T.z;
      q0 = lane < nr ? alpha * (a.v ? __ldg(vp + lane) : 1.f) : 0.f;
      q1 = lane + 32 < nr ? alpha * (a.v ? __ldg(vp + lane + 32) : 1.f) : 0.f;
    } else if constexpr (CS == 1) {
      (void)j;
      q0 = alpha * (vown0 * pown0);
      q1 = alpha * (vown1 * pown1);
    } else {
      // the exchange: value + tag in one 64-bit word, so no flag and no fence is needed
      const unsigned tag = tag0 + (unsigned)j;
      const unsigned long long* slot = xslot + (int64_t)(j % NS) * SW + 2 * lane;
      unsigned wv[2 * (CS + 1)];  // the values (tags checked)
      for (;;) {
        bool done = true;
#pragma unroll
        for (int b = 0; b <= CS; ++b) {
          unsigned long long w0, w1;
          ld_relaxed_gpu2(slot + b * kPkRows, w0, w1);
          wv[2 * b] = (unsigned)w0;
          wv[2 * b + 1] = (unsigned)w1;
          done &= (unsigned)(w0 >> 32) == tag && (unsigned)(w1 >> 32) == tag;
        }
        if (done) break;
        if (a.nap > 0) {
          __nanosleep(a.nap);
        } else if (a.nap < 0) {  // a busy pause: no memory traffic, the warp stays scheduled
          const long long c0 = clock64();
          while (clock64() - c0 < -a.nap) {
          }
        }
      }
      float p0 = 0.f, p1 = 0.f;
#pragma unroll
      for (int b = 0; b < CS; ++b) {  // block order: identical in every CTA
        p0 += __uint_as_float(wv[2 * b]);
        p1 += __uint_as_float(wv[2 * b + 1]);
      }
      q0 = alpha * (__uint_as_float(wv[2 * CS]) * p0);
      q1 = alpha * (__uint_as_float(wv[2 * CS + 1]) * p1);
    }
    if (lane >= nr) q0 = 0.f;
    if (lane + 32 >= nr) q1 = 0.f;
    pk_sts(qu_base + 4 * lane, q0);
    pk_sts(qu_base + 128 + 4 * lane, q1);
  };

  float sc = 1.f;      // 2^(26 - E): the cap is 2^E
  double quantum = 0;  // 2^(E - 26)
  auto set_scale = [&](int e) {
    e = min(max(e, -95), 100);
    sc = ldexpf(1.f, 26 - e);
    quantum = ldexp(1.0, e - 26);
  };
  set_scale(0);

  // ---- SCAT(j): Eq. (3) from the segment, re-read.  SAFE (every |x q| of the tile below the
  // cap, from the plan's max |x| of the tile): no per-entry checks; else terms beyond the cap
  // and non-finite terms are flagged too.  Flagged entries (and int32 wraps) spill after.
  // pf: the segment's first window, loaded by the caller before the exchange poll (its load
  // latency hides behind the wait; ncu r02c: 13 % of k_pk's stall samples sat on that load)
  auto scatter = [&](const uint4& T, const uint32_t (&pcw)[8], const float (&pxv)[8], bool pf) {
    __syncwarp();
    const float q0 = pk_lds_v(qu_base + 4 * lane), q1 = pk_lds_v(qu_base + 128 + 4 * lane);
    const float qs0 = q0 * sc, qs1 = q1 * sc;
    pk_sts(qs_base + 4 * lane, qs0);
    pk_sts(qs_base + 128 + 4 * lane, qs1);
    const float xm = __uint_as_float(T.w);
    const bool safe = __all_sync(0xffffffffu, fabsf(qs0) * xm < 2.0e9f && fabsf(qs1) * xm < 2.0e9f);
    __syncwarp();
    const int len = seg_len(T);
    auto run = [&](auto SAFE) {
      for (int s0 = 0; s0 < len; s0 += 256) {
        uint32_t cw[8];
        float xv[8];
        if (pf && s0 == 0) {
#pragma unroll
          for (int e = 0; e < 8; ++e) cw[e] = pcw[e], xv[e] = pxv[e];
        } else {
          ld_step(T, s0, std::false_type{}, cw, xv);
        }
        const unsigned abase = acc_base + (s0 + 8 * lane < len ? 0u : 4u * (lane + 1));  // lane's dummy
        unsigned rare = 0;
#pragma unroll
        for (int e = 0; e < 8; ++e) {
          const float ts = xv[e] * pk_lds(qs_base + (cw[e] >> 24));
          int qi = __float2int_rn(ts);
          if constexpr (!decltype(SAFE)::value) {
            const bool big = !(fabsf(ts) < kPkCap);  // beyond the int32 range, or NaN
            if (big) qi = 0;
            rare = (rare << 1) | (unsigned)big;
          }
          const int old = pk_atom_add(abase + (cw[e] & kPkOffMask), qi);  // native ATOMS.ADD
          const unsigned nw = (unsigned)old + (unsigned)qi;
          const unsigned ovf = ((unsigned)old ^ nw) & ((unsigned)qi ^ nw);  // sign bit: int32 wrap
          if constexpr (decltype(SAFE)::value) rare = pk_push_sign(rare, ovf);
          else rare |= ovf >> 31;
        }
        if (rare) {  // rare: bit 7 - e flags entry e
#pragma unroll
          for (int e = 0; e < 8; ++e) {
            if ((rare >> (7 - e)) & 1u) {
              const float ts = xv[e] * pk_lds_v(qs_base + (cw[e] >> 24));
              const int col = (int)((cw[e] & kPkOffMask) >> 2);
              if (!(fabsf(ts) < kPkCap))  // beyond the cap / Inf / NaN (IEEE propagation, reading R8)
                atomicAdd(spill + col, (double)(xv[e] * pk_lds_v(qu_base + (cw[e] >> 24))));
              else  // the int32 sum wrapped: carry 2^32 quanta
                atomicAdd(spill + col, ts > 0.f ? 4294967296.0 * quantum : -4294967296.0 * quantum);
            }
          }
        }
      }
    };
    if (safe) run(std::true_type{});
    else run(std::false_type{});
  };

  // largest finite |x q| of a tile (the first rounds only)
  auto tmax_of = [&](const uint4& T) -> float {
    __syncwarp();
    float tm = 0.f;
    for (int s0 = 0; s0 < seg_len(T); s0 += 256) {
      uint32_t cw[8];
      float xv[8];
      ld_step(T, s0, std::true_type{}, cw, xv);
#pragma unroll
      for (int e = 0; e < 8; ++e) {
        const float t = fabsf(xv[e] * pk_lds_v(qu_base + (cw[e] >> 24)));
        if (t <= 3.402823466e38f) tm = fmaxf(tm, t);
      }
    }
    return tm;
  };

  // ---- the dots of the first D tiles, then rounds of one scatter per warp until the CTA's
  // cap is set (all warps take part in every round: the loop condition is CTA-uniform)
  for (int i = 0; i < D; ++i)
    if (i < nt) dot(i);
  int j = 0;
  for (;;) {
    const bool have = j < nt;
    uint4 T = make_uint4(0, 0, 0, 0);
    float tm = 0.f;
    if (have) {
      if (j + D < nt) dot(j + D);
      T = ring[warp][j % kPkRing];
      qcalc(T, j);
      tm = tmax_of(T);
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) tm = fmaxf(tm, __shfl_xor_sync(0xffffffffu, tm, d));
    if (lane == 0 && tm > 0.f) atomicMax(&s_tmax, __float_as_uint(tm));
    const int any = __syncthreads_or(have);
    const float mx = __uint_as_float(*(volatile unsigned*)&s_tmax);
    if (mx > 0.f) {
      int e0;
      frexpf(mx, &e0);  // mx < 2^e0
      set_scale(e0 + a.hbits);
    }
    // (while every finite term so far is 0, the provisional scale adds zeros; non-finite terms spill)
    if (have) {
      uint32_t pcw[8];
      float pxv[8];
      scatter(T, pcw, pxv, false);
      ++j;
    }
    if (mx > 0.f || !any) break;
  }

  if (a.trace) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tr1));
  // ---- steady state
  for (; j < nt; ++j) {
    if (j + D < nt) dot(j + D);
    const uint4 T = ring[warp][j % kPkRing];
    uint32_t pcw[8];
    float pxv[8];
    if constexpr (PFS) ld_step(T, 0, std::false_type{}, pcw, pxv);  // in flight during the poll
    qcalc(T, j);
    scatter(T, pcw, pxv, PFS);
  }
  if (a.trace && lane == 0) {
    unsigned long long tr2;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tr2));
    unsigned long long* tp = a.trace + ((int64_t)blockIdx.x * NW + warp) * 8;
    tp[0] = tr0;
    tp[1] = tr2;
    tp[2] = (unsigned long long)nt;
    tp[3] = tr1;
    tp[4] = tp[5] = tp[6] = tp[7] = 0;
  }

  __syncthreads();
  double* dst = a.part + (int64_t)g * a.n + c0;
  for (int i = threadIdx.x; i < bwk; i += BS) dst[i] = (double)acc[i] * quantum;
}

__global__ void k_pk_finalize(int64_t n, int bw, int groups, const double* __restrict__ part,
                              double* __restrict__ spill, const float* __restrict__ z, double beta, int add_beta_z,
                              int accumulate, float* w, unsigned* epoch) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int gi = 0; gi < groups; ++gi) s += part[(int64_t)gi * n + j];  // fixed order
    const int64_t b = j / bw;
    double* sp = spill + j + b;  // [block][bw + 1]
    s += *sp;
    if (add_beta_z && beta != 0.0) s += beta * (double)z[j];
    if (accumulate) s += (double)w[j];
    w[j] = (float)s;
    *sp = 0.0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) *epoch += 1u;
}

// ------------------------------------------------------------------------------ plan side
// (1) entries of each row in each column block
__global__ void k_pk_count(int64_t m, const int64_t* __restrict__ rowptr, const int32_t* __restrict__ colidx,
                           int cs, int bw, uint32_t* __restrict__ cnt) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < m; r += (int64_t)gridDim.x * blockDim.x) {
    uint32_t c[kPkMaxCS] = {};
    const int64_t e = rowptr[r + 1];
    for (int64_t i = rowptr[r]; i < e; ++i) {
      const int b = colidx[i] / bw;
#pragma unroll
      for (int kk = 0; kk < kPkMaxCS; ++kk) c[kk] += (uint32_t)(b == kk);
    }
    for (int kk = 0; kk < cs; ++kk) cnt[(int64_t)kk * m + r] = c[kk];
  }
}

// (2) tiles of each 64-row group (greedy): bit i of gmask set where a tile starts at row 64 g + i
__device__ __forceinline__ bool pk_is_long(const uint32_t* cnt, int64_t m, int cs, int64_t r, int span) {
  for (int kk = 0; kk < cs; ++kk)
    if (cnt[(int64_t)kk * m + r] > (uint32_t)span) return true;
  return false;
}
__global__ void k_pk_tiles(int64_t m, int gr, int cs, int span, const uint32_t* __restrict__ cnt,
                           unsigned long long* __restrict__ gmask, int64_t* __restrict__ gcount) {
  const int64_t ng = (m + gr - 1) / gr;
  for (int64_t gi = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; gi < ng; gi += (int64_t)gridDim.x * blockDim.x) {
    uint32_t accs[kPkMaxCS] = {};
    unsigned long long mask = 0;
    int ntl = 0;
    bool fresh = true;  // the next row starts a tile
    for (int i = 0; i < gr && gi * gr + i < m; ++i) {
      const int64_t r = gi * gr + i;
      if (pk_is_long(cnt, m, cs, r, span)) {
        mask |= 1ull << i;
        ++ntl;
        fresh = true;
        continue;
      }
      bool fit = !fresh;
      for (int kk = 0; kk < cs && fit; ++kk) fit = accs[kk] + cnt[(int64_t)kk * m + r] <= (uint32_t)span;
      if (!fit) {
        mask |= 1ull << i;
        ++ntl;
        for (int kk = 0; kk < cs; ++kk) accs[kk] = 0;
      }
      for (int kk = 0; kk < cs; ++kk) accs[kk] += cnt[(int64_t)kk * m + r];
      fresh = false;
    }
    gmask[gi] = mask;
    gcount[gi] = ntl;
  }
}

// (3) tile rows and segment lengths; al = the lengths rounded up to 8 (scanned into offsets)
__global__ void k_pk_tile_rows(int64_t m, int gr, int cs, int64_t ntiles, const uint32_t* __restrict__ cnt,
                               const unsigned long long* __restrict__ gmask, const int64_t* __restrict__ gbase,
                               int64_t* __restrict__ tile_row, uint32_t* __restrict__ tlen, int64_t* __restrict__ al) {
  const int64_t ng = (m + gr - 1) / gr;
  for (int64_t gi = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; gi < ng; gi += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long mask = gmask[gi];
    int64_t t = gbase[gi] - 1;
    uint32_t len[kPkMaxCS] = {};
    auto flush = [&]() {
      if (t < 0) return;
      for (int kk = 0; kk < cs; ++kk) {
        tlen[(int64_t)kk * ntiles + t] = len[kk];
        al[(int64_t)kk * ntiles + t] = (int64_t)((len[kk] + 7u) & ~7u);
        len[kk] = 0;
      }
    };
    for (int i = 0; i < gr && gi * gr + i < m; ++i) {
      const int64_t r = gi * gr + i;
      if ((mask >> i) & 1ull) {
        flush();
        ++t;
        tile_row[t] = r;
      }
      for (int kk = 0; kk < cs; ++kk) len[kk] += cnt[(int64_t)kk * m + r];
    }
    flush();
    if (gi == ng - 1) tile_row[ntiles] = m;
  }
}

__global__ void k_pk_desc(int64_t total, int64_t ntiles, const int64_t* __restrict__ off,
                          const uint32_t* __restrict__ tlen, const int64_t* __restrict__ tile_row,
                          uint4* __restrict__ desc) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t = i % ntiles;
    const unsigned nr = (unsigned)(tile_row[t + 1] - tile_row[t]);
    desc[i] = make_uint4((unsigned)(off[i] >> 3), tlen[i] | (nr << 25), (unsigned)tile_row[t], 0u);
  }
}

__global__ void k_pk_fill(int64_t n, uint32_t* __restrict__ p, uint32_t v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}

// (4) the entries: a warp per 64-row group, lanes over a row's entries; block-k entries keep
// their order (stable), so non-canonical rows are packed as given (reading R7).  Entry word:
// byte offset of the column inside its block | row inside the tile << 26.  Also the largest
// |x| of every (tile, block) segment (+Inf if a value is not finite): the scatter's no-check test.
template <typename V>
__global__ void k_pk_scatter(int64_t m, int gr, int cs, int bw, int64_t ntiles, const int64_t* __restrict__ rowptr,
                             const int32_t* __restrict__ colidx, const V* __restrict__ val,
                             const unsigned long long* __restrict__ gmask, const int64_t* __restrict__ gbase,
                             uint4* __restrict__ desc, uint32_t* __restrict__ cr, V* __restrict__ pval) {
  const int lane = threadIdx.x & 31;
  const unsigned lt = pk_lanemask_lt();
  const int64_t ng = (m + gr - 1) / gr;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x / 32);
  for (int64_t gi = blockIdx.x * (int64_t)(blockDim.x / 32) + (threadIdx.x >> 5); gi < ng; gi += nw) {
    const unsigned long long mask = gmask[gi];
    int64_t t = gbase[gi] - 1;
    int64_t run[kPkMaxCS] = {};
    float xm[kPkMaxCS] = {};
    unsigned rid = 0;
    auto flush = [&]() {
      if (t < 0) return;
      for (int kk = 0; kk < cs; ++kk) {
        float v = xm[kk];
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, d));
        if (lane == 0) desc[(int64_t)kk * ntiles + t].w = __float_as_uint(v);
        xm[kk] = 0.f;
      }
    };
    for (int i = 0; i < gr && gi * gr + i < m; ++i) {
      const int64_t r = gi * gr + i;
      if ((mask >> i) & 1ull) {
        flush();
        ++t;
        rid = 0;
        for (int kk = 0; kk < cs; ++kk) run[kk] = (int64_t)desc[(int64_t)kk * ntiles + t].x * 8;
      }
      const int64_t e = rowptr[r + 1];
      for (int64_t i0 = rowptr[r]; i0 < e; i0 += 32) {
        const int64_t ii = i0 + lane;
        const bool ok = ii < e;
        const int col = ok ? colidx[ii] : 0;
        const int b = col / bw;
        int64_t pos = -1;
        const V x = ok && val ? val[ii] : V(0);
        const float ax = fabs((double)x) <= 3.0e38 ? (float)fabs((double)x) : __int_as_float(0x7f800000);
        for (int kk = 0; kk < cs; ++kk) {
          const unsigned bm = __ballot_sync(0xffffffffu, ok && b == kk);
          if (ok && b == kk) {
            pos = run[kk] + __popc(bm & lt);
            xm[kk] = fmaxf(xm[kk], ax);
          }
          run[kk] += __popc(bm);
        }
        if (ok) {
          cr[pos] = ((uint32_t)(col - b * bw) * 4u) | (rid << kPkRidShift);
          pval[pos] = x;
        }
      }
      ++rid;
    }
    flush();
  }
}

// (4b) shared-memory bank balancing.  In the pass, step e of a window has the 32 lanes gather
// y[col] and add into w[col] for their e-th entries: the instruction costs as many shared-memory
// wavefronts as the most loaded bank (col mod 32).  Inside a lane the entries of one row can be
// permuted freely (the dot's segmented sum only needs each row contiguous across lanes), so for
// every window, slot by slot, the lanes with the fewest choices first, each lane puts into slot
// e the entry of its current row whose bank is least used by the lanes placed so far.  On
// C4-shaped rows this lowers the mean max bank load from 3.5 to 2.4 (tools/banksim.py).
// A warp per (tile, block) segment; the window staged in shared memory.
template <typename V>
__global__ void __launch_bounds__(256) k_pk_bankopt(int64_t nseg, const uint4* __restrict__ desc,
                                                    uint32_t* __restrict__ cr, V* __restrict__ pval, int bmask,
                                                    int ls) {
  __shared__ uint32_t sc[8][32][9];
  __shared__ V sv[8][32][9];
  __shared__ int cnt[8][32];
  __shared__ unsigned char ld[8][8][32];  // local search: load of bank b in slot e
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  const int64_t nw = (int64_t)gridDim.x * 8;
  for (int64_t sg = blockIdx.x * (int64_t)8 + wi; sg < nseg; sg += nw) {
    const uint4 T = desc[sg];
    const int len = (int)(T.y & 0x1FFFFFFu);
    const int64_t base = (int64_t)T.x * 8;
    for (int s0 = 0; s0 < len; s0 += 256) {
      const int o = s0 + 8 * lane;
      const bool act = o < len;  // the lane's 8 entries are inside the (8-padded) segment
      if (act)
        for (int e = 0; e < 8; ++e) sc[wi][lane][e] = cr[base + o + e], sv[wi][lane][e] = pval[base + o + e];
      __syncwarp();
      for (int e = 0; e < 8; ++e) {
        cnt[wi][lane] = 0;
        // choices of this lane for slot e: the remaining entries of the row at slot e
        int k = 0;
        if (act) {
          const uint32_t r = sc[wi][lane][e] >> 24;
          k = 1;
          while (e + k < 8 && (sc[wi][lane][e + k] >> 24) == r) ++k;
        }
        __syncwarp();
        for (int want = 1; want <= 8; ++want) {
          unsigned mset = __ballot_sync(0xffffffffu, k == want);
          while (mset) {
            const int l = __ffs(mset) - 1;
            mset &= mset - 1;
            if (lane == l) {
              int best = e, bc = 1 << 30;
              for (int jj = e; jj < e + k; ++jj) {
                const int c = cnt[wi][(sc[wi][lane][jj] >> 2) & bmask];
                if (c < bc) bc = c, best = jj;
              }
              const uint32_t tw = sc[wi][lane][e];
              const V tv = sv[wi][lane][e];
              sc[wi][lane][e] = sc[wi][lane][best];
              sv[wi][lane][e] = sv[wi][lane][best];
              sc[wi][lane][best] = tw;
              sv[wi][lane][best] = tv;
              ++cnt[wi][(sc[wi][lane][e] >> 2) & bmask];
            }
            __syncwarp();
          }
        }
      }
      // local search (lane 0; FP_PK_NOLS=1 skips it): while a slot's most loaded bank can give
      // an entry to a less loaded bank by swapping two slots of one lane (same row), without
      // raising the other slot's maximum, swap.  Simulated on C4-shaped windows (tools/banksim.py):
      // mean max load 2.39 (greedy) -> 2.03, lower bound 1.80.  Measured: C4 5.65 -> 5.56 ms
      // (pack 0.33 -> 1.3 s), C3 / S3 within 1 %.
      if (ls) {
        for (int e = 0; e < 8; ++e) ld[wi][e][lane] = 0;
        __syncwarp();
        if (lane == 0) {
          for (int l = 0; l < 32; ++l)
            if (s0 + 8 * l < len)
              for (int e = 0; e < 8; ++e) ++ld[wi][e][(sc[wi][l][e] >> 2) & bmask];
          auto slot_max = [&](int e) {
            int mm = 0;
            for (int b = 0; b <= bmask; ++b) mm = max(mm, (int)ld[wi][e][b]);
            return mm;
          };
          for (int it = 0; it < 32; ++it) {
            bool improved = false;
            for (int e = 0; e < 8; ++e) {
              const int mx = slot_max(e);
              if (mx <= 1) continue;
              for (int l = 0; l < 32; ++l) {
                if (s0 + 8 * l >= len) continue;
                const int b = (sc[wi][l][e] >> 2) & bmask;
                if (ld[wi][e][b] != mx) continue;
                for (int f = 0; f < 8; ++f) {
                  if (f == e || (sc[wi][l][f] >> 24) != (sc[wi][l][e] >> 24)) continue;
                  const int b2 = (sc[wi][l][f] >> 2) & bmask;
                  if (b2 == b || ld[wi][e][b2] + 1 >= mx || ld[wi][f][b] + 1 >= mx ||
                      ld[wi][f][b] + 1 > slot_max(f))
                    continue;
                  --ld[wi][e][b], ++ld[wi][e][b2], --ld[wi][f][b2], ++ld[wi][f][b];
                  const uint32_t tw = sc[wi][l][e];
                  const V tv = sv[wi][l][e];
                  sc[wi][l][e] = sc[wi][l][f], sv[wi][l][e] = sv[wi][l][f];
                  sc[wi][l][f] = tw, sv[wi][l][f] = tv;
                  improved = true;
                  break;
                }
                if (ld[wi][e][b] < mx) break;  // this slot's maximum bank gave one up: next slot
              }
            }
            if (!improved) break;
          }
        }
        __syncwarp();
      }
      if (act)
        for (int e = 0; e < 8; ++e) cr[base + o + e] = sc[wi][lane][e], pval[base + o + e] = sv[wi][lane][e];
      __syncwarp();
    }
  }
}

// (4c) one column block (k_pk1): every 256-entry window of a segment stored lane-interleaved --
// the 16-byte piece k of lane l's 8 entries at (k G + l) 16 bytes, G = the window's groups of 8
// -- so the pass's 16-byte loads of a window (shared memory after the bulk copy, or global) are
// conflict-free / coalesced while lane l still holds the logical entries 8l..8l+7.  A warp per
// segment, in place (every lane's loads precede the stores).
template <typename V>
__global__ void k_pk_interleave(int64_t nseg, const uint4* __restrict__ desc, uint32_t* __restrict__ cr,
                                V* __restrict__ pval) {
  constexpr int PV = 16 / (int)sizeof(V);  // values per 16-byte piece
  const int lane = threadIdx.x & 31;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x / 32);
  for (int64_t sg = blockIdx.x * (int64_t)(blockDim.x / 32) + (threadIdx.x >> 5); sg < nseg; sg += nw) {
    const uint4 D = desc[sg];
    const int len8 = (int)(((D.y & 0x1FFFFFFu) + 7u) & ~7u);
    const int64_t base = (int64_t)D.x * 8;
    for (int s0 = 0; s0 < len8; s0 += 256) {
      const int G = min(32, (len8 - s0) >> 3);
      uint32_t c[8];
      V x[8];
      const int64_t b = base + s0;
      if (lane < G)
        for (int e = 0; e < 8; ++e) c[e] = cr[b + 8 * lane + e], x[e] = pval[b + 8 * lane + e];
      __syncwarp();
      if (lane < G)
        for (int e = 0; e < 8; ++e) {
          cr[b + 4 * ((e >> 2) * G + lane) + (e & 3)] = c[e];
          pval[b + PV * ((e / PV) * G + lane) + e % PV] = x[e];
        }
      __syncwarp();
    }
  }
}

// (5) warp-quad partition: tile ranges of equal nonzero + row cost
__global__ void k_pk_partition(int64_t ntiles, int nq, const int64_t* __restrict__ tile_row,
                               const int64_t* __restrict__ rowptr, int32_t* __restrict__ wtile, int rc, int tc) {
  const int qi = blockIdx.x * blockDim.x + threadIdx.x;
  if (qi > nq) return;
  // work before tile t: its nonzeros + rc per row + tc per tile
  auto cost = [&](int64_t t) { const int64_t r = tile_row[t]; return rowptr[r] - rowptr[0] + rc * r + tc * t; };
  const int64_t total = cost(ntiles);
  const int64_t target = (int64_t)((__int128)total * qi / nq);
  int64_t lo = 0, hi = ntiles;  // smallest t with cost(t) >= target
  while (lo < hi) {
    const int64_t mid = (lo + hi) / 2;
    if (cost(mid) >= target) hi = mid;
    else lo = mid + 1;
  }
  wtile[qi] = (int32_t)(qi == nq ? ntiles : lo);
}

template <int CS, int YM>
const void* pk_kernel(int bs) {
  return bs == 768 ? (const void*)k_pk<CS, YM, 768> : (const void*)k_pk<CS, YM, 1024>;
}
const void* pk_pick(int cs, bool has_y, int bs) {
  switch (cs) {
    case 2: return has_y ? pk_kernel<2, 1>(bs) : pk_kernel<2, 0>(bs);
    case 4: return has_y ? pk_kernel<4, 1>(bs) : pk_kernel<4, 0>(bs);
    case 8: return has_y ? pk_kernel<8, 1>(bs) : pk_kernel<8, 0>(bs);
  }
  return nullptr;
}

int pk_headroom() {
  static const int h = [] {
    const char* e = std::getenv("FP_PK_HEADROOM");
    return e ? std::atoi(e) : 3;
  }();
  return h;
}

}  // namespace

// the single-block pass (cs == 1, fp32 / fp64)
template <int BS1>
const void* pk1_pick_bs(fp_dtype dt, bool has_y) {
  if (dt == FP_F64) return has_y ? (const void*)k_pk1<double, 1, BS1> : (const void*)k_pk1<double, 0, BS1>;
  return has_y ? (const void*)k_pk1<float, 1, BS1> : (const void*)k_pk1<float, 0, BS1>;
}
const void* pk1_pick(fp_dtype dt, bool has_y, int bs) {
  return bs == 1024 ? pk1_pick_bs<1024>(dt, has_y)
                    : (bs == 768 ? pk1_pick_bs<768>(dt, has_y)
                                 : (bs == 640 ? pk1_pick_bs<640>(dt, has_y) : pk1_pick_bs<512>(dt, has_y)));
}
size_t pk1_slot_bytes(fp_dtype dt) { return (size_t)256 * (4 + dtype_size(dt)) + (size_t)kPkRows * dtype_size(dt) + 16; }
size_t pk1_smem_n(int64_t n, fp_dtype dt, bool has_y, int bs, int ns) {
  const size_t ts = dtype_size(dt);
  const size_t ys = has_y ? (size_t)((n + 4) & ~3) * ts : 0;
  return (size_t)(bs / 32) * ns * pk1_slot_bytes(dt) + (size_t)(bs / 32) * 32 * 16 + (size_t)3 * (bs / 32) * kPkRows * ts + ys +
         (size_t)((n + 36) & ~3) * 4 * (dt == FP_F64 ? 2 : 1);
}
// tile slots per warp of k_pk1's shared-memory ring: fp64 as many as fit (at most kPk1MaxNS)
// next to y, the partial w and the row arrays; fp32 none (its 32 warps hide the load latency
// themselves, and the ring's shared-memory traffic costs more).  Measured (r02c): C3 (fp64,
// 512 threads) 0.968 ms without the ring, 0.899 / 0.897 / 0.901 ms with 2 / 3 / 4 slots; S3
// (fp32, 1024 threads) 0.513 ms without, 0.596 with 2-4.  FP_PK1_NS (measurement) overrides.
int pk1_ring_ns(int64_t n, fp_dtype dt, int bs) {
  const size_t room = device_info(current_device()).smem_optin_per_block - 2048;  // - static
  const size_t base = pk1_smem_n(n, dt, true, bs, 0);
  const int fit = room > base ? (int)std::min<size_t>((room - base) / ((size_t)(bs / 32) * pk1_slot_bytes(dt)), kPk1MaxNS) : 0;
  int ns = dt == FP_F64 ? fit : 0;
  if (const char* e = std::getenv("FP_PK1_NS")) ns = std::max(0, std::min(fit, std::atoi(e)));
  return ns;
}
// columns one CTA holds (y + the fixed-point partial in the opt-in shared memory)
int packed_max_bw() {
  const size_t room = device_info(current_device()).smem_optin_per_block - kPkStatic;
  return (int)std::min<size_t>(room / 8 - 40, (kPkOffMask >> 2) - 1);  // + the zero / dummy slots
}
// the single-block pass k_pk1 (static shared memory: 3 x 32 x 64 values)
int packed1_max_n(fp_dtype dt) {
  // default CTAs (fp32 1024, fp64 512 threads): row arrays + descriptor batches + static
  const size_t nw = dt == FP_F64 ? 16 : 32;
  const size_t stat = (size_t)3 * nw * kPkRows * dtype_size(dt) + nw * 512 + 2048;
  const size_t room = device_info(current_device()).smem_optin_per_block - stat;
  return (int)std::min<size_t>(room / (dt == FP_F64 ? 16 : 8) - 48, (kPkOffMask >> 2) - 1);
}

int packed_cs(int64_t n, fp_dtype dt) {
  if (n <= packed1_max_n(dt)) return 1;
  if (dt == FP_F64) return 0;
  const int64_t mb = packed_max_bw();
  for (int cs : {2, 4, 8})
    if ((n + cs - 1) / cs <= mb) return cs;
  return 0;
}

void packed_free(Packed* p) {
  if (!p) return;
  for (void* b : {(void*)p->tile_desc, (void*)p->wtile, (void*)p->cr, (void*)p->val, (void*)p->xch,
                  (void*)p->epoch, (void*)p->part, (void*)p->spill, (void*)p->trace, (void*)p->rowdot,
                  (void*)p->hcol, (void*)p->hrow, p->hval, (void*)p->hitems, (void*)p->dotlist})
    if (b) cudaFree(b);
  delete p;
}

fp_status packed_build(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                       const void* val, fp_dtype dtype, int cs_force, Packed** out, cudaStream_t s) {
  *out = nullptr;
  FP_REQUIRE(valid_dtype(dtype), FP_ERR_INVALID_ARG, "fp_csr_plan_pack: bad dtype");
  FP_REQUIRE(val || nnz == 0, FP_ERR_INVALID_ARG, "fp_csr_plan_pack: val is NULL");
  FP_REQUIRE(m >= 1 && n >= 1, FP_ERR_UNSUPPORTED, "fp_csr_plan_pack: empty matrix");
  FP_REQUIRE(m < INT32_MAX, FP_ERR_UNSUPPORTED, "fp_csr_plan_pack: m >= 2^31");
  // too wide for the shared memory of a CTA group (fp64 beyond one block, fp32 beyond 8): the
  // L2-sized column blocks of variant 20 (FP_PK_L2=1 forces them: tests, measurement)
  const char* fl2 = std::getenv("FP_PK_L2");
  if ((fl2 && std::atoi(fl2) != 0) || (cs_force <= 0 && packed_cs(n, dtype) == 0)) {
    Packed* q = new (std::nothrow) Packed;
    FP_REQUIRE(q, FP_ERR_NOMEM, "fp_csr_plan_pack: out of host memory");
    q->m = m;
    q->n = n;
    q->nnz = nnz;
    q->rowptr = rowptr;
    q->dtype = dtype;
    fp_status st = l2block_build(m, n, nnz, rowptr, colidx, val, dtype, q, s);
    if (st != FP_OK) {
      packed_free(q);
      return st;
    }
    *out = q;
    return FP_OK;
  }
  const int cs = cs_force > 0 ? cs_force : packed_cs(n, dtype);
  FP_REQUIRE(cs == 1 || cs == 2 || cs == 4 || cs == 8, FP_ERR_UNSUPPORTED,
             "fp_csr_plan_pack: n = %lld needs more than %s column blocks", (long long)n,
             dtype == FP_F64 ? "one (fp64)" : "8");
  FP_REQUIRE(dtype == FP_F32 || cs == 1, FP_ERR_UNSUPPORTED, "fp_csr_plan_pack: fp64 packs one column block only");
  const int bw = (int)((n + cs - 1) / cs);
  FP_REQUIRE(cs == 1 ? n <= packed1_max_n(dtype) : bw <= packed_max_bw(), FP_ERR_UNSUPPORTED,
             "fp_csr_plan_pack: n = %lld too wide for %d blocks", (long long)n, cs);
  const size_t vs = dtype_size(dtype);
  // one block: a tile is one window (loaded once); measurement knobs (cs > 1): FP_PK_SPAN (entries
  // per block segment before a row goes alone), FP_PK_ROWS (rows per tile: 16 / 32 / 64)
  int span = cs == 1 ? 256 : kPkLong;
  if (const char* e = std::getenv("FP_PK_SPAN"); e && cs > 1 && std::atoi(e) >= 256) span = std::atoi(e);
  int gr = kPkRows;
  if (const char* e = std::getenv("FP_PK_ROWS"); e && (std::atoi(e) == 16 || std::atoi(e) == 32)) gr = std::atoi(e);
  const DeviceInfo& di = device_info(current_device());
  int groups = cs == 1 ? di.sm_count : di.sm_count / cs;
  // column-block groups (cs > 1): CTAs of FP_PK_BSN threads (1024 default; 768: 85 registers,
  // the scatter's first window prefetched before the exchange poll)
  int bs = kPkBS;
  if (const char* e = std::getenv("FP_PK_BSN"); e && cs > 1 && std::atoi(e) == 768) bs = 768;
  int ns1 = 0;
  if (cs == 1) {  // the single-block pass: CTAs of FP_PK_BS1 (512 default) threads, as many as fit
    // measured: S3 (fp32) 0.51 ms at 1024 threads vs 0.67 at 512; C3 (fp64) 1.00 ms at 512
    // (127 registers) vs 1.21 at 1024 (64 registers: spills).  Round 2c (ring, v in the slot):
    // C3 512 / 640 / 768 / 1024 threads 0.890 / 0.922 / 1.075 / 1.467 ms; S3 0.654 / 0.565 /
    // 0.517 / 0.490 ms
    const char* e = std::getenv("FP_PK_BS1");
    const int eb = e ? std::atoi(e) : 0;
    bs = (eb == 1024 || eb == 768 || eb == 640 || eb == 512) ? eb : (dtype == FP_F64 ? 512 : 1024);
    const void* f1 = pk1_pick(dtype, true, bs);
    set_max_dynamic_smem(f1);
    ns1 = pk1_ring_ns(n, dtype, bs);
    FP_REQUIRE(pk1_smem_n(n, dtype, true, bs, ns1) + 2048 <= di.smem_optin_per_block, FP_ERR_UNSUPPORTED,
               "fp_csr_plan_pack: n = %lld too wide for %d-thread CTAs", (long long)n, bs);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, f1, bs, pk1_smem_n(n, dtype, true, bs, ns1));
    groups = di.sm_count * std::max(1, occ);
  }
  if (const char* e = std::getenv("FP_PK_GROUPS")) {  // fewer CTA groups (tests: several local ranks
    const int gg = std::atoi(e);                       // must fit the GPU at once)
    if (gg > 0 && gg < groups) groups = gg;
  }
  Packed* p = new (std::nothrow) Packed;
  FP_REQUIRE(p, FP_ERR_NOMEM, "fp_csr_plan_pack: out of host memory");
  p->m = m;
  p->n = n;
  p->nnz = nnz;
  p->cs = cs;
  p->bw = bw;
  p->groups = groups;
  p->rowptr = rowptr;
  p->dtype = dtype;
  p->bs = bs;
  p->trace_warps = bs / 32;
  p->ns1 = ns1;
  const int64_t ng = (m + gr - 1) / gr;
  uint32_t* cnt = nullptr;
  unsigned long long* gmask = nullptr;
  int64_t* gcount = nullptr;
  int64_t* gbase = nullptr;
  int64_t* al = nullptr;
  int64_t* off = nullptr;
  uint32_t* tlen = nullptr;
  int64_t* tile_row = nullptr;
  void* tmp = nullptr;
  auto cleanup = [&]() {
    for (void* b : {(void*)cnt, (void*)gmask, (void*)gcount, (void*)gbase, (void*)al, (void*)off, (void*)tlen,
                    (void*)tile_row, tmp})
      if (b) cudaFree(b);
  };
  auto fail = [&](cudaError_t e, const char* what) {
    cudaGetLastError();
    set_error("fp_csr_plan_pack: %s: %s", what, cudaGetErrorString(e));
    cleanup();
    packed_free(p);
    return e == cudaErrorMemoryAllocation ? FP_ERR_NOMEM : FP_ERR_CUDA;
  };
#define PK_TRY(call, what)                 \
  do {                                     \
    cudaError_t e_ = (call);               \
    if (e_ != cudaSuccess) return fail(e_, what); \
  } while (0)
  PK_TRY(cudaMalloc((void**)&cnt, (size_t)cs * m * 4), "alloc");
  PK_TRY(cudaMalloc((void**)&gmask, (size_t)ng * 8), "alloc");
  PK_TRY(cudaMalloc((void**)&gcount, (size_t)ng * 8), "alloc");
  PK_TRY(cudaMalloc((void**)&gbase, (size_t)ng * 8), "alloc");
  const int tb = 256;
  const int grid_r = (int)std::min<int64_t>((m + tb - 1) / tb, (int64_t)di.sm_count * 32);
  const int grid_g = (int)std::min<int64_t>((ng + tb - 1) / tb, (int64_t)di.sm_count * 32);
  k_pk_count<<<grid_r, tb, 0, s>>>(m, rowptr, colidx, cs, bw, cnt);
  k_pk_tiles<<<grid_g, tb, 0, s>>>(m, gr, cs, span, cnt, gmask, gcount);
  size_t tb_bytes = 0;
  PK_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb_bytes, gcount, gbase, ng, s), "scan");
  size_t tmp_bytes = tb_bytes;
  PK_TRY(cudaMalloc(&tmp, tmp_bytes), "alloc");
  PK_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb_bytes, gcount, gbase, ng, s), "scan");
  int64_t hb[2] = {0, 0};
  PK_TRY(cudaMemcpyAsync(&hb[0], gbase + ng - 1, 8, cudaMemcpyDeviceToHost, s), "copy");
  PK_TRY(cudaMemcpyAsync(&hb[1], gcount + ng - 1, 8, cudaMemcpyDeviceToHost, s), "copy");
  PK_TRY(cudaStreamSynchronize(s), "sync");
  const int64_t ntiles = hb[0] + hb[1];
  p->ntiles = ntiles;
  const int64_t segs = (int64_t)cs * ntiles;
  PK_TRY(cudaMalloc((void**)&tile_row, (size_t)(ntiles + 1) * 8), "alloc");
  PK_TRY(cudaMalloc((void**)&tlen, (size_t)segs * 4), "alloc");
  PK_TRY(cudaMalloc((void**)&al, (size_t)segs * 8), "alloc");
  PK_TRY(cudaMalloc((void**)&off, (size_t)segs * 8), "alloc");
  k_pk_tile_rows<<<grid_g, tb, 0, s>>>(m, gr, cs, ntiles, cnt, gmask, gbase, tile_row, tlen, al);
  PK_TRY(cub::DeviceScan::ExclusiveSum(nullptr, tb_bytes, al, off, segs, s), "scan");
  if (tb_bytes > tmp_bytes) {
    cudaFree(tmp);
    tmp = nullptr;
    tmp_bytes = tb_bytes;
    PK_TRY(cudaMalloc(&tmp, tmp_bytes), "alloc");
  }
  PK_TRY(cub::DeviceScan::ExclusiveSum(tmp, tb_bytes, al, off, segs, s), "scan");
  int64_t ht[2] = {0, 0};
  PK_TRY(cudaMemcpyAsync(&ht[0], off + segs - 1, 8, cudaMemcpyDeviceToHost, s), "copy");
  PK_TRY(cudaMemcpyAsync(&ht[1], al + segs - 1, 8, cudaMemcpyDeviceToHost, s), "copy");
  PK_TRY(cudaStreamSynchronize(s), "sync");
  const int64_t total = ht[0] + ht[1];
  if (total / 8 >= (int64_t)UINT32_MAX) return fail(cudaErrorInvalidValue, "too many nonzeros for 32-bit offsets");
  p->entries = total;
  PK_TRY(cudaMalloc((void**)&p->tile_desc, (size_t)segs * sizeof(uint4)), "alloc");
  k_pk_desc<<<(int)std::min<int64_t>((segs + tb - 1) / tb, (int64_t)di.sm_count * 32), tb, 0, s>>>(
      segs, ntiles, off, tlen, tile_row, p->tile_desc);
  const int64_t cap = total + 8;  // + the padding block the inactive lanes load
  PK_TRY(cudaMalloc((void**)&p->cr, (size_t)cap * 4), "alloc");
  PK_TRY(cudaMalloc((void**)&p->val, (size_t)cap * vs), "alloc");
  // padding entries (segment tails up to the next 16-byte boundary): the block's zero / dummy
  // column, the tile's last row slot, value 0
  k_pk_fill<<<(int)std::min<int64_t>((cap + tb - 1) / tb, (int64_t)di.sm_count * 32), tb, 0, s>>>(
      cap, p->cr, ((uint32_t)bw * 4u) | ((uint32_t)(kPkRows - 1) << kPkRidShift));
  PK_TRY(cudaMemsetAsync(p->val, 0, (size_t)cap * vs, s), "memset");
  const int sgrid = (int)std::min<int64_t>((ng + 7) / 8, (int64_t)di.sm_count * 16);
  if (dtype == FP_F64)
    k_pk_scatter<double><<<sgrid, 256, 0, s>>>(m, gr, cs, bw, ntiles, rowptr, colidx, (const double*)val, gmask, gbase,
                                              p->tile_desc, p->cr, (double*)p->val);
  else
    k_pk_scatter<float><<<sgrid, 256, 0, s>>>(m, gr, cs, bw, ntiles, rowptr, colidx, (const float*)val, gmask, gbase,
                                             p->tile_desc, p->cr, (float*)p->val);
  if (std::getenv("FP_PK_NOBANK") == nullptr)  // measurement: FP_PK_NOBANK=1 keeps the row order
  {
    const int bgrid = (int)std::min<int64_t>((segs + 7) / 8, (int64_t)di.sm_count * 8);
    const int ls = std::getenv("FP_PK_NOLS") == nullptr;  // measurement: greedy only
    if (dtype == FP_F64)  // 8-byte y gathers: bank pairs (col mod 16)
      k_pk_bankopt<double><<<bgrid, 256, 0, s>>>(segs, p->tile_desc, p->cr, (double*)p->val, 15, ls);
    else
      k_pk_bankopt<float><<<bgrid, 256, 0, s>>>(segs, p->tile_desc, p->cr, (float*)p->val, 31, ls);
  }
  if (cs == 1) {  // k_pk1's lane-interleaved windows (after the bank balancing, which is by logical slot)
    const int igrid = (int)std::min<int64_t>((segs + 7) / 8, (int64_t)di.sm_count * 16);
    if (dtype == FP_F64)
      k_pk_interleave<double><<<igrid, 256, 0, s>>>(segs, p->tile_desc, p->cr, (double*)p->val);
    else
      k_pk_interleave<float><<<igrid, 256, 0, s>>>(segs, p->tile_desc, p->cr, (float*)p->val);
  }
  const int nq = groups * (bs / 32);
  if (ntiles >= INT32_MAX) return fail(cudaErrorInvalidValue, "too many tiles");
  PK_TRY(cudaMalloc((void**)&p->wtile, (size_t)(nq + 1) * 4), "alloc");
  {  // measurement knobs: FP_PK_ROWCOST (default kPkRowCost), FP_PK_TILECOST (default 0)
    const char* r = std::getenv("FP_PK_ROWCOST");
    const char* t = std::getenv("FP_PK_TILECOST");
    k_pk_partition<<<(nq + 1 + 127) / 128, 128, 0, s>>>(ntiles, nq, tile_row, rowptr, p->wtile,
                                                         r ? std::atoi(r) : kPkRowCost, t ? std::atoi(t) : 0);
  }
  // per-call state: exchange slots (zero), the call counter (starts at 1), partials, spill (zero)
  const int ns = cs > 1 ? PkSlots<1>::NS : 1;
  const size_t xbytes = (size_t)groups * (bs / 32) * ns * (cs + 1) * kPkRows * 8;
  PK_TRY(cudaMalloc((void**)&p->xch, xbytes), "alloc");
  PK_TRY(cudaMemsetAsync(p->xch, 0, xbytes, s), "memset");
  PK_TRY(cudaMalloc((void**)&p->epoch, 16), "alloc");
  const unsigned one = 1;
  PK_TRY(cudaMemcpyAsync(p->epoch, &one, 4, cudaMemcpyHostToDevice, s), "copy");
  PK_TRY(cudaMalloc((void**)&p->part, (size_t)groups * n * 8), "alloc");
  const size_t spb = (size_t)cs * (bw + 1) * 8;  // [block][bw + 1] (+ the dummy column)
  PK_TRY(cudaMalloc((void**)&p->spill, spb), "alloc");
  PK_TRY(cudaMemsetAsync(p->spill, 0, spb, s), "memset");
  // tiles per warp-quad must stay below 2^20 (the exchange tag)
  {
    std::vector<int32_t> hw(nq + 1);
    PK_TRY(cudaMemcpyAsync(hw.data(), p->wtile, (size_t)(nq + 1) * 4, cudaMemcpyDeviceToHost, s), "copy");
    PK_TRY(cudaStreamSynchronize(s), "sync");
    int64_t mx = 0;
    for (int i = 0; i < nq; ++i) mx = std::max<int64_t>(mx, (int64_t)hw[i + 1] - hw[i]);
    p->max_tiles_per_warp = mx;
    if (mx >= (1 << 20)) {
      cleanup();
      packed_free(p);
      set_error("fp_csr_plan_pack: %lld tiles for one warp (limit 2^20)", (long long)mx);
      return FP_ERR_UNSUPPORTED;
    }
  }
#undef PK_TRY
  cleanup();
  *out = p;
  return FP_OK;
}

size_t pk1_smem(const Packed* p, bool has_y) { return pk1_smem_n(p->n, p->dtype, has_y, p->bs, p->ns1); }

fp_status packed_exec(Packed* p, const PatternArgs& a, cudaStream_t s) {
  if (p->mode == 1) return l2block_exec(p, a, s);
  const bool has_y = a.y != nullptr;
  if (p->cs == 1) {
    const void* f1 = pk1_pick(p->dtype, has_y, p->bs);
    set_max_dynamic_smem(f1);
    Pk1Args k{};
    k.m = p->m;
    k.n = p->n;
    k.ntiles = p->ntiles;
    k.ns = p->ns1;
    k.tile_desc = p->tile_desc;
    k.wtile = p->wtile;
    k.cr = p->cr;
    k.val = p->val;
    k.y = a.y;
    k.v = a.v;
    k.alpha = a.alpha;
    k.hbits = pk_headroom();
    k.part = p->part;
    k.spill = p->spill;
    void* args[] = {&k};
    FP_CUDA(cudaLaunchKernel(f1, dim3(p->groups), dim3(p->bs), args, pk1_smem(p, has_y), s));
    const int fb = 256;
    const int fg = (int)std::min<int64_t>((p->n + fb - 1) / fb, 8 * (int64_t)device_info(current_device()).sm_count);
    if (p->dtype == FP_F64)
      k_pk1_finalize<double><<<fg, fb, 0, s>>>(p->n, p->groups, p->part, p->spill, (const double*)a.z, a.beta,
                                               a.add_beta_z ? 1 : 0, a.accumulate ? 1 : 0, (double*)a.w);
    else
      k_pk1_finalize<float><<<fg, fb, 0, s>>>(p->n, p->groups, p->part, p->spill, (const float*)a.z, a.beta,
                                              a.add_beta_z ? 1 : 0, a.accumulate ? 1 : 0, (float*)a.w);
    FP_CUDA(cudaGetLastError());
    return FP_OK;
  }
  const void* f = pk_pick(p->cs, has_y, p->bs);
  FP_REQUIRE(f, FP_ERR_UNSUPPORTED, "fp_csr_plan_exec: no packed kernel for %d blocks", p->cs);
  set_max_dynamic_smem(f);
  PkArgs k{};
  k.n = p->n;
  k.bw = p->bw;
  k.groups = p->groups;
  k.ntiles = p->ntiles;
  k.tile_desc = p->tile_desc;
  k.padidx = p->entries;
  k.wtile = p->wtile;
  k.cr = p->cr;
  k.val = (const float*)p->val;
  k.y = (const float*)a.y;
  k.v = (const float*)a.v;
  k.alpha = (float)a.alpha;
  k.hbits = pk_headroom();
  k.xch = p->xch;
  k.epoch = p->epoch;
  k.part = p->part;
  k.spill = p->spill;
  k.trace = nullptr;
  {  // measurement knob: FP_PK_NAP = ns a warp sleeps between polls (0: spin, the default;
     // 64 ns left some warp-quads 2x behind on C4: 13.4 vs 7.9 ms)
    const char* f = std::getenv("FP_PK_PF");
    k.pf = f ? std::atoi(f) : 2;  // measured on C4: none 5.71, per-lane 5.69, bulk 5.63 ms
    const char* n = std::getenv("FP_PK_NAP");
    k.nap = n ? std::atoi(n) : 0;
  }
  if (std::getenv("FP_PK_TRACE")) {  // measurement: per-warp timing of the pass (kept in the plan)
    if (!p->trace) cudaMalloc((void**)&p->trace, (size_t)p->groups * p->cs * (p->bs / 32) * 64);
    k.trace = p->trace;
  }
  const size_t smem = ((has_y ? (size_t)((p->bw + 4) & ~3) : 0) + (size_t)p->bw + 33) * 4;
  void* args[] = {&k};
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(p->groups * p->cs);
  cfg.blockDim = dim3(p->bs);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;  // the CTAs of a group wait on each other
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = p->cs > 1 ? 1 : 0;
  FP_CUDA(cudaLaunchKernelExC(&cfg, f, args));
  const int fb = 256;
  const int fg = (int)std::min<int64_t>((p->n + fb - 1) / fb, 8 * (int64_t)device_info(current_device()).sm_count);
  k_pk_finalize<<<fg, fb, 0, s>>>(p->n, p->bw, p->groups, p->part, p->spill, (const float*)a.z, a.beta,
                                  a.add_beta_z ? 1 : 0, a.accumulate ? 1 : 0, (float*)a.w, p->epoch);
  FP_CUDA(cudaGetLastError());
  return FP_OK;
}

void packed_launch(const Packed* p, fp_launch* L) {
  if (p->mode == 1) return l2block_launch(p, L);
  *L = fp_launch{};
  L->variant = FP_VAR_CSR_PACKED;
  L->vs = 32;
  L->tl = kPkLong;
  L->bs = p->bs;
  L->grid = p->groups * p->cs;
  L->cluster = p->cs;
  L->smem_bytes = p->cs == 1 ? (int)pk1_smem(p, true) : ((p->bw + 4) & ~3) * 4 + (p->bw + 33) * 4;
  L->tl = p->cs == 1 ? 256 : kPkLong;
  L->blocks_per_sm = 1;
  cudaFuncAttributes fa{};
  if (cudaFuncGetAttributes(&fa, p->cs == 1 ? pk1_pick(p->dtype, true, p->bs) : pk_pick(p->cs, true, p->bs)) == cudaSuccess)
    L->regs_per_thread = fa.numRegs;
  else cudaGetLastError();
}

}  // namespace fp
