// common.cuh -- shared internals of libfusedpat (error state, device info, per-stream
// workspace, sm_100a load/reduce primitives).  Product code only; no oracle code here.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "fusedpat.h"

namespace fp {

// ---------------------------------------------------------------------------- errors
void set_error(const char* fmt, ...);
const char* last_error_text();
fp_status cuda_fail(cudaError_t e, const char* what);

#define FP_CUDA(call)                                          \
  do {                                                         \
    cudaError_t e_ = (call);                                   \
    if (e_ != cudaSuccess) return ::fp::cuda_fail(e_, #call);  \
  } while (0)

#define FP_REQUIRE(cond, status, ...)      \
  do {                                     \
    if (!(cond)) {                         \
      ::fp::set_error(__VA_ARGS__);        \
      return status;                       \
    }                                      \
  } while (0)

// ---------------------------------------------------------------------------- device info
struct DeviceInfo {
  int ordinal;
  int sm_count;
  int max_threads_per_sm;
  int max_blocks_per_sm;
  int regs_per_sm;
  size_t smem_per_sm;
  size_t smem_optin_per_block;
  size_t l2_bytes;
};
const DeviceInfo& device_info(int ordinal);
int current_device();

// ---------------------------------------------------------------------------- workspace
// One per (device, stream).  acc: fp64 grid accumulator, ALWAYS all-zero between launches
// (the finalising CTA re-zeroes what it consumed).  counters: [0] CTA-done ticket,
// [1] dynamic row-chunk counter; both reset to 0 by the finalising CTA.
// Extra per-workspace buffers (workspace_buffer slots).
enum { kWsBins = 0, kWsBinsZero = 1, kWsSlots = 4 };
struct Workspace {
  double* acc = nullptr;
  size_t acc_cap = 0;          // elements
  unsigned long long* counters = nullptr;
  void* scratch = nullptr;     // general device scratch (row stats, CG scalars)
  size_t scratch_cap = 0;      // bytes
  void* buf[kWsSlots] = {};    // kWsBins: variant-17 messages; kWsBinsZero: its all-zero vectors
  size_t buf_cap[kWsSlots] = {};
};
// Returns nullptr (and sets the error) on allocation failure.  Growing allocates a larger
// buffer and retires the old one (freed by release_all_workspaces); steady-state calls never
// allocate.  Calls made while the stream is being captured get their own workspace.
Workspace* workspace(cudaStream_t s, size_t acc_elems, size_t scratch_bytes);
// Slot `slot` of the (device, stream[, capture]) workspace with at least `bytes`; a new
// allocation is zero-filled when `zero` (callers that need an all-zero invariant keep it).
void* workspace_buffer(cudaStream_t s, int slot, size_t bytes, bool zero);
void release_all_workspaces();
// cudaFuncAttributeMaxDynamicSharedMemorySize = the device's per-block maximum, once per kernel
void set_max_dynamic_smem(const void* f);

// ---------------------------------------------------------------------------- helpers
inline size_t dtype_size(fp_dtype t) { return t == FP_F64 ? 8 : 4; }
inline bool valid_dtype(fp_dtype t) { return t == FP_F32 || t == FP_F64; }

// [a, a+na) and [b, b+nb) byte ranges overlap?
inline bool overlaps(const void* a, size_t na, const void* b, size_t nb) {
  if (!a || !b || na == 0 || nb == 0) return false;
  uintptr_t x = (uintptr_t)a, y = (uintptr_t)b;
  return x < y + nb && y < x + na;
}

}  // namespace fp

// ------------------------------------------------------------------------------------------
// Device primitives (sm_100a).
// ------------------------------------------------------------------------------------------
#ifdef __CUDACC__
namespace fpd {

// Streaming read-once loads of X: bypass L1 allocation, evict-first in L2 (X is far larger
// than L2 and never re-read within a call).  256-bit loads are sm_100 LDG.E.256.
__device__ __forceinline__ void ld_stream32(const float* p, float (&r)[8]) {
  asm("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]), "=f"(r[6]), "=f"(r[7])
               : "l"(p));
}
__device__ __forceinline__ void ld_stream32(const double* p, double (&r)[4]) {
  asm("ld.global.nc.L1::no_allocate.L2::evict_first.v4.f64 {%0,%1,%2,%3}, [%4];"
               : "=d"(r[0]), "=d"(r[1]), "=d"(r[2]), "=d"(r[3])
               : "l"(p));
}
__device__ __forceinline__ void ld_stream16(const float* p, float (&r)[4]) {
  asm("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3])
               : "l"(p));
}
__device__ __forceinline__ void ld_stream16(const double* p, double (&r)[2]) {
  asm("ld.global.nc.L1::no_allocate.L2::256B.v2.f64 {%0,%1}, [%2];" : "=d"(r[0]), "=d"(r[1]) : "l"(p));
}
__device__ __forceinline__ void ld_stream4(const float* p, float (&r)[1]) {
  asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r[0]) : "l"(p));
}
__device__ __forceinline__ void ld_stream4(const double* p, double (&r)[1]) {
  asm("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(r[0]) : "l"(p));
}

// Load E = CB/sizeof(T) consecutive elements (CB-byte aligned).
template <int CB, typename T, int E>
__device__ __forceinline__ void ld_chunk(const T* p, T (&r)[E]) {
  if constexpr (CB == 32) {
    ld_stream32(p, r);
  } else if constexpr (CB == 16) {
    ld_stream16(p, r);
  } else {
    ld_stream4(p, r);
  }
}

// Read-once streaming loads for CSR structure (colidx / val / rowptr).
__device__ __forceinline__ int ld_once(const int* p) {
  int r;
  asm("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ float ld_once(const float* p) {
  float r;
  asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ double ld_once(const double* p) {
  double r;
  asm("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(r) : "l"(p));
  return r;
}

// ---- mbarrier + bulk (TMA) copies global -> shared (SASS UBLKCP.S.G + SYNCS.*)
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
// generic-proxy accesses of shared memory before this point are ordered before later
// async-proxy (bulk copy) writes to it
__device__ __forceinline__ void fence_proxy_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// bytes: multiple of 16; src, dst 16-byte aligned
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// Cluster-scope one-way signalling (no cluster barrier, no MEMBAR.GPU): st.async writes a value
// into a peer CTA's shared memory and credits its bytes to the peer's mbarrier (complete_tx);
// the peer waits on that mbarrier with cluster-scope acquire.
__device__ __forceinline__ unsigned mapa_u32(unsigned addr, unsigned rank) {
  unsigned r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
__device__ __forceinline__ void st_async(unsigned raddr, float v, unsigned rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b32 [%0], %1, [%2];" ::"r"(raddr),
               "r"(__float_as_uint(v)), "r"(rbar)
               : "memory");
}
__device__ __forceinline__ void st_async(unsigned raddr, double v, unsigned rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(raddr),
               "l"(__double_as_longlong(v)), "r"(rbar)
               : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, unsigned parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAITC_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAITC_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// 16-byte shared-memory vectors (LDS.128) for the bulk-copy ring
template <typename T>
struct Vec16;
template <>
struct Vec16<float> {
  using type = float4;
  __device__ __forceinline__ static void unpack(const float4& t, float* o) {
    o[0] = t.x; o[1] = t.y; o[2] = t.z; o[3] = t.w;
  }
};
template <>
struct Vec16<double> {
  using type = double2;
  __device__ __forceinline__ static void unpack(const double2& t, double* o) {
    o[0] = t.x; o[1] = t.y;
  }
};

// Gathers of y that should stay in L1 (y is re-read randomly; X streams past it).
// cp.async.bulk.prefetch.L2: one instruction pulls a contiguous byte range into L2 (TMA unit;
// no registers, no completion to wait for).  The range is widened to 16-byte alignment.
__device__ __forceinline__ void prefetch_l2(const void* p, size_t bytes) {
  const uintptr_t a = reinterpret_cast<uintptr_t>(p) & ~(uintptr_t)15;
  const uintptr_t e = (reinterpret_cast<uintptr_t>(p) + bytes + 15) & ~(uintptr_t)15;
  if (e > a)
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a), "r"((unsigned)(e - a)) : "memory");
}

// one shared-memory compare-and-swap of a float / double (returns the previous value)
__device__ __forceinline__ float cas_shared(float* p, float cmp, float val) {
  return __int_as_float(atomicCAS(reinterpret_cast<int*>(p), __float_as_int(cmp), __float_as_int(val)));
}
__device__ __forceinline__ double cas_shared(double* p, double cmp, double val) {
  return __longlong_as_double((long long)atomicCAS(reinterpret_cast<unsigned long long*>(p),
                                                   (unsigned long long)__double_as_longlong(cmp),
                                                   (unsigned long long)__double_as_longlong(val)));
}
__device__ __forceinline__ bool same_bits(float a, float b) { return __float_as_int(a) == __float_as_int(b); }
__device__ __forceinline__ bool same_bits(double a, double b) { return __double_as_longlong(a) == __double_as_longlong(b); }

__device__ __forceinline__ float ld_keep(const float* p) {
  float r;
  asm("ld.global.nc.L1::evict_last.f32 %0, [%1];" : "=f"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ double ld_keep(const double* p) {
  double r;
  asm("ld.global.nc.L1::evict_last.f64 %0, [%1];" : "=d"(r) : "l"(p));
  return r;
}

// Fire-and-forget fp reduction into global memory (SASS REDG.E.ADD.F32/F64).
__device__ __forceinline__ void red_add(float* p, float v) { atomicAdd(p, v); }
__device__ __forceinline__ void red_add(double* p, double v) { atomicAdd(p, v); }

// Sum over the VS lanes of a vector (VS a power of two <= 32, vectors aligned in the warp);
// every lane of the vector receives the total.
template <int VS, typename T>
__device__ __forceinline__ T vector_allreduce(T x) {
#pragma unroll
  for (int off = VS / 2; off > 0; off >>= 1) x += __shfl_xor_sync(0xffffffffu, x, off);
  return x;
}

}  // namespace fpd
#endif
