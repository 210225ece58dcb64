// comm.cu -- multi-GPU row sharding: NCCL communicator, one in-place
// allreduce of w per evaluation, nnz-balanced shard bounds, the *_dist entry points.
//
// Eq. (1) is a sum over rows of X[r,:]^T (v[r] X[r,:] y) (Eq. 2/3), so a row
// partition needs exactly one exchange: the n-vector sum of per-rank partials.  beta*z is
// added on rank 0 only (reading R18).  The paper is single-GPU; this layer is new.
#include <cuda.h>
#include <nccl.h>
#include <string.h>

#include <algorithm>
#include <chrono>
#include <condition_variable>
#include <memory>
#include <mutex>
#include <vector>

#include "kernels.cuh"

constexpr int kMaxPeers = 8;  // one NVSwitch node

// Host rendezvous of a single-process local group.  A device allocation is an implicit
// synchronisation point between streams: a rank allocating its workspace on its first call
// would wait for another rank's barrier kernel, which waits for the allocating rank -- so the
// ranks of one process meet on the host before any of them launches its barrier kernel (by
// then every rank has finished allocating).  Not needed across processes.
struct LocalSync {
  std::mutex mu;
  std::condition_variable cv;
  int P = 1, count = 0;
  uint64_t gen = 0;
  bool arrive_and_wait() {
    std::unique_lock<std::mutex> lk(mu);
    const uint64_t g = gen;
    if (++count == P) {
      count = 0;
      ++gen;
      cv.notify_all();
      return true;
    }
    return cv.wait_for(lk, std::chrono::seconds(30), [&] { return gen != g; });
  }
};

// Peer (P2P) exchange state.  Every rank owns a symmetric buffer [D0: cap][D1: cap][flags:
// kMaxPeers x u64] mapped into every other rank (CUDA IPC across processes, plain pointers in a
// single-process group).  Call e writes its partial into D[e & 1] of its own buffer, publishes
// epoch e into flags[rank] of every rank, waits until its own flags[k] >= e for all k, then
// every rank sums D_k[e & 1] over k in rank order (identical bits on every rank).  Reuse of
// D[e & 1] at call e + 2 is safe: passing call e + 1's barrier means every peer finished
// reading call e.
struct fp_comm {
  ncclComm_t nccl = nullptr;
  int rank = 0;
  int size = 1;
  int device = 0;
  int mode = FP_COMM_NCCL;
  size_t cap = 0;                             // bytes of one D buffer
  unsigned char* sym = nullptr;               // own symmetric buffer
  unsigned char* peer[kMaxPeers] = {};        // every rank's buffer (peer[rank] == sym)
  bool ipc_mapped[kMaxPeers] = {};            // opened with cudaIpcOpenMemHandle
  uint64_t epoch = 0;
  unsigned* timeout_flag = nullptr;           // device: set if a barrier gave up waiting
  std::shared_ptr<LocalSync> lsync;           // local groups only
  // NVLS (FP_COMM_NVLS): one multicast object over all ranks' physical buffers (same layout
  // as sym); uc = this rank's unicast mapping, mc = the multicast mapping
  CUmemGenericAllocationHandle mc_handle = 0, ph_handle = 0;
  unsigned char* uc = nullptr;
  unsigned char* mc = nullptr;
  size_t mc_size = 0;
  bool nvls = false;
};

namespace fp {
fp_status run_dense(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
fp_status run_csr(const PatternArgs& a, const fp_launch* override_, cudaStream_t s);
PatternArgs dense_args(int64_t m, int64_t n, const void* X, int64_t ld, const void* y, const void* v, const void* z,
                       double alpha, double beta, void* w, fp_dtype dtype);
PatternArgs csr_args(int64_t m, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* colidx,
                     const void* val, const void* y, const void* v, const void* z, double alpha, double beta, void* w,
                     fp_dtype dtype);

static fp_status nccl_fail(ncclResult_t r, const char* what) {
  set_error("%s: %s", what, ncclGetErrorString(r));
  return FP_ERR_NCCL;
}
}  // namespace fp

namespace {
fp_status peer_begin(fp_comm* c, size_t bytes, cudaStream_t s, void** D);
fp_status peer_finish(fp_comm* c, int64_t n, fp_dtype dt, const void* z, double beta, void* w, cudaStream_t s);

// Peer-mode pattern with a CSR plan (fp_csr_plan_dist): as dist_peer, the local pass on the plan
fp_status dist_peer_plan(fp::PatternArgs a, const fp_csr_plan* plan, fp_comm* comm, cudaStream_t s) {
  if (a.n == 0) return FP_OK;
  void* D = nullptr;
  fp_status st = peer_begin(comm, (size_t)a.n * fp::dtype_size(a.dtype), s, &D);
  if (st != FP_OK) return st;
  void* w = a.w;
  const void* z = a.z;
  const double beta = a.beta;
  a.w = D;
  a.add_beta_z = false;
  st = fp::plan_run(plan, a, s);
  if (st != FP_OK) return st;
  return peer_finish(comm, a.n, a.dtype, beta != 0.0 ? z : nullptr, beta, w, s);
}

// Peer-mode pattern: the local pass writes this rank's partial alpha X_r^T(v_r (.) X_r y)
// straight into its symmetric D buffer (no beta z), then the exchange sums the ranks' D in
// rank order and adds beta z once: every rank ends with the same bits.
fp_status dist_peer(fp::PatternArgs a, bool csr, fp_comm* comm, cudaStream_t s) {
  if (a.n == 0) return FP_OK;
  void* D = nullptr;
  fp_status st = peer_begin(comm, (size_t)a.n * fp::dtype_size(a.dtype), s, &D);
  if (st != FP_OK) return st;
  void* w = a.w;
  const void* z = a.z;
  const double beta = a.beta;
  a.w = D;
  a.add_beta_z = false;
  st = csr ? fp::run_csr(a, nullptr, s) : fp::run_dense(a, nullptr, s);
  if (st != FP_OK) return st;
  return peer_finish(comm, a.n, a.dtype, beta != 0.0 ? z : nullptr, beta, w, s);
}
}  // namespace

namespace {

struct PeerTab {
  unsigned char* p[kMaxPeers];
  size_t cap;
  int P, rank;
  uint64_t epoch;
  unsigned* timeout_flag;
};

__device__ __forceinline__ uint64_t* flags_of(unsigned char* buf, size_t cap) {
  return reinterpret_cast<uint64_t*>(buf + 2 * cap);
}

// Publish this rank's arrival (epoch) into every rank's flags[rank], then (wait = 1) wait
// until every rank has arrived here.  One warp; release/acquire at system scope (the flags and
// the D buffers are read over NVLink).  Gives up after ~20 s (sets *timeout_flag) rather than
// hang.  wait = 0: publish only (single-device local groups, see peer_finish).
__global__ void k_peer_barrier(const PeerTab t, int wait) {
  const int lane = threadIdx.x;
  __threadfence_system();
  if (lane < t.P) {
    uint64_t* f = flags_of(t.p[lane], t.cap) + t.rank;
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(t.epoch) : "memory");
  }
  if (wait && lane < t.P) {
    const uint64_t* f = flags_of(t.p[t.rank], t.cap) + lane;
    uint64_t t0, now, v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    while (true) {
      asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(f) : "memory");
      if (v >= t.epoch) break;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
      if (now - t0 > 20000000000ull) {
        atomicExch(t.timeout_flag, 1u);
        break;
      }
      __nanosleep(100);
    }
  }
  __syncwarp();
}

// w[j] = sum_k D_k[j] (rank order, fp64 accumulation) + beta z[j]: the same bits on every rank
template <typename T>
__global__ void k_peer_sum(const PeerTab t, int64_t n, const T* __restrict__ z, double beta, T* w) {
  const size_t off = (t.epoch & 1) * t.cap;
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;
#pragma unroll 1
    for (int k = 0; k < t.P; ++k) s += (double)reinterpret_cast<const T*>(t.p[k] + off)[j];
    if (z && beta != 0.0) s += beta * (double)z[j];
    w[j] = (T)s;
  }
}

__global__ void k_copy_bytes(unsigned char* __restrict__ d, const unsigned char* __restrict__ s, size_t bytes) {
  const size_t n16 = ((uintptr_t)d % 16 == 0 && (uintptr_t)s % 16 == 0) ? bytes / 16 : 0;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x)
    reinterpret_cast<uint4*>(d)[i] = reinterpret_cast<const uint4*>(s)[i];
  for (size_t i = n16 * 16 + (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < bytes;
       i += (size_t)gridDim.x * blockDim.x)
    d[i] = s[i];
}

// NVLS barrier: one multimem red increments the epoch counter in EVERY rank's copy (release,
// system scope); then wait until the local copy reaches P * epoch (acquire).
__global__ void k_nvls_barrier(unsigned long long* mc_cnt, const unsigned long long* uc_cnt, unsigned long long target,
                               unsigned* timeout_flag) {
  if (threadIdx.x != 0) return;
  __threadfence_system();
  asm volatile("multimem.red.release.sys.global.add.u64 [%0], %1;" ::"l"(mc_cnt), "l"(1ull) : "memory");
  uint64_t t0, now;
  unsigned long long v;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  while (true) {
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(uc_cnt) : "memory");
    if (v >= target) break;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
    if (now - t0 > 20000000000ull) {
      atomicExch(timeout_flag, 1u);
      break;
    }
    __nanosleep(100);
  }
}

// w[j] = (in-switch sum over ranks of D[j]) + beta z[j]: multimem.ld_reduce on the multicast
// address returns the sum of every rank's copy in one load
__device__ __forceinline__ double ld_reduce(const double* p) {
  double v;
  asm volatile("multimem.ld_reduce.relaxed.sys.global.add.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ float ld_reduce(const float* p) {
  float v;
  asm volatile("multimem.ld_reduce.relaxed.sys.global.add.f32 %0, [%1];" : "=f"(v) : "l"(p) : "memory");
  return v;
}
template <typename T>
__global__ void k_nvls_sum(const T* mcD, int64_t n, const T* __restrict__ z, double beta, T* w) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    double s = (double)ld_reduce(mcD + j);
    if (z && beta != 0.0) s += beta * (double)z[j];
    w[j] = (T)s;
  }
}

PeerTab peer_tab(const fp_comm* c) {
  PeerTab t{};
  for (int k = 0; k < c->size; ++k) t.p[k] = c->peer[k];
  t.cap = c->cap;
  t.P = c->size;
  t.rank = c->rank;
  t.epoch = c->epoch;
  t.timeout_flag = c->timeout_flag;
  return t;
}

bool capturing(cudaStream_t s) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(s, &st) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return st != cudaStreamCaptureStatusNone;
}

// Start call e: returns this rank's D[e & 1] (where the local partial goes).
fp_status peer_begin(fp_comm* c, size_t bytes, cudaStream_t s, void** D) {
  FP_REQUIRE(bytes <= c->cap, FP_ERR_INVALID_ARG, "peer exchange: %zu B exceed the %zu B enabled", bytes, c->cap);
  FP_REQUIRE(!capturing(s), FP_ERR_UNSUPPORTED,
             "peer exchange: not capturable in a CUDA graph (its epoch advances per call); use NCCL mode");
  c->epoch += 1;
  *D = (c->nvls ? c->uc : c->sym) + (c->epoch & 1) * c->cap;
  return FP_OK;
}

// Finish call e: barrier, then w = sum_k D_k + beta z.
//
// Single-device local groups (lsync): the ranks' kernels share one GPU, and nothing makes
// separate launches that wait on one another run at the same time (a spinning barrier can
// hold resources a peer's persistent or cooperative pass needs: deadlock, or a context-switch
// timeout).  So no kernel ever waits there for a launch that has not completed: each rank
// publishes its flag with a non-waiting launch, synchronises its stream, meets the others on
// the host (every rank's partial and flag are then complete), and only then launches the
// barrier, whose wait is satisfied on its first poll.  Across GPUs (IPC / NVLS) each rank's
// barrier kernel runs on its own device and publishes + waits in one launch.
fp_status peer_finish(fp_comm* c, int64_t n, fp_dtype dt, const void* z, double beta, void* w, cudaStream_t s) {
  if (c->lsync) {
    k_peer_barrier<<<1, 32, 0, s>>>(peer_tab(c), 0);
    FP_CUDA(cudaGetLastError());
    FP_CUDA(cudaStreamSynchronize(s));
    FP_REQUIRE(c->lsync->arrive_and_wait(), FP_ERR_CUDA, "local group: ranks did not meet within 30 s");
  }
  if (c->nvls) {
    unsigned long long* cnt_off = (unsigned long long*)(2 * c->cap);
    k_nvls_barrier<<<1, 32, 0, s>>>((unsigned long long*)(c->mc + (size_t)cnt_off),
                                    (const unsigned long long*)(c->uc + (size_t)cnt_off),
                                    (unsigned long long)c->size * c->epoch, c->timeout_flag);
    FP_CUDA(cudaGetLastError());
    const int grid = (int)std::min<int64_t>((n + 255) / 256, 4 * fp::device_info(c->device).sm_count);
    const size_t off = (c->epoch & 1) * c->cap;
    if (n > 0) {
      if (dt == FP_F64)
        k_nvls_sum<double><<<grid, 256, 0, s>>>((const double*)(c->mc + off), n, (const double*)z, beta, (double*)w);
      else
        k_nvls_sum<float><<<grid, 256, 0, s>>>((const float*)(c->mc + off), n, (const float*)z, beta, (float*)w);
      FP_CUDA(cudaGetLastError());
    }
    return FP_OK;
  }
  const PeerTab t = peer_tab(c);
  k_peer_barrier<<<1, 32, 0, s>>>(t, 1);
  FP_CUDA(cudaGetLastError());
  const int grid = (int)std::min<int64_t>((n + 255) / 256, 4 * fp::device_info(c->device).sm_count);
  if (n > 0) {
    if (dt == FP_F64) k_peer_sum<double><<<grid, 256, 0, s>>>(t, n, (const double*)z, beta, (double*)w);
    else k_peer_sum<float><<<grid, 256, 0, s>>>(t, n, (const float*)z, beta, (float*)w);
    FP_CUDA(cudaGetLastError());
  }
  return FP_OK;
}

// Load the exchange kernels now (lazy module loading would load them at their first launch,
// and a load synchronises the device: in a single-process group a rank could then wait, before
// launching its barrier kernel, for another rank's barrier kernel that waits for it).
void preload_exchange_kernels() {
  cudaFuncAttributes fa;
  const void* ks[] = {(const void*)k_peer_barrier, (const void*)k_peer_sum<float>, (const void*)k_peer_sum<double>,
                      (const void*)k_copy_bytes, (const void*)k_nvls_barrier, (const void*)k_nvls_sum<float>,
                      (const void*)k_nvls_sum<double>};
  for (const void* k : ks)
    if (cudaFuncGetAttributes(&fa, k) != cudaSuccess) cudaGetLastError();
}

fp_status alloc_sym(fp_comm* c, size_t cap) {
  preload_exchange_kernels();
  const size_t bytes = 2 * cap + kMaxPeers * sizeof(uint64_t);
  FP_CUDA(cudaSetDevice(c->device));
  FP_CUDA(cudaMalloc((void**)&c->sym, bytes));
  FP_CUDA(cudaMemset(c->sym, 0, bytes));
  FP_CUDA(cudaMalloc((void**)&c->timeout_flag, sizeof(unsigned)));
  FP_CUDA(cudaMemset(c->timeout_flag, 0, sizeof(unsigned)));
  c->cap = cap;
  c->peer[c->rank] = c->sym;
  return FP_OK;
}

// ---- CUDA driver entry points for NVLS (no link-time dependency on libcuda)
template <typename F>
bool drv(const char* name, F*& f) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess) {
    cudaGetLastError();
    return false;
  }
  f = reinterpret_cast<F*>(p);
  return true;
}

#define FP_CU(call)                                                              \
  do {                                                                           \
    CUresult r_ = (call);                                                        \
    if (r_ != CUDA_SUCCESS) {                                                    \
      fp::set_error("NVLS: %s failed (CUresult %d)", #call, (int)r_);            \
      return FP_ERR_CUDA;                                                        \
    }                                                                            \
  } while (0)

struct Drv {
  decltype(&cuMulticastCreate) mcCreate = nullptr;
  decltype(&cuMulticastAddDevice) mcAdd = nullptr;
  decltype(&cuMulticastBindMem) mcBind = nullptr;
  decltype(&cuMulticastUnbind) mcUnbind = nullptr;
  decltype(&cuMulticastGetGranularity) mcGran = nullptr;
  decltype(&cuMemCreate) memCreate = nullptr;
  decltype(&cuMemRelease) memRelease = nullptr;
  decltype(&cuMemAddressReserve) vaReserve = nullptr;
  decltype(&cuMemAddressFree) vaFree = nullptr;
  decltype(&cuMemMap) memMap = nullptr;
  decltype(&cuMemUnmap) memUnmap = nullptr;
  decltype(&cuMemSetAccess) memSetAccess = nullptr;
  decltype(&cuMemGetAllocationGranularity) memGran = nullptr;
  decltype(&cuMemExportToShareableHandle) memExport = nullptr;
  decltype(&cuMemImportFromShareableHandle) memImport = nullptr;
  bool ok = false;
};
const Drv& driver() {
  static Drv d = [] {
    Drv x;
    x.ok = drv("cuMulticastCreate", x.mcCreate) && drv("cuMulticastAddDevice", x.mcAdd) &&
           drv("cuMulticastBindMem", x.mcBind) && drv("cuMulticastUnbind", x.mcUnbind) &&
           drv("cuMulticastGetGranularity", x.mcGran) && drv("cuMemCreate", x.memCreate) &&
           drv("cuMemRelease", x.memRelease) && drv("cuMemAddressReserve", x.vaReserve) &&
           drv("cuMemAddressFree", x.vaFree) && drv("cuMemMap", x.memMap) && drv("cuMemUnmap", x.memUnmap) &&
           drv("cuMemSetAccess", x.memSetAccess) && drv("cuMemGetAllocationGranularity", x.memGran) &&
           drv("cuMemExportToShareableHandle", x.memExport) &&
           drv("cuMemImportFromShareableHandle", x.memImport);
    return x;
  }();
  return d;
}

fp_status nccl_barrier(fp_comm* c, cudaStream_t s) {
  float* d = nullptr;
  FP_CUDA(cudaMalloc((void**)&d, sizeof(float)));
  ncclResult_t r = ncclAllReduce(d, d, 1, ncclFloat32, ncclSum, c->nccl, s);
  cudaStreamSynchronize(s);
  cudaFree(d);
  if (r != ncclSuccess) return fp::nccl_fail(r, "ncclAllReduce(barrier)");
  return FP_OK;
}

fp_status nvls_setup(fp_comm* c, size_t cap, cudaStream_t s) {
  const Drv& D = driver();
  FP_REQUIRE(D.ok, FP_ERR_UNSUPPORTED, "NVLS: CUDA driver multicast entry points unavailable");
  int mcsup = 0;
  cudaDeviceGetAttribute(&mcsup, (cudaDeviceAttr)CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, c->device);
  FP_REQUIRE(mcsup, FP_ERR_UNSUPPORTED, "NVLS: device %d does not support multicast", c->device);
  CUmulticastObjectProp mp{};
  mp.numDevices = (unsigned)c->size;
  mp.handleTypes = CU_MEM_HANDLE_TYPE_FABRIC;
  const size_t want = 2 * cap + 256;
  mp.size = want;
  size_t gmc = 0, gph = 0;
  FP_CU(D.mcGran(&gmc, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED));
  CUmemAllocationProp pp{};
  pp.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  pp.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  pp.location.id = c->device;
  FP_CU(D.memGran(&gph, &pp, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED));
  const size_t g = gmc > gph ? gmc : gph;
  const size_t size = (want + g - 1) / g * g;
  mp.size = size;
  // the multicast object: created on rank 0, imported elsewhere through a fabric handle
  unsigned char* dh = nullptr;
  if (c->size > 1) FP_CUDA(cudaMalloc((void**)&dh, sizeof(CUmemFabricHandle)));
  if (c->rank == 0) {
    // fabric handles (what the other ranks import); a POSIX-fd type for a single rank if the
    // fabric type is refused
    CUresult cr = D.mcCreate(&c->mc_handle, &mp);
    if (cr != CUDA_SUCCESS && c->size == 1) {
      mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
      cr = D.mcCreate(&c->mc_handle, &mp);
    }
    FP_CU(cr);
    if (c->size > 1) {
      CUmemFabricHandle fh;
      FP_CU(D.memExport(&fh, c->mc_handle, CU_MEM_HANDLE_TYPE_FABRIC, 0));
      FP_CUDA(cudaMemcpy(dh, &fh, sizeof(fh), cudaMemcpyHostToDevice));
    }
  }
  if (c->size > 1) {
    ncclResult_t r = ncclBroadcast(dh, dh, sizeof(CUmemFabricHandle), ncclUint8, 0, c->nccl, s);
    if (r != ncclSuccess) return fp::nccl_fail(r, "ncclBroadcast(fabric handle)");
    CUmemFabricHandle fh;
    FP_CUDA(cudaMemcpyAsync(&fh, dh, sizeof(fh), cudaMemcpyDeviceToHost, s));
    FP_CUDA(cudaStreamSynchronize(s));
    cudaFree(dh);
    if (c->rank != 0) FP_CU(D.memImport(&c->mc_handle, &fh, CU_MEM_HANDLE_TYPE_FABRIC));
  }
  CUdevice dev = (CUdevice)c->device;
  FP_CU(D.mcAdd(c->mc_handle, dev));
  if (c->size > 1) {
    fp_status st = nccl_barrier(c, s);  // every device added before any binds
    if (st != FP_OK) return st;
  }
  FP_CU(D.memCreate(&c->ph_handle, size, &pp, 0));
  FP_CU(D.mcBind(c->mc_handle, 0, c->ph_handle, 0, size, 0));
  CUdeviceptr uva = 0, mva = 0;
  FP_CU(D.vaReserve(&uva, size, g, 0, 0));
  FP_CU(D.memMap(uva, size, 0, c->ph_handle, 0));
  FP_CU(D.vaReserve(&mva, size, g, 0, 0));
  FP_CU(D.memMap(mva, size, 0, c->mc_handle, 0));
  CUmemAccessDesc ad{};
  ad.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ad.location.id = c->device;
  ad.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  FP_CU(D.memSetAccess(uva, size, &ad, 1));
  FP_CU(D.memSetAccess(mva, size, &ad, 1));
  c->uc = (unsigned char*)uva;
  c->mc = (unsigned char*)mva;
  c->mc_size = size;
  c->cap = cap;
  c->nvls = true;
  FP_CUDA(cudaMemset(c->uc, 0, size));
  FP_CUDA(cudaDeviceSynchronize());
  if (c->size > 1) return nccl_barrier(c, s);  // every copy zeroed before any red lands
  return FP_OK;
}

void nvls_release(fp_comm* c) {
  const Drv& D = driver();
  if (!D.ok) return;
  cudaDeviceSynchronize();
  if (c->mc) D.memUnmap((CUdeviceptr)c->mc, c->mc_size), D.vaFree((CUdeviceptr)c->mc, c->mc_size);
  if (c->uc) D.memUnmap((CUdeviceptr)c->uc, c->mc_size), D.vaFree((CUdeviceptr)c->uc, c->mc_size);
  if (c->mc_handle && c->ph_handle) D.mcUnbind(c->mc_handle, (CUdevice)c->device, 0, c->mc_size);
  if (c->ph_handle) D.memRelease(c->ph_handle);
  if (c->mc_handle) D.memRelease(c->mc_handle);
  c->mc = c->uc = nullptr;
  c->mc_handle = c->ph_handle = 0;
  c->nvls = false;
}

}  // namespace

#define FP_NCCL(call)                                      \
  do {                                                     \
    ncclResult_t r_ = (call);                              \
    if (r_ != ncclSuccess) return fp::nccl_fail(r_, #call); \
  } while (0)

extern "C" {

fp_status fp_comm_get_unique_id(unsigned char id[128]) {
  FP_REQUIRE(id, FP_ERR_INVALID_ARG, "fp_comm_get_unique_id: id is NULL");
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
  ncclUniqueId u;
  FP_NCCL(ncclGetUniqueId(&u));
  memcpy(id, &u, 128);
  return FP_OK;
}

fp_status fp_comm_init(fp_comm** comm, int nranks, int rank, const unsigned char id[128], int device) {
  FP_REQUIRE(comm && id && nranks >= 1 && rank >= 0 && rank < nranks, FP_ERR_INVALID_ARG,
             "fp_comm_init: bad arguments (nranks=%d rank=%d)", nranks, rank);
  FP_CUDA(cudaSetDevice(device));
  ncclUniqueId u;
  memcpy(&u, id, 128);
  fp_comm* c = new fp_comm();
  c->rank = rank;
  c->size = nranks;
  c->device = device;
  ncclResult_t r = ncclCommInitRank(&c->nccl, nranks, u, rank);
  if (r != ncclSuccess) {
    delete c;
    return fp::nccl_fail(r, "ncclCommInitRank");
  }
  *comm = c;
  return FP_OK;
}

fp_status fp_comm_destroy(fp_comm* comm) {
  if (!comm) return FP_OK;
  cudaSetDevice(comm->device);
  cudaDeviceSynchronize();
  for (int k = 0; k < kMaxPeers; ++k)
    if (comm->ipc_mapped[k]) cudaIpcCloseMemHandle(comm->peer[k]);
  if (comm->sym) cudaFree(comm->sym);
  if (comm->timeout_flag) cudaFree(comm->timeout_flag);
  if (comm->nvls) nvls_release(comm);
  ncclResult_t r = comm->nccl ? ncclCommDestroy(comm->nccl) : ncclSuccess;
  delete comm;
  if (r != ncclSuccess) return fp::nccl_fail(r, "ncclCommDestroy");
  return FP_OK;
}

int fp_comm_rank(const fp_comm* comm) { return comm ? comm->rank : -1; }
int fp_comm_size(const fp_comm* comm) { return comm ? comm->size : -1; }

fp_status fp_allreduce(fp_comm* comm, void* buf, int64_t n, fp_dtype dtype, fp_stream stream) {
  FP_REQUIRE(comm && fp::valid_dtype(dtype) && n >= 0 && (n == 0 || buf), FP_ERR_INVALID_ARG,
             "fp_allreduce: bad arguments");
  // no short cut for one rank: the collective runs (a copy in place) so that every *_dist call
  // exercises the same NCCL path at any world size
  if (n == 0) return FP_OK;
  if (comm->mode == FP_COMM_PEER || comm->mode == FP_COMM_NVLS) {
    cudaStream_t s = (cudaStream_t)stream;
    void* D = nullptr;
    const size_t bytes = (size_t)n * fp::dtype_size(dtype);
    fp_status st = peer_begin(comm, bytes, s, &D);
    if (st != FP_OK) return st;
    // a kernel, not cudaMemcpyAsync: a same-device copy may serialise against other streams
    const int grid = (int)std::min<int64_t>(((int64_t)bytes / 16 + 255) / 256 + 1, 1024);
    k_copy_bytes<<<grid, 256, 0, s>>>((unsigned char*)D, (const unsigned char*)buf, bytes);
    FP_CUDA(cudaGetLastError());
    return peer_finish(comm, n, dtype, nullptr, 0.0, buf, s);
  }
  FP_REQUIRE(comm->nccl, FP_ERR_INVALID_ARG, "fp_allreduce: communicator has no NCCL backend (local group)");
  FP_NCCL(ncclAllReduce(buf, buf, (size_t)n, dtype == FP_F64 ? ncclFloat64 : ncclFloat32, ncclSum, comm->nccl,
                        (cudaStream_t)stream));
  return FP_OK;
}

// ----------------------------------------------------------------------- shard bounds (host)
fp_status fp_shard_rows_dense(int64_t m, int nranks, int64_t* bounds) {
  FP_REQUIRE(m >= 0 && nranks >= 1 && bounds, FP_ERR_INVALID_ARG, "fp_shard_rows_dense: bad arguments");
  for (int k = 0; k <= nranks; ++k) bounds[k] = (m * k) / nranks;
  return FP_OK;
}

fp_status fp_shard_rows_csr(int64_t m, const int64_t* rowptr, int nranks, int64_t* bounds) {
  FP_REQUIRE(m >= 0 && nranks >= 1 && bounds && rowptr, FP_ERR_INVALID_ARG, "fp_shard_rows_csr: bad arguments");
  const int64_t base = rowptr[0], nnz = rowptr[m] - rowptr[0];
  FP_REQUIRE(nnz >= 0, FP_ERR_INVALID_CSR, "fp_shard_rows_csr: rowptr[m] < rowptr[0]");
  bounds[0] = 0;
  bounds[nranks] = m;
  for (int k = 1; k < nranks; ++k) {
    // first row r with rowptr[r] - base >= k*nnz/P (binary search; rows are never split)
    const int64_t t = (int64_t)(((long double)nnz * k) / nranks);
    int64_t lo = 0, hi = m;
    while (lo < hi) {
      int64_t mid = lo + (hi - lo) / 2;
      if (rowptr[mid] - base < t) lo = mid + 1;
      else hi = mid;
    }
    bounds[k] = lo < bounds[k - 1] ? bounds[k - 1] : lo;
  }
  return FP_OK;
}

// --------------------------------------------------------------------- peer mode setup
// Collective: every rank allocates its symmetric buffer, exports a CUDA IPC handle, the
// handles are all-gathered through NCCL, and every rank maps every peer's buffer.
fp_status fp_comm_enable_peer(fp_comm* comm, int64_t max_bytes, fp_stream stream) {
  FP_REQUIRE(comm && max_bytes > 0, FP_ERR_INVALID_ARG, "fp_comm_enable_peer: bad arguments");
  FP_REQUIRE(comm->size <= kMaxPeers, FP_ERR_UNSUPPORTED, "fp_comm_enable_peer: at most %d ranks", kMaxPeers);
  if (comm->sym) {
    FP_REQUIRE((size_t)max_bytes <= comm->cap, FP_ERR_INVALID_ARG, "fp_comm_enable_peer: already enabled smaller");
    comm->mode = FP_COMM_PEER;
    return FP_OK;
  }
  FP_REQUIRE(comm->nccl, FP_ERR_INVALID_ARG, "fp_comm_enable_peer: needs an NCCL communicator");
  const size_t cap = ((size_t)max_bytes + 255) / 256 * 256;
  fp_status st = alloc_sym(comm, cap);
  if (st != FP_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  cudaIpcMemHandle_t mine;
  FP_CUDA(cudaIpcGetMemHandle(&mine, comm->sym));
  unsigned char* dh = nullptr;
  FP_CUDA(cudaMalloc((void**)&dh, (size_t)comm->size * sizeof(cudaIpcMemHandle_t)));
  FP_CUDA(cudaMemcpyAsync(dh + (size_t)comm->rank * sizeof(mine), &mine, sizeof(mine), cudaMemcpyHostToDevice, s));
  ncclResult_t r = ncclAllGather(dh + (size_t)comm->rank * sizeof(mine), dh, sizeof(mine), ncclUint8, comm->nccl, s);
  if (r != ncclSuccess) {
    cudaFree(dh);
    return fp::nccl_fail(r, "ncclAllGather(ipc handles)");
  }
  std::vector<cudaIpcMemHandle_t> all(comm->size);
  FP_CUDA(cudaMemcpyAsync(all.data(), dh, (size_t)comm->size * sizeof(mine), cudaMemcpyDeviceToHost, s));
  FP_CUDA(cudaStreamSynchronize(s));
  cudaFree(dh);
  for (int k = 0; k < comm->size; ++k) {
    if (k == comm->rank) continue;
    void* p = nullptr;
    FP_CUDA(cudaIpcOpenMemHandle(&p, all[k], cudaIpcMemLazyEnablePeerAccess));
    comm->peer[k] = (unsigned char*)p;
    comm->ipc_mapped[k] = true;
  }
  comm->mode = FP_COMM_PEER;
  return FP_OK;
}

// NVLS: one multicast object (CUDA driver API, resolved at run time) over every rank's buffer.
// Rank 0 creates it and exports a fabric handle, broadcast through NCCL; every rank adds its
// device, binds a physical allocation and maps both the unicast and the multicast range.
fp_status fp_comm_enable_nvls(fp_comm* comm, int64_t max_bytes, fp_stream stream) {
  FP_REQUIRE(comm && max_bytes > 0, FP_ERR_INVALID_ARG, "fp_comm_enable_nvls: bad arguments");
  if (comm->nvls) {
    FP_REQUIRE((size_t)max_bytes <= comm->cap, FP_ERR_INVALID_ARG, "fp_comm_enable_nvls: already enabled smaller");
    comm->mode = FP_COMM_NVLS;
    return FP_OK;
  }
  FP_REQUIRE(!comm->sym, FP_ERR_UNSUPPORTED, "fp_comm_enable_nvls: peer mode already enabled on this communicator");
  FP_REQUIRE(comm->nccl, FP_ERR_INVALID_ARG, "fp_comm_enable_nvls: needs an NCCL communicator");
  FP_CUDA(cudaSetDevice(comm->device));
  preload_exchange_kernels();
  cudaStream_t s = (cudaStream_t)stream;
  fp_status st = nvls_setup(comm, ((size_t)max_bytes + 255) / 256 * 256, s);
  if (st != FP_OK) {
    nvls_release(comm);
    return st;
  }
  FP_CUDA(cudaMalloc((void**)&comm->timeout_flag, sizeof(unsigned)));
  FP_CUDA(cudaMemset(comm->timeout_flag, 0, sizeof(unsigned)));
  comm->mode = FP_COMM_NVLS;
  return FP_OK;
}

fp_status fp_comm_set_mode(fp_comm* comm, int mode) {
  FP_REQUIRE(comm && (mode == FP_COMM_NCCL || mode == FP_COMM_PEER || mode == FP_COMM_NVLS), FP_ERR_INVALID_ARG,
             "fp_comm_set_mode: bad arguments");
  FP_REQUIRE(mode != FP_COMM_PEER || comm->sym, FP_ERR_INVALID_ARG, "fp_comm_set_mode: peer mode not enabled");
  FP_REQUIRE(mode != FP_COMM_NVLS || comm->nvls, FP_ERR_INVALID_ARG, "fp_comm_set_mode: NVLS not enabled");
  FP_REQUIRE(mode != FP_COMM_NCCL || comm->nccl, FP_ERR_INVALID_ARG, "fp_comm_set_mode: no NCCL backend");
  comm->mode = mode;
  return FP_OK;
}

int fp_comm_mode(const fp_comm* comm) { return comm ? comm->mode : -1; }

// Single-process group of `nranks` communicators on ONE device whose symmetric buffers are
// plain device allocations (no IPC, no NCCL): the peer exchange as across GPUs (same
// symmetric-buffer layout, epoch flags, rank-ordered sum), for tests and for replicas sharing
// a GPU.  Ranks must be driven concurrently from one host thread each: a rank's call returns
// after every rank reached its exchange (host rendezvous).  No device-side wait of one rank's
// kernel on another's launch (peer_finish).
fp_status fp_comm_init_local_group(int nranks, int device, int64_t max_bytes, fp_comm** comms) {
  FP_REQUIRE(comms && nranks >= 1 && nranks <= kMaxPeers && max_bytes > 0, FP_ERR_INVALID_ARG,
             "fp_comm_init_local_group: bad arguments (1 <= nranks <= %d)", kMaxPeers);
  const size_t cap = ((size_t)max_bytes + 255) / 256 * 256;
  for (int r = 0; r < nranks; ++r) {
    comms[r] = new fp_comm();
    comms[r]->rank = r;
    comms[r]->size = nranks;
    comms[r]->device = device;
    comms[r]->mode = FP_COMM_PEER;
    fp_status st = alloc_sym(comms[r], cap);
    if (st != FP_OK) {
      for (int k = 0; k <= r; ++k) fp_comm_destroy(comms[k]);
      return st;
    }
  }
  auto sync = std::make_shared<LocalSync>();
  sync->P = nranks;
  for (int r = 0; r < nranks; ++r) {
    for (int k = 0; k < nranks; ++k) comms[r]->peer[k] = comms[k]->sym;
    comms[r]->lsync = sync;
  }
  return FP_OK;
}

// 1 if a peer barrier of this communicator ever timed out (its results are then invalid).
int fp_comm_timed_out(const fp_comm* comm) {
  if (!comm || !comm->timeout_flag) return 0;
  unsigned h = 0;
  if (cudaMemcpy(&h, comm->timeout_flag, sizeof(h), cudaMemcpyDeviceToHost) != cudaSuccess) return -1;
  return h ? 1 : 0;
}

// --------------------------------------------------------------------- distributed pattern
fp_status fp_dense_dist(int64_t m_local, int64_t n, const void* X, int64_t ld, const void* y, const void* v,
                        const void* z, double alpha, double beta, void* w, fp_dtype dtype, fp_comm* comm,
                        fp_stream stream) {
  FP_REQUIRE(comm, FP_ERR_INVALID_ARG, "fp_dense_dist: comm is NULL");
  fp::PatternArgs a = fp::dense_args(m_local, n, X, ld, y, v, z, alpha, beta, w, dtype);
  if (comm->mode != FP_COMM_NCCL) return dist_peer(a, false, comm, (cudaStream_t)stream);
  a.add_beta_z = comm->rank == 0;
  fp_status st = fp::run_dense(a, nullptr, (cudaStream_t)stream);
  if (st != FP_OK) return st;
  return fp_allreduce(comm, w, n, dtype, stream);
}

fp_status fp_csr_dist(int64_t m_local, int64_t n, int64_t nnz_local, const int64_t* rowptr, const int32_t* colidx,
                      const void* val, const void* y, const void* v, const void* z, double alpha, double beta,
                      void* w, fp_dtype dtype, fp_comm* comm, fp_stream stream) {
  FP_REQUIRE(comm, FP_ERR_INVALID_ARG, "fp_csr_dist: comm is NULL");
  fp::PatternArgs a = fp::csr_args(m_local, n, nnz_local, rowptr, colidx, val, y, v, z, alpha, beta, w, dtype);
  if (comm->mode != FP_COMM_NCCL) return dist_peer(a, true, comm, (cudaStream_t)stream);
  a.add_beta_z = comm->rank == 0;
  fp_status st = fp::run_csr(a, nullptr, (cudaStream_t)stream);
  if (st != FP_OK) return st;
  return fp_allreduce(comm, w, n, dtype, stream);
}

fp_status fp_csr_plan_dist(const fp_csr_plan* plan, fp_comm* comm, const void* val, const void* y, const void* v,
                           const void* z, double alpha, double beta, void* w, fp_stream stream) {
  FP_REQUIRE(plan && comm, FP_ERR_INVALID_ARG, "fp_csr_plan_dist: plan or comm is NULL");
  int64_t m = 0, n = 0, nnz = 0;
  const int64_t* rowptr = nullptr;
  const int32_t* colidx = nullptr;
  fp_dtype dt = FP_F32;
  fp::plan_shape(plan, &m, &n, &nnz, &rowptr, &colidx, &dt);
  fp::PatternArgs a = fp::csr_args(m, n, nnz, rowptr, colidx, val, y, v, z, alpha, beta, w, dt);
  if (comm->mode != FP_COMM_NCCL) return dist_peer_plan(a, plan, comm, (cudaStream_t)stream);
  a.add_beta_z = comm->rank == 0;
  fp_status st = fp::plan_run(plan, a, (cudaStream_t)stream);
  if (st != FP_OK) return st;
  return fp_allreduce(comm, w, n, dt, stream);
}

}  // extern "C"
