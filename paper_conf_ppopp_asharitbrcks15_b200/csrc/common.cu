// common.cu -- error state, device info cache, per-stream workspaces.
#include <stdarg.h>
#include <stdio.h>

#include <map>
#include <mutex>
#include <set>
#include <utility>
#include <vector>

#include "common.cuh"

namespace fp {

static thread_local char g_last_error[512] = "";

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_last_error, sizeof(g_last_error), fmt, ap);
  va_end(ap);
}

const char* last_error_text() { return g_last_error; }

fp_status cuda_fail(cudaError_t e, const char* what) {
  set_error("%s: %s (%s)", what, cudaGetErrorString(e), cudaGetErrorName(e));
  if (e == cudaErrorMemoryAllocation) return FP_ERR_NOMEM;
  return FP_ERR_CUDA;
}

int current_device() {
  int d = 0;
  cudaGetDevice(&d);
  return d;
}

const DeviceInfo& device_info(int ordinal) {
  static std::mutex mu;
  static std::map<int, DeviceInfo> cache;
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(ordinal);
  if (it != cache.end()) return it->second;
  DeviceInfo d{};
  d.ordinal = ordinal;
  cudaDeviceProp p{};
  if (cudaGetDeviceProperties(&p, ordinal) == cudaSuccess) {
    d.sm_count = p.multiProcessorCount;
    d.max_threads_per_sm = p.maxThreadsPerMultiProcessor;
    d.max_blocks_per_sm = p.maxBlocksPerMultiProcessor;
    d.regs_per_sm = p.regsPerMultiprocessor;
    d.smem_per_sm = p.sharedMemPerMultiprocessor;
    d.smem_optin_per_block = p.sharedMemPerBlockOptin;
    d.l2_bytes = p.l2CacheSize;
  } else {
    d.sm_count = 148; d.max_threads_per_sm = 2048; d.max_blocks_per_sm = 32; d.regs_per_sm = 65536;
    d.smem_per_sm = 228 * 1024; d.smem_optin_per_block = 227 * 1024; d.l2_bytes = 126u << 20;
  }
  return cache.emplace(ordinal, d).first->second;
}

// ---------------------------------------------------------------------------- workspace
// Keyed by (device, stream, capture id).  A call made while `s` is being captured into a CUDA
// graph gets a workspace of its own (capture id != 0) that is never regrown or freed while the
// library is loaded: the graph keeps the pointers baked into its kernel nodes, and two graphs
// -- or a graph and direct calls on the capture stream -- never share accumulators/tickets.
// Buffers replaced by a larger allocation are retired (freed only by release_all_workspaces),
// so a pointer handed to a launch another host thread has not enqueued yet stays valid.
namespace {
std::mutex g_ws_mu;
struct WsKey {
  int dev;
  cudaStream_t s;
  unsigned long long cap;
  bool operator<(const WsKey& o) const {
    if (dev != o.dev) return dev < o.dev;
    if (s != o.s) return s < o.s;
    return cap < o.cap;
  }
};
std::map<WsKey, Workspace*> g_ws;
std::vector<std::pair<int, void*>> g_retired;  // (device, pointer)
std::map<int, cudaStream_t> g_init_stream;     // per device: zero-fills outside any capture

unsigned long long capture_id(cudaStream_t s) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  unsigned long long id = 0;
  if (cudaStreamGetCaptureInfo(s, &st, &id) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return st == cudaStreamCaptureStatusActive ? id : 0;
}

// cudaMalloc + zero fill that is legal while another stream of this thread is capturing
// (relaxed capture mode for the allocation; the fill runs on a private stream and is waited
// for, so it is never recorded into the graph)
cudaError_t alloc_zeroed(void** p, size_t bytes, bool zero, int dev) {
  cudaStreamCaptureMode mode = cudaStreamCaptureModeRelaxed;
  cudaThreadExchangeStreamCaptureMode(&mode);
  cudaError_t e = cudaMalloc(p, bytes);
  if (e == cudaSuccess && zero) {
    cudaStream_t& is = g_init_stream[dev];
    if (!is) e = cudaStreamCreateWithFlags(&is, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaMemsetAsync(*p, 0, bytes, is);
    if (e == cudaSuccess) e = cudaStreamSynchronize(is);
  }
  cudaThreadExchangeStreamCaptureMode(&mode);
  return e;
}

Workspace* get_ws(cudaStream_t s, int dev) {
  Workspace*& ws = g_ws[WsKey{dev, s, capture_id(s)}];
  if (!ws) ws = new Workspace();
  return ws;
}

void retire(int dev, void* p) {
  if (p) g_retired.emplace_back(dev, p);
}
}  // namespace

Workspace* workspace(cudaStream_t s, size_t acc_elems, size_t scratch_bytes) {
  int dev = current_device();
  std::lock_guard<std::mutex> lk(g_ws_mu);
  Workspace* ws = get_ws(s, dev);
  if (!ws->counters) {
    if (alloc_zeroed((void**)&ws->counters, 4 * sizeof(unsigned long long), true, dev) != cudaSuccess) {
      ws->counters = nullptr;
      set_error("workspace: cudaMalloc(counters) failed");
      return nullptr;
    }
  }
  if (acc_elems > ws->acc_cap) {
    size_t cap = acc_elems < 4096 ? 4096 : acc_elems + acc_elems / 2;
    double* p = nullptr;
    if (alloc_zeroed((void**)&p, cap * sizeof(double), true, dev) != cudaSuccess) {
      set_error("workspace: cudaMalloc(acc, %zu doubles) failed", cap);
      return nullptr;
    }
    retire(dev, ws->acc);
    ws->acc = p;
    ws->acc_cap = cap;
  }
  if (scratch_bytes > ws->scratch_cap) {
    void* p = nullptr;
    const size_t cap = scratch_bytes + scratch_bytes / 2;
    if (alloc_zeroed(&p, cap, false, dev) != cudaSuccess) {
      set_error("workspace: cudaMalloc(scratch, %zu B) failed", cap);
      return nullptr;
    }
    retire(dev, ws->scratch);
    ws->scratch = p;
    ws->scratch_cap = cap;
  }
  return ws;
}

void* workspace_buffer(cudaStream_t s, int slot, size_t bytes, bool zero) {
  int dev = current_device();
  std::lock_guard<std::mutex> lk(g_ws_mu);
  Workspace* ws = get_ws(s, dev);
  if (slot < 0 || slot >= kWsSlots) return nullptr;
  if (bytes > ws->buf_cap[slot]) {
    void* p = nullptr;
    const size_t cap = bytes + bytes / 8;
    if (alloc_zeroed(&p, cap, zero, dev) != cudaSuccess) {
      cudaGetLastError();
      set_error("workspace: cudaMalloc(%zu B) failed", cap);
      return nullptr;
    }
    retire(dev, ws->buf[slot]);
    ws->buf[slot] = p;
    ws->buf_cap[slot] = cap;
  }
  return ws->buf[slot];
}

void release_all_workspaces() {
  std::lock_guard<std::mutex> lk(g_ws_mu);
  int prev = current_device();
  for (auto& kv : g_ws) {
    cudaSetDevice(kv.first.dev);
    cudaDeviceSynchronize();
    Workspace* ws = kv.second;
    if (ws) {
      cudaFree(ws->acc);
      cudaFree(ws->counters);
      cudaFree(ws->scratch);
      for (int i = 0; i < kWsSlots; ++i) cudaFree(ws->buf[i]);
      delete ws;
    }
  }
  g_ws.clear();
  for (auto& r : g_retired) {
    cudaSetDevice(r.first);
    cudaDeviceSynchronize();
    cudaFree(r.second);
  }
  g_retired.clear();
  cudaSetDevice(prev);
}

// The dynamic shared-memory cap of a kernel is raised once to the per-block maximum instead of
// per call to the call's size: a concurrent call with a smaller size can no longer lower it
// between another thread's set and launch.  (The cap does not change occupancy; the launch's
// actual size does.)
void set_max_dynamic_smem(const void* f) {
  static std::mutex mu;
  static std::set<const void*> done;
  std::lock_guard<std::mutex> lk(mu);
  if (done.count(f)) return;
  const int dev = current_device();
  cudaFuncAttributes fa{};
  if (cudaFuncGetAttributes(&fa, f) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  // static + dynamic shared memory of a block must stay within the opt-in limit
  const int cap = (int)device_info(dev).smem_optin_per_block - (int)fa.sharedSizeBytes;
  if (cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, cap) == cudaSuccess) done.insert(f);
  else cudaGetLastError();
}

}  // namespace fp

extern "C" const char* fp_last_error(void) { return fp::last_error_text(); }
