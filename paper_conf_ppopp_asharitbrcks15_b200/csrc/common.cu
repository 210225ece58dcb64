// common.cu -- error state, device info cache, per-stream workspaces.
#include <stdarg.h>
#include <stdio.h>

#include <map>
#include <mutex>
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
namespace {
std::mutex g_ws_mu;
std::map<std::pair<int, cudaStream_t>, Workspace*> g_ws;
}  // namespace

Workspace* workspace(cudaStream_t s, size_t acc_elems, size_t scratch_bytes) {
  int dev = current_device();
  std::lock_guard<std::mutex> lk(g_ws_mu);
  Workspace*& ws = g_ws[{dev, s}];
  if (!ws) ws = new Workspace();
  if (!ws->counters) {
    if (cudaMalloc(&ws->counters, 4 * sizeof(unsigned long long)) != cudaSuccess) {
      set_error("workspace: cudaMalloc(counters) failed");
      return nullptr;
    }
    cudaMemsetAsync(ws->counters, 0, 4 * sizeof(unsigned long long), s);
  }
  if (acc_elems > ws->acc_cap) {
    size_t cap = acc_elems < 4096 ? 4096 : acc_elems;
    double* p = nullptr;
    if (cudaMalloc(&p, cap * sizeof(double)) != cudaSuccess) {
      set_error("workspace: cudaMalloc(acc, %zu doubles) failed", cap);
      return nullptr;
    }
    cudaMemsetAsync(p, 0, cap * sizeof(double), s);
    if (ws->acc) {
      cudaStreamSynchronize(s);   // previous launches on s may still use the old buffer
      cudaFree(ws->acc);
    }
    ws->acc = p;
    ws->acc_cap = cap;
  }
  if (scratch_bytes > ws->scratch_cap) {
    void* p = nullptr;
    if (cudaMalloc(&p, scratch_bytes) != cudaSuccess) {
      set_error("workspace: cudaMalloc(scratch, %zu B) failed", scratch_bytes);
      return nullptr;
    }
    if (ws->scratch) {
      cudaStreamSynchronize(s);
      cudaFree(ws->scratch);
    }
    ws->scratch = p;
    ws->scratch_cap = scratch_bytes;
  }
  return ws;
}

void release_all_workspaces() {
  std::lock_guard<std::mutex> lk(g_ws_mu);
  int prev = current_device();
  for (auto& kv : g_ws) {
    cudaSetDevice(kv.first.first);
    cudaDeviceSynchronize();
    Workspace* ws = kv.second;
    if (ws) {
      cudaFree(ws->acc);
      cudaFree(ws->counters);
      cudaFree(ws->scratch);
      delete ws;
    }
  }
  g_ws.clear();
  cudaSetDevice(prev);
}

}  // namespace fp

extern "C" const char* fp_last_error(void) { return fp::last_error_text(); }
