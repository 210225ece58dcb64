// die_probe.cu -- which die's L2 / HBM homes each chunk of a buffer, seen from each SM.
// One CTA (one thread) per SM: for every chunk of G bytes of a 64 MB buffer, warm the line
// into L2 (ld.global.cg), then time one dependent ld.global.cg (L2 hit; a far-die hit crosses
// the die-to-die link).  Prints, per chunk, the mean latency seen from SMs whose id is in the
// lower / upper half, and a latency-vs-SM summary.  nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned smid() {
  unsigned r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

__global__ void k_probe(const int* __restrict__ buf, size_t G, int nchunks, unsigned* lat, unsigned* sm_of_cta) {
  if (threadIdx.x != 0) return;
  const unsigned s = smid();
  sm_of_cta[blockIdx.x] = s;
  int sink = 0;
  for (int c = 0; c < nchunks; ++c) {
    const int* p = buf + (size_t)c * (G / 4);
    int v;
    asm volatile("ld.global.cg.s32 %0, [%1];" : "=r"(v) : "l"(p));  // bring into L2
    sink += v;
    const long long t0 = clock64();
    asm volatile("ld.global.cg.s32 %0, [%1];" : "=r"(v) : "l"(p + (sink & 0)));
    sink += v;
    const long long t1 = clock64() + (sink & 0);
    lat[(size_t)blockIdx.x * nchunks + c] = (unsigned)(t1 - t0);
  }
  if (sink == 12345) lat[0] = 0;
}

int main(int argc, char** argv) {
  const size_t G = argc > 1 ? (size_t)atol(argv[1]) : 4096;
  const size_t bytes = 64ull << 20;
  const int nchunks = (int)(bytes / G) > 4096 ? 4096 : (int)(bytes / G);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int* buf;
  cudaMalloc(&buf, bytes);
  cudaMemset(buf, 0, bytes);
  unsigned *lat, *smo;
  cudaMalloc(&lat, (size_t)sms * nchunks * 4);
  cudaMalloc(&smo, sms * 4);
  k_probe<<<sms, 32>>>(buf, G, nchunks, lat, smo);
  cudaDeviceSynchronize();
  std::vector<unsigned> h((size_t)sms * nchunks), hs(sms);
  cudaMemcpy(h.data(), lat, h.size() * 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(hs.data(), smo, sms * 4, cudaMemcpyDeviceToHost);
  if (argc > 2) {  // raw dump for offline analysis: [sms] smid, then [sms][nchunks] latency
    FILE* f = fopen(argv[2], "wb");
    fwrite(hs.data(), 4, sms, f);
    fwrite(h.data(), 4, h.size(), f);
    fclose(f);
  }
  // per chunk: latency from each SM; classify SMs by correlation with chunk 0's pattern
  printf("G=%zu chunks=%d sms=%d err=%s\n", G, nchunks, sms, cudaGetErrorString(cudaGetLastError()));
  // latency of chunk c from SM (cta) b
  auto L = [&](int b, int c) { return (double)h[(size_t)b * nchunks + c]; };
  // SM grouping: for chunk 0..3 print latency per SM id order
  for (int c = 0; c < 4; ++c) {
    printf("chunk %d:", c);
    for (int b = 0; b < sms; ++b) printf(" %u:%.0f", hs[b], L(b, c));
    printf("\n");
  }
  // per chunk: mean latency from SMs with smid < sms/2 vs >= sms/2
  int near_lo = 0;
  printf("chunk pattern (L = lower-half SMs faster, U = upper faster, ? = no clear difference):\n");
  for (int c = 0; c < nchunks && c < 512; ++c) {
    double a = 0, b2 = 0; int na = 0, nb = 0;
    for (int b = 0; b < sms; ++b) {
      if ((int)hs[b] < sms / 2) { a += L(b, c); ++na; } else { b2 += L(b, c); ++nb; }
    }
    a /= na; b2 /= nb;
    const char ch = a + 60 < b2 ? 'L' : (b2 + 60 < a ? 'U' : '?');
    near_lo += ch == 'L';
    putchar(ch);
    if (c % 128 == 127) putchar('\n');
  }
  printf("\n");
  return 0;
}
