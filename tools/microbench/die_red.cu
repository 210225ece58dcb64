// die_red.cu -- do die-local copies of w help random fp32 reds?  (C4's bound: 2e9 random
// red.global.add.f32 into a 400 KB w, half of them crossing the die-to-die link.)
// 1. classify 4 KB pages of a 16 MB pool by home die: one CTA per SM times a returning
//    atom.add on every page (atomics always go to the home L2); SMs split into two groups by
//    agreement of their near/far pattern with SM 0's.
// 2. time 2^31 random reds into (a) one ordinary 400 KB array, (b) one copy per SM group built
//    from pages homed on that group's die (page table in shared memory).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }

__global__ void k_cal(unsigned* pool, int npages, unsigned* lat, unsigned* sm_of) {
  __shared__ volatile unsigned s_dep[2];
  if (threadIdx.x) return;
  s_dep[0] = 0;
  sm_of[blockIdx.x] = smid();
  for (int p = 0; p < npages; ++p) {
    unsigned* a = pool + (size_t)p * 1024;
    const long long t0 = clock64();
    const unsigned v = atomicAdd(a, 1u);
    const unsigned d = s_dep[v >> 31];  // volatile read that needs the atomic's result
    const long long t1 = clock64();
    lat[(size_t)blockIdx.x * npages + p] = (unsigned)(t1 - t0) + d;
  }
}

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}

template <int MODE>
__global__ void k_red(float* w, const float* const* tab, int npg, const uint64_t* mask, int n, int iters) {
  __shared__ float* s_tab[256];
  const unsigned g = (unsigned)((mask[smid() >> 6] >> (smid() & 63)) & 1ull);
  if (MODE == 1) {
    for (int i = threadIdx.x; i < npg; i += blockDim.x) s_tab[i] = (float*)tab[g * npg + i];
    __syncthreads();
  }
  uint32_t st = (blockIdx.x * blockDim.x + threadIdx.x) * 2654435761u;
  for (int i = 0; i < iters; ++i) {
    st = hash32(st + i);
    const int c = (int)(st % (uint32_t)n);
    if (MODE == 0) atomicAdd(w + c, 1.0f);
    else atomicAdd(s_tab[c >> 10] + (c & 1023), 1.0f);
  }
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int npages = 4096;
  unsigned *pool, *lat, *smo;
  cudaMalloc(&pool, (size_t)npages * 4096);
  cudaMemset(pool, 0, (size_t)npages * 4096);
  cudaMalloc(&lat, (size_t)sms * npages * 4);
  cudaMalloc(&smo, sms * 4);
  k_cal<<<sms, 32>>>(pool, npages, lat, smo);
  cudaDeviceSynchronize();
  std::vector<unsigned> L((size_t)sms * npages), S(sms);
  cudaMemcpy(L.data(), lat, L.size() * 4, cudaMemcpyDeviceToHost);
  cudaMemcpy(S.data(), smo, sms * 4, cudaMemcpyDeviceToHost);
  { FILE* f = fopen("gpurun_out/die_atom.bin", "wb"); if (f) { fwrite(S.data(), 4, sms, f); fwrite(L.data(), 4, L.size(), f); fclose(f); } }
  // near/far per (sm, page): below the page's median
  std::vector<char> nearv((size_t)sms * npages);
  for (int p = 0; p < npages; ++p) {
    std::vector<unsigned> col(sms);
    for (int b = 0; b < sms; ++b) col[b] = L[(size_t)b * npages + p];
    std::vector<unsigned> srt = col;
    std::nth_element(srt.begin(), srt.begin() + sms / 2, srt.end());
    const unsigned med = srt[sms / 2];
    for (int b = 0; b < sms; ++b) nearv[(size_t)b * npages + p] = col[b] + 100 < med + 100 && col[b] < med;
  }
  std::vector<int> grp(sms);
  for (int b = 0; b < sms; ++b) {
    int agree = 0;
    for (int p = 0; p < npages; ++p) agree += nearv[(size_t)b * npages + p] == nearv[p];
    grp[b] = agree > npages / 2 ? 0 : 1;
  }
  // page home: group whose mean latency is lower by > 150 cycles
  std::vector<int> home(npages, -1);
  int cnt[2] = {0, 0};
  for (int p = 0; p < npages; ++p) {
    double m[2] = {0, 0}; int k[2] = {0, 0};
    for (int b = 0; b < sms; ++b) { m[grp[b]] += L[(size_t)b * npages + p]; k[grp[b]]++; }
    m[0] /= k[0]; m[1] /= k[1];
    if (m[0] + 150 < m[1]) home[p] = 0; else if (m[1] + 150 < m[0]) home[p] = 1;
    if (home[p] >= 0) cnt[home[p]]++;
  }
  int g0 = 0; for (int b = 0; b < sms; ++b) g0 += grp[b] == 0;
  printf("SM groups: %d / %d; pages homed: %d / %d / unknown %d\n", g0, sms - g0, cnt[0], cnt[1], npages - cnt[0] - cnt[1]);
  uint64_t hmask[3] = {0, 0, 0};
  for (int b = 0; b < sms; ++b) if (grp[b]) hmask[S[b] >> 6] |= 1ull << (S[b] & 63);
  const int n = 100000, npg = (n + 1023) / 1024;
  std::vector<const float*> htab(2 * npg);
  int used[2] = {0, 0};
  for (int p = 0; p < npages && (used[0] < npg || used[1] < npg); ++p) {
    const int h = home[p];
    if (h >= 0 && used[h] < npg) htab[h * npg + used[h]++] = (const float*)((char*)pool + (size_t)p * 4096);
  }
  printf("pages used %d %d of %d\n", used[0], used[1], npg);
  const float** dtab; uint64_t* dmask; float* w;
  cudaMalloc(&dtab, htab.size() * 8);
  cudaMemcpy(dtab, htab.data(), htab.size() * 8, cudaMemcpyHostToDevice);
  cudaMalloc(&dmask, 24);
  cudaMemcpy(dmask, hmask, 24, cudaMemcpyHostToDevice);
  cudaMalloc(&w, n * 4);
  cudaMemset(w, 0, n * 4);
  const int iters = 1 << 14, grid = sms * 4, bs = 256;
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  for (int mode = 0; mode < 2; ++mode) {
    for (int r = 0; r < 3; ++r) {
      cudaEventRecord(a);
      if (mode == 0) k_red<0><<<grid, bs>>>(w, dtab, npg, dmask, n, iters);
      else k_red<1><<<grid, bs>>>(w, dtab, npg, dmask, n, iters);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b);
      const double reds = (double)grid * bs * iters;
      printf("mode %d (%s): %.3f ms  %.1f Greds/s\n", mode, mode ? "die-local copies" : "one array", ms, reds / ms / 1e6);
    }
  }
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
