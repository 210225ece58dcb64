// EXPERIMENT (not built into libfusedpat; kept with its measurement, DESIGN.md §5 C4):
// the die-local copies of w wired into the CSR L2 path as they were measured on C4 --
// 26.5 ms with the copies vs 17.2 ms without (the per-nonzero page-table lookup costs more
// on the loaded L1/shared pipe than the die-local reds save).  To re-run it, move it back to
// csrc/ with the matching CsrKArgs fields (die_tab, die_npg, die_mask) and W_ADD addressing.
// die.cu -- die-local copies of w for the CSR L2 path (a10 of SURVEY 8 on a two-die B200).
//
// B200 is two dies; every 4 KB page of device memory is homed in one die's L2, and an atomic
// from an SM of the other die crosses the die-to-die link and costs both dies' L2 tag
// lookups.  C4's bound is that lookup rate: its 2e9 random reds into w land on a
// far page half the time.  tools/microbench/die_red.cu measured random fp32 reds into a
// 400 KB w at 152 Greds/s, and at 183 Greds/s when each die group reduces into its own copy of
// w built from pages homed on its die.
//
// Neither the page homing nor the SM-to-die assignment is exposed by CUDA, so both are
// measured once per workspace: one single-thread CTA per SM times a returning atomicAdd on
// every page of a 16 MB pool (an L2 atomic always executes in the home L2: ~300 vs ~700
// cycles).  SMs are grouped by agreement of their near/far pattern, pages by which group
// reaches them faster.  Correctness never depends on the classification: any CTA may reduce
// into any copy, the fold sums both copies into w.
#include <algorithm>
#include <vector>

#include "csr_kernels.cuh"

namespace fp {

namespace {

constexpr int kDiePoolPages = 4096;  // 16 MB
constexpr size_t kPage = 4096;

__global__ void k_die_calibrate(unsigned* pool, int npages, unsigned* lat, unsigned* sm_of) {
  __shared__ volatile unsigned s_dep[2];
  if (threadIdx.x != 0) return;
  s_dep[0] = 0;
  unsigned sm;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
  sm_of[blockIdx.x] = sm;
  for (int p = 0; p < npages; ++p) {
    unsigned* a = pool + (size_t)p * (kPage / 4);
    const long long t0 = clock64();
    const unsigned v = atomicAdd(a, 1u);
    const unsigned d = s_dep[v >> 31];  // needs the atomic's return: the clock waits for it
    const long long t1 = clock64();
    lat[(size_t)blockIdx.x * npages + p] = (unsigned)(t1 - t0) + d;
  }
}

// w[j] += copy0[j] + copy1[j]; both copies re-zeroed (page-table addressed)
template <typename T>
__global__ void k_die_fold(T* __restrict__ w, const unsigned long long* __restrict__ tab, int npg, int64_t n) {
  constexpr int PER = (int)(kPage / sizeof(T));
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    T* a = (T*)tab[j / PER] + (j % PER);
    T* b = (T*)tab[npg + j / PER] + (j % PER);
    w[j] += *a + *b;
    *a = T(0);
    *b = T(0);
  }
}

bool calibrate(Workspace* ws, cudaStream_t s) {
  const int sms = device_info(current_device()).sm_count;
  unsigned *lat = nullptr, *smo = nullptr;
  if (cudaMalloc(&ws->die_pool, (size_t)kDiePoolPages * kPage) != cudaSuccess ||
      cudaMalloc(&lat, (size_t)sms * kDiePoolPages * 4) != cudaSuccess || cudaMalloc(&smo, (size_t)sms * 4) != cudaSuccess) {
    cudaGetLastError();
    cudaFree(lat);
    cudaFree(smo);
    return false;
  }
  cudaMemsetAsync(ws->die_pool, 0, (size_t)kDiePoolPages * kPage, s);
  k_die_calibrate<<<sms, 32, 0, s>>>((unsigned*)ws->die_pool, kDiePoolPages, lat, smo);
  std::vector<unsigned> L((size_t)sms * kDiePoolPages), S(sms);
  cudaMemcpyAsync(L.data(), lat, L.size() * 4, cudaMemcpyDeviceToHost, s);
  cudaMemcpyAsync(S.data(), smo, (size_t)sms * 4, cudaMemcpyDeviceToHost, s);
  // the calibration atomics leave counts in the pool: zero it again (the copies' invariant)
  cudaMemsetAsync(ws->die_pool, 0, (size_t)kDiePoolPages * kPage, s);
  const bool ok = cudaStreamSynchronize(s) == cudaSuccess;
  cudaFree(lat);
  cudaFree(smo);
  if (!ok) {
    cudaGetLastError();
    return false;
  }
  // near/far per (CTA, page): below the page's median latency over all CTAs
  std::vector<char> nearv((size_t)sms * kDiePoolPages);
  std::vector<unsigned> col(sms);
  for (int p = 0; p < kDiePoolPages; ++p) {
    for (int b = 0; b < sms; ++b) col[b] = L[(size_t)b * kDiePoolPages + p];
    std::vector<unsigned> srt = col;
    std::nth_element(srt.begin(), srt.begin() + sms / 2, srt.end());
    const unsigned med = srt[sms / 2];
    for (int b = 0; b < sms; ++b) nearv[(size_t)b * kDiePoolPages + p] = col[b] < med;
  }
  // SM groups: agreement with CTA 0's pattern
  std::vector<int> grp(sms);
  int ng[2] = {0, 0};
  for (int b = 0; b < sms; ++b) {
    int agree = 0;
    for (int p = 0; p < kDiePoolPages; ++p) agree += nearv[(size_t)b * kDiePoolPages + p] == nearv[p];
    grp[b] = agree > kDiePoolPages / 2 ? 0 : 1;
    ng[grp[b]]++;
  }
  if (ng[0] == 0 || ng[1] == 0) return false;  // one die (or no measurable difference)
  // page home: the group that reaches it faster by a clear margin; ambiguous pages unused
  ws->die_pages = new int[2 * kDiePoolPages];
  ws->die_npages[0] = ws->die_npages[1] = 0;
  for (int p = 0; p < kDiePoolPages; ++p) {
    double m[2] = {0.0, 0.0};
    for (int b = 0; b < sms; ++b) m[grp[b]] += L[(size_t)b * kDiePoolPages + p];
    m[0] /= ng[0];
    m[1] /= ng[1];
    int h = -1;
    if (m[0] + 150.0 < m[1]) h = 0;
    else if (m[1] + 150.0 < m[0]) h = 1;
    if (h >= 0) ws->die_pages[h * kDiePoolPages + ws->die_npages[h]++] = p;
  }
  for (int b = 0; b < sms; ++b)
    if (grp[b] && S[b] < 192) ws->die_mask[S[b] >> 6] |= 1ull << (S[b] & 63);
  return ws->die_npages[0] >= kDieMaxPages && ws->die_npages[1] >= kDieMaxPages;
}

}  // namespace

bool die_copies(Workspace* ws, int64_t n, size_t s, cudaStream_t st) {
  static const bool enabled = [] {  // FP_DIE_COPIES=0 disables them (measurement)
    const char* e = getenv("FP_DIE_COPIES");
    return !(e && e[0] == '0');
  }();
  if (!enabled || n <= 0) return false;
  const int npg = (int)(((size_t)n * s + kPage - 1) / kPage);
  if (npg > kDieMaxPages) return false;
  if (ws->die_state == 0) ws->die_state = calibrate(ws, st) ? 1 : -1;
  if (ws->die_state != 1) return false;
  if (ws->die_tab_npg != npg) {
    std::vector<unsigned long long> h(2 * (size_t)npg);
    for (int g = 0; g < 2; ++g)
      for (int i = 0; i < npg; ++i)
        h[(size_t)g * npg + i] =
            (unsigned long long)((char*)ws->die_pool + (size_t)ws->die_pages[g * kDiePoolPages + i] * kPage);
    if (!ws->die_tab && cudaMalloc(&ws->die_tab, 2 * kDieMaxPages * sizeof(unsigned long long)) != cudaSuccess) {
      cudaGetLastError();
      ws->die_state = -1;
      return false;
    }
    cudaStreamSynchronize(st);  // a previous launch may still read the old table
    cudaMemcpy(ws->die_tab, h.data(), h.size() * sizeof(unsigned long long), cudaMemcpyHostToDevice);
    ws->die_tab_npg = npg;
  }
  return true;
}

fp_status launch_die_fold(Workspace* ws, void* w, int64_t n, fp_dtype dt, cudaStream_t s) {
  const int fb = 256;
  const int fg = (int)std::min<int64_t>((n + fb - 1) / fb, 4 * device_info(current_device()).sm_count);
  if (dt == FP_F64) k_die_fold<double><<<fg, fb, 0, s>>>((double*)w, ws->die_tab, ws->die_tab_npg, n);
  else k_die_fold<float><<<fg, fb, 0, s>>>((float*)w, ws->die_tab, ws->die_tab_npg, n);
  FP_CUDA(cudaGetLastError());
  return FP_OK;
}

}  // namespace fp
