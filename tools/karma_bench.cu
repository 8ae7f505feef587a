// Standalone A/B timing of the karma pass (karma_kernel + compact_fused_kernel,
// the production launcher from kernels.cu, compiled into this file so KDE_TUNE_KARMA_*
// macro variants stay self-contained):
//   karma_bench n [reps]
// Synthetic retained contributions c ~ U(0, 2/n), karma ~ U(-1, 1) (a few % flagged),
// absolute loss, no streaming tail.  L2 flushed (512 MiB write) before every rep.
// Prints one JSON line: medians of the two kernels (CUDA events on the launching stream).
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_sigmod_heimelkm15_b200/csrc/kernels.cu"

using namespace kde;

#define CK(x)                                                                  \
  do {                                                                         \
    cudaError_t e_ = (x);                                                      \
    if (e_ != cudaSuccess) {                                                   \
      fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
      exit(1);                                                                 \
    }                                                                          \
  } while (0)

int main(int argc, char** argv) {
  const int64_t n = argc > 1 ? atoll(argv[1]) : (1ll << 22);
  const int reps = argc > 2 ? atoi(argv[2]) : 50;
  const int nb = karma_blocks(n);
  std::vector<float> hc(n);
  std::vector<double> hk(n);
  uint64_t x = 88172645463325252ull;
  auto rnd = [&]() { x ^= x << 13; x ^= x >> 7; x ^= x << 17; return (double)(x >> 11) * (1.0 / 9007199254740992.0); };
  for (int64_t i = 0; i < n; ++i) {
    hc[i] = (float)(rnd() * 2.0 / (double)n);
    hk[i] = 2.0 * rnd() - 1.0;
  }
  float *c, *lo, *hi;
  double *k, *phat, *p;
  uint32_t* bitmap;
  int32_t* counts;
  int64_t* offsets;
  unsigned* done;
  int64_t *idx, *total;
  char* flush;
  const size_t flush_bytes = 512ull << 20;
  const int64_t npad = (n + 2047) / 2048 * 2048;
  CK(cudaMalloc(&c, npad * 4));
  CK(cudaMalloc(&k, npad * 8));
  CK(cudaMalloc(&lo, 64));
  CK(cudaMalloc(&hi, 64));
  CK(cudaMalloc(&phat, 8));
  CK(cudaMalloc(&p, 8));
  CK(cudaMalloc(&bitmap, ((n + 31) / 32 + 1024) * 4));
  CK(cudaMalloc(&counts, (nb + 1) * 4));
  CK(cudaMalloc(&offsets, (nb + 1) * 8));
  CK(cudaMalloc(&done, 8));
  CK(cudaMalloc(&idx, n * 8));
  CK(cudaMalloc(&total, 8));
  CK(cudaMalloc(&flush, flush_bytes));
  CK(cudaMemcpy(c, hc.data(), n * 4, cudaMemcpyHostToDevice));
  CK(cudaMemset(done, 0, 8));
  const double hp = 1.0 / (double)n * 0.5, pp = 0.3;
  CK(cudaMemcpy(phat, &hp, 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(p, &pp, 8, cudaMemcpyHostToDevice));
  KarmaParamsDev kp{};
  kp.loss = 1;
  kp.empty_region = 0;
  kp.k_max = 4.0;
  kp.threshold = -0.99;
  StreamTail tail{};
  cudaStream_t s;
  CK(cudaStreamCreate(&s));
  cudaEvent_t e0, e1, e2;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaEventCreate(&e2));
  std::vector<float> tk, tc;
  int64_t tot = 0;
  for (int r = 0; r < reps + 3; ++r) {
    CK(cudaMemcpyAsync(k, hk.data(), n * 8, cudaMemcpyHostToDevice, s));
    CK(cudaMemsetAsync(flush, r & 0xff, flush_bytes, s));
    CK(cudaEventRecord(e0, s));
    karma_kernel<<<nb, kKarmaThreads, 0, s>>>(c, k, n, (double)n, phat, p, kp, lo, hi, 1, nullptr, bitmap, counts,
                                              offsets, done + 1, (int)nb);
    CK(cudaEventRecord(e1, s));
    compact_fused_kernel<<<nb, kKarmaThreads, 0, s>>>(bitmap, n, offsets, nb, 0, idx, n, total, done, tail);
    CK(cudaEventRecord(e2, s));
    CK(cudaStreamSynchronize(s));
    CK(cudaGetLastError());
    float a, b;
    CK(cudaEventElapsedTime(&a, e0, e1));
    CK(cudaEventElapsedTime(&b, e1, e2));
    if (r >= 3) {
      tk.push_back(a * 1e3f);
      tc.push_back(b * 1e3f);
    }
  }
  CK(cudaMemcpy(&tot, total, 8, cudaMemcpyDeviceToHost));
  std::sort(tk.begin(), tk.end());
  std::sort(tc.begin(), tc.end());
  const double km = tk[tk.size() / 2], cm = tc[tc.size() / 2];
  printf("{\"n\":%lld,\"PB\":%d,\"MINB\":%d,\"karma_us\":%.2f,\"karma_GBps\":%.1f,\"compact_us\":%.2f,\"flagged\":%lld}\n",
         (long long)n, KDE_TUNE_KARMA_PB, KDE_TUNE_KARMA_MINB, km, (double)n * 20.125 / km * 1e-3, cm,
         (long long)tot);
  return 0;
}
