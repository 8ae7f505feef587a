// Tuning sweep for the batched scan: boxes per thread (QT), resident CTAs per
// SM (MINB) and waves.  Standalone (no Python): synthetic uniform data,
// random boxes, CUDA-event timing (median of 5 launches after 2 warm-ups).
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <cmath>
#include "../paper_conf_sigmod_heimelkm15_b200/csrc/scan.cuh"

using namespace kde;

template <int D, int QT, int MINB, int PU = 1>
void run(int64_t n, int64_t q, int waves, const float* cols, int64_t ld, const float* lo, const float* hi,
         const DevConsts* consts, double* partials, int sms) {
  ScanBatchedArgs a{};
  a.cols = cols; a.ld = ld; a.n = n; a.lo = lo; a.hi = hi; a.q = q; a.consts = consts; a.partials = partials;
  int64_t qtiles, splits, len;
  a.qb = batched_qb(q);
  batched_grid(q, n, a.qb, MINB, sms, waves, &qtiles, &splits, &len);
  a.split_len = len;
  dim3 grid((unsigned)qtiles, (unsigned)splits);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  std::vector<float> ts;
  for (int r = 0; r < 7; ++r) {
    cudaEventRecord(e0);
    cudaError_t err = launch_batched_tg<D, true, QT, MINB, PU>(a, grid, 0);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    if (err != cudaSuccess) { printf("err %s\n", cudaGetErrorString(err)); return; }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    if (r >= 2) ts.push_back(ms);
  }
  std::sort(ts.begin(), ts.end());
  const double ms = ts[ts.size() / 2];
  printf("{\"D\":%d,\"PU\":%d,\"QT\":%d,\"MINB\":%d,\"waves\":%d,\"grid\":[%lld,%lld],\"ms\":%.3f,\"Gptq_s\":%.1f}\n", D, PU, QT, MINB,
         waves, (long long)qtiles, (long long)splits, ms, n * (double)q / (ms * 1e-3) / 1e9);
}

template <int D>
void setup_and_sweep(int64_t n, int64_t q, int sms) {
  const int64_t ld = (n + 1023) / 1024 * 1024;
  std::vector<float> h_cols(ld * D), h_lo(q * D), h_hi(q * D);
  srand(1);
  for (auto& x : h_cols) x = 100.0f * rand() / RAND_MAX;
  for (int64_t k = 0; k < q * D; ++k) {
    float c = 100.0f * rand() / RAND_MAX, w = 5.0f + 30.0f * rand() / RAND_MAX;
    h_lo[k] = c - w / 2; h_hi[k] = c + w / 2;
  }
  DevConsts hc{};
  const double h = 100.0 * pow((double)n, -1.0 / (D + 4)) * 0.29;
  for (int j = 0; j < D; ++j) {
    hc.h[j] = h; hc.ap[j] = (float)(1.2011224087864498 / (1.4142135623730951 * h)); hc.renc[2 * j] = fenc_range(0.f); hc.renc[2 * j + 1] = fenc_range(100.f);
    hc.gconst[j] = 1.0 / (1.7724538509055160 * 1.2011224087864498 * h);
  }
  float *cols, *lo, *hi; DevConsts* c; double* part;
  cudaMalloc(&cols, ld * D * 4); cudaMalloc(&lo, q * D * 4); cudaMalloc(&hi, q * D * 4);
  cudaMalloc(&c, sizeof(DevConsts)); cudaMalloc(&part, (size_t)sms * 16 * (D + 1) * q * 8);
  cudaMemcpy(cols, h_cols.data(), ld * D * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(lo, h_lo.data(), q * D * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(hi, h_hi.data(), q * D * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(c, &hc, sizeof(hc), cudaMemcpyHostToDevice);
#define R(QT, MINB, W) run<D, QT, MINB>(n, q, W, cols, ld, lo, hi, c, part, sms);
#define RU(QT, MINB, W, PU) run<D, QT, MINB, PU>(n, q, W, cols, ld, lo, hi, c, part, sms);
  if constexpr (D <= 3) {
    RU(1, 4, 4, 2) R(1, 4, 4) RU(1, 4, 4, 4) RU(1, 3, 4, 2) RU(1, 4, 8, 2)
  } else if constexpr (D <= 6) {
    R(1, 4, 4) RU(1, 4, 4, 2) RU(1, 3, 4, 2)
  } else {
    R(1, 3, 4) RU(1, 3, 4, 2) RU(1, 2, 4, 2)
  }
  cudaFree(cols); cudaFree(lo); cudaFree(hi); cudaFree(c); cudaFree(part);
}

int main() {
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  setup_and_sweep<3>(1 << 20, 100, sms);   // batch-optimisation training set size
  setup_and_sweep<3>(1 << 20, 300, sms);
  setup_and_sweep<3>(1 << 20, 10000, sms);
  setup_and_sweep<5>(1 << 22, 4096, sms);
  setup_and_sweep<8>(1 << 22, 4096, sms);
  return 0;
}
