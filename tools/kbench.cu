// Standalone single-configuration benchmark of the production scan launchers
// (launch_single_t / launch_batched_t, the same template instances libkde
// uses), for ncu captures and quick A/B runs of kernel variants:
//   kbench single  D grad n       [reps]
//   kbench batched D grad n q     [reps]
// Synthetic uniform data in [0, 100)^D, boxes of width 5..35, Scott-like h.
// Prints one JSON line (median of reps after 3 warm-ups, CUDA events).
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "../paper_conf_sigmod_heimelkm15_b200/csrc/scan.cuh"

using namespace kde;

// mirror of scan_single_grid (scan_dispatch.cu), so this file needs no link
// against libkde objects and macro variants of the kernels stay self-contained
static int kb_single_grid(int d, bool grad, int64_t n, int num_sms) {
  if (single_uses_tma(d)) {
    int64_t grid = (int64_t)num_sms * single_tma_occ(d);
    const int64_t ntiles = (n + kSingleTile - 1) / kSingleTile;
    if (grid > ntiles) grid = ntiles;
    return (int)(grid < 1 ? 1 : grid);
  }
  int64_t grid = (int64_t)num_sms * single_occ(d, grad);
  const int64_t need = ((n + 15) / 16 + kSingleThreads - 1) / kSingleThreads;
  if (grid > need) grid = need;
  return (int)(grid < 1 ? 1 : grid);
}

template <int D>
int run(bool batched, bool grad, int64_t n, int64_t q, int reps) {
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int64_t ld = (n + kColAlign - 1) / kColAlign * kColAlign;
  std::vector<float> h_cols(ld * D, 0.0f), h_lo(q * D), h_hi(q * D);
  srand(1);
  for (int j = 0; j < D; ++j)
    for (int64_t i = 0; i < n; ++i) h_cols[j * ld + i] = 100.0f * rand() / RAND_MAX;
  for (int64_t k = 0; k < q * D; ++k) {
    float c = 100.0f * rand() / RAND_MAX, w = 5.0f + 30.0f * rand() / RAND_MAX;
    h_lo[k] = c - w / 2;
    h_hi[k] = c + w / 2;
  }
  DevConsts hc{};
  hc.kernel = kGaussian;
  const double h = 100.0 * pow((double)n, -1.0 / (D + 4)) * 0.29;
  for (int j = 0; j < D; ++j) {
    hc.h[j] = h;
    hc.ap[j] = (float)(1.2011224087864498 / (1.4142135623730951 * h));
    hc.renc[2 * j] = fenc_range(0.f);
    hc.renc[2 * j + 1] = fenc_range(100.f);
    hc.gconst[j] = 1.0 / (1.7724538509055160 * 1.2011224087864498 * h);
  }
  float *cols, *lo, *hi;
  DevConsts* c;
  double *buf, *sums;
  unsigned* cnt;
  const size_t bufsz = (size_t)std::max<int64_t>(sms * 64 * (D + 1), (int64_t)sms * 16 * (D + 1) * q) * 8;
  cudaMalloc(&cols, ld * D * 4);
  cudaMalloc(&lo, q * D * 4);
  cudaMalloc(&hi, q * D * 4);
  cudaMalloc(&c, sizeof(DevConsts));
  cudaMalloc(&buf, bufsz);
  cudaMalloc(&sums, 64 * 8);
  cudaMalloc(&cnt, 4);
  cudaMemset(cnt, 0, 4);
  cudaMemcpy(cols, h_cols.data(), ld * D * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(lo, h_lo.data(), q * D * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(hi, h_hi.data(), q * D * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(c, &hc, sizeof(hc), cudaMemcpyHostToDevice);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  std::vector<float> ts;
  int splits = 0;
  for (int r = 0; r < reps + 3; ++r) {
    cudaEventRecord(e0);
    cudaError_t err;
    if (batched) {
      ScanBatchedArgs a{};
      a.cols = cols; a.ld = ld; a.n = n; a.lo = lo; a.hi = hi; a.q = q; a.consts = c; a.partials = buf;
      err = launch_batched_t<D>(grad, a, sms, &splits, 0, false);
    } else {
      ScanSingleArgs a{};
      a.cols = cols; a.ld = ld; a.n = n; a.lo = lo; a.hi = hi; a.consts = c; a.block_partials = buf;
      a.counter = cnt; a.sums_out = sums; a.n_global = (double)n;
      err = launch_single_t<D>(grad, a, kb_single_grid(D, grad, n, sms), 0);
    }
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    if (err != cudaSuccess || cudaGetLastError() != cudaSuccess) {
      printf("{\"error\":\"%s\"}\n", cudaGetErrorString(err));
      return 1;
    }
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (r >= 3) ts.push_back(ms);
  }
  std::sort(ts.begin(), ts.end());
  const double ms = ts[ts.size() / 2];
  double s0 = 0.0;
  if (!batched) cudaMemcpy(&s0, sums, 8, cudaMemcpyDeviceToHost);
  printf("{\"kind\":\"%s\",\"D\":%d,\"grad\":%d,\"n\":%lld,\"q\":%lld,\"us\":%.2f,\"GBps\":%.0f,\"Gptq_s\":%.1f,"
         "\"splits\":%d,\"S0\":%.9g}\n",
         batched ? "batched" : "single", D, (int)grad, (long long)n, (long long)q, ms * 1e3,
         batched ? 0.0 : n * 4.0 * D / (ms * 1e-3) / 1e9, (double)n * q / (ms * 1e-3) / 1e9, splits, s0);
  return 0;
}

int main(int argc, char** argv) {
  if (argc < 5) {
    fprintf(stderr, "usage: kbench single|batched D grad n [q] [reps]\n");
    return 2;
  }
  const bool batched = !strcmp(argv[1], "batched");
  const int d = atoi(argv[2]);
  const bool grad = atoi(argv[3]) != 0;
  const int64_t n = atoll(argv[4]);
  const int64_t q = batched ? atoll(argv[5]) : 1;
  const int reps = argc > (batched ? 6 : 5) ? atoi(argv[batched ? 6 : 5]) : 10;
  switch (d) {
    case 3: return run<3>(batched, grad, n, q, reps);
    case 5: return run<5>(batched, grad, n, q, reps);
    case 8: return run<8>(batched, grad, n, q, reps);
    case 10: return run<10>(batched, grad, n, q, reps);
  }
  fprintf(stderr, "D must be 3, 5, 8 or 10\n");
  return 2;
}
