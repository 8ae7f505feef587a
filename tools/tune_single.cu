// Tuning sweep for the single-box scan: points per vector load (VW), resident
// CTAs per SM (OCC), register double-buffered prefetch (PF).  Synthetic
// uniform data, one box, CUDA-event timing (median of 7 after 3 warm-ups).
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <cmath>
#include "../paper_conf_sigmod_heimelkm15_b200/csrc/scan.cuh"

using namespace kde;

template <int D, bool GRAD, int VW, int OCC, bool PF>
void run(ScanSingleArgs a, int sms) {
  const int64_t items = (a.n + 15) / 16;
  int grid = sms * OCC;
  if (grid > (items + 255) / 256) grid = (int)((items + 255) / 256);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  std::vector<float> ts;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(e0);
    cudaError_t err = launch_single_variant<D, GRAD, VW, OCC, PF>(a, grid, 0);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    if (err != cudaSuccess) { printf("err %s\n", cudaGetErrorString(err)); return; }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    if (r >= 3) ts.push_back(ms);
  }
  std::sort(ts.begin(), ts.end());
  const double ms = ts[ts.size() / 2];
  printf("{\"D\":%d,\"grad\":%d,\"VW\":%d,\"OCC\":%d,\"PF\":%d,\"us\":%.2f,\"GBps\":%.0f}\n", D, (int)GRAD, VW, OCC,
         (int)PF, ms * 1e3, a.n * 4.0 * D / (ms * 1e-3) / 1e9);
}

template <int D>
void sweep(int64_t n, int sms) {
  const int64_t ld = (n + 1023) / 1024 * 1024;
  std::vector<float> hcols(ld * D);
  srand(2);
  for (auto& x : hcols) x = 100.0f * rand() / RAND_MAX;
  float hl[16], hh[16];
  for (int j = 0; j < D; ++j) { hl[j] = 40; hh[j] = 60; }
  DevConsts hc{};
  const double h = 100.0 * pow((double)n, -1.0 / (D + 4)) * 0.29;
  for (int j = 0; j < D; ++j) {
    hc.h[j] = h; hc.ap[j] = (float)(1.2011224087864498 / (1.4142135623730951 * h)); hc.tmin[j] = 0.f; hc.tmax[j] = 100.f;
    hc.gconst[j] = 1.0 / (1.7724538509055160 * 1.2011224087864498 * h);
  }
  float *cols, *lo, *hi; DevConsts* c; double *bp, *sums; unsigned* cnt;
  cudaMalloc(&cols, ld * D * 4); cudaMalloc(&lo, 64); cudaMalloc(&hi, 64); cudaMalloc(&c, sizeof(DevConsts));
  cudaMalloc(&bp, sms * 8 * 17 * 8); cudaMalloc(&sums, 17 * 8); cudaMalloc(&cnt, 4); cudaMemset(cnt, 0, 4);
  cudaMemcpy(cols, hcols.data(), ld * D * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(lo, hl, 64, cudaMemcpyHostToDevice); cudaMemcpy(hi, hh, 64, cudaMemcpyHostToDevice);
  cudaMemcpy(c, &hc, sizeof(hc), cudaMemcpyHostToDevice);
  ScanSingleArgs a{};
  a.cols = cols; a.ld = ld; a.n = n; a.lo = lo; a.hi = hi; a.consts = c; a.c_out = nullptr; a.block_partials = bp;
  a.counter = cnt; a.sums_out = sums; a.fin_out = nullptr; a.n_global = (double)n;
#define R(G, VW, OCC, PF) run<D, G, VW, OCC, PF>(a, sms);
  R(false, 2, 4, true) R(false, 2, 4, false) R(false, 1, 4, true) R(false, 1, 4, false) R(false, 4, 4, false)
  R(false, 2, 3, true) R(false, 1, 6, false) R(false, 1, 8, false) R(false, 2, 6, false)
  R(true, 2, 3, true) R(true, 2, 3, false) R(true, 1, 3, true) R(true, 1, 4, false) R(true, 1, 4, true)
  R(true, 2, 2, true) R(true, 1, 6, false)
  cudaFree(cols); cudaFree(lo); cudaFree(hi); cudaFree(c); cudaFree(bp); cudaFree(sums); cudaFree(cnt);
}

int main() {
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  sweep<5>(1 << 24, sms);
  sweep<10>(1 << 22, sms);
  return 0;
}
