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

template <int D, bool GRAD, int TILE, int STAGES, int OCC>
void run_tma(ScanSingleArgs a, int sms) {
  int grid = sms * OCC;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  std::vector<float> ts;
  for (int r = 0; r < 10; ++r) {
    cudaEventRecord(e0);
    cudaError_t err = launch_single_tma_variant<D, GRAD, TILE, STAGES, OCC>(a, grid, 0);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    if (err != cudaSuccess) { printf("err %s\n", cudaGetErrorString(err)); return; }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    if (r >= 3) ts.push_back(ms);
  }
  std::sort(ts.begin(), ts.end());
  const double ms = ts[ts.size() / 2];
  double res[17]; cudaMemcpy(res, a.sums_out, 8, cudaMemcpyDeviceToHost);
  printf("{\"D\":%d,\"grad\":%d,\"kernel\":\"tma\",\"TILE\":%d,\"STAGES\":%d,\"OCC\":%d,\"us\":%.2f,\"GBps\":%.0f,\"S0\":%.6f}\n",
         D, (int)GRAD, TILE, STAGES, OCC, ms * 1e3, a.n * 4.0 * D / (ms * 1e-3) / 1e9, res[0]);
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
    hc.h[j] = h; hc.ap[j] = (float)(1.2011224087864498 / (1.4142135623730951 * h)); hc.renc[2 * j] = fenc_range(0.f); hc.renc[2 * j + 1] = fenc_range(100.f);
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
#define T(G, TILE, ST, OCC) run_tma<D, G, TILE, ST, OCC>(a, sms);
  R(false, 2, 4, false) R(true, 2, 3, false)
  { double r0[17]; cudaMemcpy(r0, a.sums_out, 8, cudaMemcpyDeviceToHost); printf("{\"ref_S0\":%.6f}\n", r0[0]); }
  T(false, 1024, 4, 2) T(false, 512, 4, 4) T(false, 512, 3, 4) T(false, 256, 4, 4) T(false, 1024, 3, 2)
  T(false, 512, 6, 3) T(false, 256, 8, 4)
  T(true, 1024, 4, 2) T(true, 512, 4, 3) T(true, 512, 4, 2) T(true, 256, 4, 3) T(true, 256, 8, 3)
  cudaFree(cols); cudaFree(lo); cudaFree(hi); cudaFree(c); cudaFree(bp); cudaFree(sums); cudaFree(cnt);
}

int main() {
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  sweep<5>(1 << 24, sms);
  sweep<10>(1 << 22, sms);
  return 0;
}
