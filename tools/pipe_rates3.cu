// Does the sm_100 FMA pipe pair packed FFMA2 (fmaheavy) with scalar FFMA
// (fmalite) in the same cycles?  Independent chains, 148*8 CTAs x 256 threads;
// lane-ops per SM per clock at 1965 MHz for several FFMA2 : FFMA mixes.
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 2048
template <int N2, int N1>
__global__ void mix(float* out, const float* in) {
  const float a = in[threadIdx.x & 7], b = in[8 + (threadIdx.x & 7)];
  float2 x2[N2 > 0 ? N2 : 1];
  float x1[N1 > 0 ? N1 : 1];
  for (int i = 0; i < N2; i++) x2[i] = make_float2(in[16 + i], in[17 + i]);
  for (int i = 0; i < N1; i++) x1[i] = in[24 + i];
  for (int it = 0; it < ITERS; ++it) {
#pragma unroll
    for (int i = 0; i < (N2 > N1 ? N2 : N1); i++) {
      if (i < N2) x2[i] = __ffma2_rn(x2[i], make_float2(a, a), make_float2(b, b));
      if (i < N1) x1[i] = fmaf(x1[i], a, b);
    }
  }
  float s = 0;
  for (int i = 0; i < N2; i++) s += x2[i].x + x2[i].y;
  for (int i = 0; i < N1; i++) s += x1[i];
  if (s == 1234.5f) out[0] = s;
}
int main() {
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  float h[64];
  for (int i = 0; i < 64; i++) h[i] = 1.0f + 1e-3f * i;
  float *in, *out;
  cudaMalloc(&in, 256);
  cudaMalloc(&out, 64);
  cudaMemcpy(in, h, 256, cudaMemcpyHostToDevice);
  const int blocks = p.multiProcessorCount * 8, threads = 256;
  cudaEvent_t s, e;
  cudaEventCreate(&s);
  cudaEventCreate(&e);
  auto run = [&](const char* name, int n2, int n1, auto k) {
    k<<<blocks, threads>>>(out, in);
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < 5; r++) {
      cudaEventRecord(s);
      k<<<blocks, threads>>>(out, in);
      cudaEventRecord(e);
      cudaEventSynchronize(e);
      float ms;
      cudaEventElapsedTime(&ms, s, e);
      if (ms < best) best = ms;
    }
    const double lanes = (double)blocks * threads * ITERS * (2.0 * n2 + n1);
    const double instr = (double)blocks * threads * ITERS * (n2 + n1) / 32.0;
    const double clk = 1.965e9 * best * 1e-3 * p.multiProcessorCount;
    printf("{\"mix\":\"%s\",\"ms\":%.4f,\"lane_ops_per_SM_clk\":%.1f,\"warp_instr_per_SMSP_clk\":%.3f}\n", name, best,
           lanes / clk, instr / clk / 4);
  };
  run("8 FFMA2", 8, 0, mix<8, 0>);
  run("8 FFMA", 0, 8, mix<0, 8>);
  run("4 FFMA2 + 4 FFMA", 4, 4, mix<4, 4>);
  run("4 FFMA2 + 8 FFMA", 4, 8, mix<4, 8>);
  run("6 FFMA2 + 2 FFMA", 6, 2, mix<6, 2>);
  run("8 FFMA2 + 8 FFMA", 8, 8, mix<8, 8>);
  return 0;
}
