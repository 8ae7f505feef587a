// FP32 issue-form microbenchmark on sm_100a: which FFMA / FFMA2 / FMUL2 / FADD2
// operand forms run at full rate.  8 independent chains per thread, 148*8 CTAs.
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 2048
__global__ void ffma_rrr(float* out, const float* in) {
  float a = in[threadIdx.x & 7], b = in[8 + (threadIdx.x & 7)];
  float x[8]; for (int i = 0; i < 8; i++) x[i] = in[16 + i];
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = fmaf(x[i], a, b);
  float s = 0; for (int i = 0; i < 8; i++) s += x[i]; if (s == 1234.5f) out[0] = s;
}
__global__ void ffma_rri(float* out, const float* in) {
  float a = in[threadIdx.x & 7];
  float x[8]; for (int i = 0; i < 8; i++) x[i] = in[16 + i];
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = fmaf(x[i], a, 0.3125f);
  float s = 0; for (int i = 0; i < 8; i++) s += x[i]; if (s == 1234.5f) out[0] = s;
}
__global__ void ffma2_rrr(float* out, const float* in) {
  float2 a = make_float2(in[threadIdx.x & 7], in[1 + (threadIdx.x & 7)]), b = make_float2(in[8], in[9]);
  float2 x[8]; for (int i = 0; i < 8; i++) x[i] = make_float2(in[16 + i], in[17 + i]);
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = __ffma2_rn(x[i], a, b);
  float s = 0; for (int i = 0; i < 8; i++) s += x[i].x + x[i].y; if (s == 1234.5f) out[0] = s;
}
__global__ void ffma2_rri(float* out, const float* in) {
  float2 a = make_float2(in[threadIdx.x & 7], in[1 + (threadIdx.x & 7)]);
  float2 x[8]; for (int i = 0; i < 8; i++) x[i] = make_float2(in[16 + i], in[17 + i]);
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = __ffma2_rn(x[i], a, make_float2(0.3125f, 0.3125f));
  float s = 0; for (int i = 0; i < 8; i++) s += x[i].x + x[i].y; if (s == 1234.5f) out[0] = s;
}
__global__ void fmul2_rr(float* out, const float* in) {
  float2 a = make_float2(in[threadIdx.x & 7], in[1 + (threadIdx.x & 7)]);
  float2 x[8]; for (int i = 0; i < 8; i++) x[i] = make_float2(in[16 + i], in[17 + i]);
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = __fmul2_rn(x[i], a);
  float s = 0; for (int i = 0; i < 8; i++) s += x[i].x + x[i].y; if (s == 1234.5f) out[0] = s;
}
__global__ void fadd_rr(float* out, const float* in) {
  float a = in[threadIdx.x & 7];
  float x[8]; for (int i = 0; i < 8; i++) x[i] = in[16 + i];
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = x[i] + a;
  float s = 0; for (int i = 0; i < 8; i++) s += x[i]; if (s == 1234.5f) out[0] = s;
}
__global__ void fmul_rr(float* out, const float* in) {
  float a = in[threadIdx.x & 7];
  float x[8]; for (int i = 0; i < 8; i++) x[i] = in[16 + i];
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = x[i] * a;
  float s = 0; for (int i = 0; i < 8; i++) s += x[i]; if (s == 1234.5f) out[0] = s;
}
__global__ void lop3_rr(float* out, const float* in) {
  unsigned a = __float_as_uint(in[threadIdx.x & 7]);
  unsigned x[8]; for (int i = 0; i < 8; i++) x[i] = __float_as_uint(in[16 + i]);
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) x[i] = (x[i] ^ a) | 0x80000000u;
  unsigned s = 0; for (int i = 0; i < 8; i++) s += x[i]; if (s == 12345u) out[0] = s;
}
__global__ void rcp_chain(float* out, const float* in) {
  float x[8]; for (int i = 0; i < 8; i++) x[i] = 1.0f + in[16 + i];
  for (int it = 0; it < ITERS; ++it)
#pragma unroll
    for (int i = 0; i < 8; i++) { float y; asm volatile("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x[i])); x[i] = y + 1.0f; }
  float s = 0; for (int i = 0; i < 8; i++) s += x[i]; if (s == 1234.5f) out[0] = s;
}
int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  float h[64]; for (int i = 0; i < 64; i++) h[i] = 1.0f + 1e-3f * i;
  float *in, *out; cudaMalloc(&in, 256); cudaMalloc(&out, 64); cudaMemcpy(in, h, 256, cudaMemcpyHostToDevice);
  int blocks = p.multiProcessorCount * 8, threads = 256;
  cudaEvent_t s, e; cudaEventCreate(&s); cudaEventCreate(&e);
  auto run = [&](const char* name, double instr_per_iter, double lanes_per_instr, auto k) {
    k<<<blocks, threads>>>(out, in); cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < 5; r++) { cudaEventRecord(s); k<<<blocks, threads>>>(out, in); cudaEventRecord(e); cudaEventSynchronize(e); float ms; cudaEventElapsedTime(&ms, s, e); if (ms < best) best = ms; }
    double instr = (double)blocks * threads * ITERS * instr_per_iter;
    double clk = 1.965e9 * best * 1e-3 * p.multiProcessorCount;
    printf("{\"op\":\"%s\",\"ms\":%.4f,\"thread_instr_per_SM_clk\":%.1f,\"lane_ops_per_SM_clk\":%.1f}\n", name, best, instr / clk, instr * lanes_per_instr / clk);
  };
  run("FFMA r,r,r", 8, 1, ffma_rrr);
  run("FFMA r,r,imm", 8, 1, ffma_rri);
  run("FFMA2 r,r,r", 8, 2, ffma2_rrr);
  run("FFMA2 r,r,imm", 8, 2, ffma2_rri);
  run("FMUL2 r,r", 8, 2, fmul2_rr);
  run("FADD r,r", 8, 1, fadd_rr);
  run("FMUL r,r", 8, 1, fmul_rr);
  run("LOP3", 8, 1, lop3_rr);
  run("MUFU.RCP + FADD", 8, 1, rcp_chain);
  return 0;
}
