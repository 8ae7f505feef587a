// Microbenchmark: issue/throughput rates of FFMA, FFMA2, MUFU.EX2, MUFU.RCP, LOP3 on sm_100a.
// Each thread runs independent chains (ILP=8) so the pipe, not latency, binds.
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 4096
__global__ void k_ffma(float* out, float a, float b) {
  float x[8]; for (int i=0;i<8;i++) x[i]=threadIdx.x*0.001f+i;
  for (int it=0; it<ITERS; ++it) {
#pragma unroll
    for (int i=0;i<8;i++) x[i]=fmaf(x[i],a,b);
  }
  float s=0; for(int i=0;i<8;i++) s+=x[i]; if (s==1234.5f) out[0]=s;
}
__global__ void k_ffma2(float* out, float a, float b) {
  float2 x[8]; for (int i=0;i<8;i++) x[i]=make_float2(threadIdx.x*0.001f+i, i*0.5f);
  float2 A=make_float2(a,a), B=make_float2(b,b);
  for (int it=0; it<ITERS; ++it) {
#pragma unroll
    for (int i=0;i<8;i++) x[i]=__ffma2_rn(x[i],A,B);
  }
  float s=0; for(int i=0;i<8;i++) s+=x[i].x+x[i].y; if (s==1234.5f) out[0]=s;
}
__global__ void k_ex2(float* out, float a) {
  float x[8]; for (int i=0;i<8;i++) x[i]=threadIdx.x*1e-6f+i*1e-3f;
  for (int it=0; it<ITERS; ++it) {
#pragma unroll
    for (int i=0;i<8;i++) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x[i])); x[i]=y; }
  }
  float s=0; for(int i=0;i<8;i++) s+=x[i]; if (s==1234.5f) out[0]=s;
}
__global__ void k_rcp(float* out, float a) {
  float x[8]; for (int i=0;i<8;i++) x[i]=1.0f+threadIdx.x*1e-6f+i*1e-3f;
  for (int it=0; it<ITERS; ++it) {
#pragma unroll
    for (int i=0;i<8;i++) { float y; asm volatile("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x[i])); x[i]=y; }
  }
  float s=0; for(int i=0;i<8;i++) s+=x[i]; if (s==1234.5f) out[0]=s;
}
__global__ void k_lop(unsigned* out, unsigned a) {
  unsigned x[8]; for (int i=0;i<8;i++) x[i]=threadIdx.x+i;
  for (int it=0; it<ITERS; ++it) {
#pragma unroll
    for (int i=0;i<8;i++) x[i]=(x[i]^a)&(x[i]|0x5555u);
  }
  unsigned s=0; for(int i=0;i<8;i++) s+=x[i]; if (s==12345u) out[0]=s;
}
// mixed: per iteration 8 FFMA2 + 1 EX2 per chain-pair ratio probe
__global__ void k_mix(float* out, float a, float b) {
  float2 x[4]; float e[4];
  for (int i=0;i<4;i++){ x[i]=make_float2(threadIdx.x*0.001f+i, i*0.5f); e[i]=i*1e-3f; }
  float2 A=make_float2(a,a), B=make_float2(b,b);
  for (int it=0; it<ITERS; ++it) {
#pragma unroll
    for (int i=0;i<4;i++) {
      x[i]=__ffma2_rn(x[i],A,B); x[i]=__ffma2_rn(x[i],A,B); x[i]=__ffma2_rn(x[i],A,B); x[i]=__ffma2_rn(x[i],A,B);
      float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(e[i])); e[i]=y;
    }
  }
  float s=0; for(int i=0;i<4;i++) s+=x[i].x+x[i].y+e[i]; if (s==1234.5f) out[0]=s;
}
int main() {
  int dev=0; cudaDeviceProp p; cudaGetDeviceProperties(&p, dev);
  int clk=0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  printf("{\"name\":\"%s\",\"sms\":%d,\"l2_bytes\":%d,\"clock_khz_attr\":%d,\"smem_optin\":%zu}\n", p.name, p.multiProcessorCount, p.l2CacheSize, clk, p.sharedMemPerBlockOptin);
  float* d; cudaMalloc(&d, 64);
  int blocks = p.multiProcessorCount*8, threads=256;
  cudaEvent_t s,e; cudaEventCreate(&s); cudaEventCreate(&e);
  auto run=[&](const char* name, double ops_per_thread_iter, auto launch){
    launch(); cudaDeviceSynchronize();
    float best=1e30f;
    for(int r=0;r<5;r++){ cudaEventRecord(s); launch(); cudaEventRecord(e); cudaEventSynchronize(e); float ms; cudaEventElapsedTime(&ms,s,e); if(ms<best)best=ms; }
    double thr_ops = (double)blocks*threads*ITERS*ops_per_thread_iter;
    double per_sm_clk_at1965 = thr_ops/(best*1e-3)/p.multiProcessorCount/1.965e9;
    printf("{\"op\":\"%s\",\"ms\":%.4f,\"Gops_per_s\":%.1f,\"lane_ops_per_SM_per_clk_at_1965\":%.2f}\n", name, best, thr_ops/(best*1e-3)/1e9, per_sm_clk_at1965);
  };
  run("FFMA (lane-ops)", 8, [&]{k_ffma<<<blocks,threads>>>(d,1.0001f,0.0001f);});
  run("FFMA2 (lane-ops, 2 per instr)", 16, [&]{k_ffma2<<<blocks,threads>>>(d,1.0001f,0.0001f);});
  run("FFMA2 (instr)", 8, [&]{k_ffma2<<<blocks,threads>>>(d,1.0001f,0.0001f);});
  run("MUFU.EX2", 8, [&]{k_ex2<<<blocks,threads>>>(d,1.0f);});
  run("MUFU.RCP", 8, [&]{k_rcp<<<blocks,threads>>>(d,1.0f);});
  run("LOP3-ish (2 ops)", 16, [&]{k_lop<<<blocks,threads>>>((unsigned*)d,0x1234u);});
  run("MIX 16 FFMA2 + 4 EX2 (instr)", 20, [&]{k_mix<<<blocks,threads>>>(d,1.0001f,0.0001f);});
  return 0;
}
