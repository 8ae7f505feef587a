// TMA streaming microbenchmark: how fast can one CTA per SM (or several) stream a d-column fp32
// sample through a ring of shared-memory tiles, with the columns stored
//   soa   : [d][n]            -> d bulk copies of TILE*4 bytes per tile (the library's layout)
//   aosoa : [n/TILE][d][TILE] -> one bulk copy of d*TILE*4 bytes per tile
// and a consumer that reads every word of the tile once (sum) before releasing it
// (last warp out refills, as the scans do).  Answers whether the single-box scan at
// d = 10 is limited by the column-split copies or by the bytes in flight.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/tma_layout_bench.cu -o tools/bin/tma_layout_bench
//   tma_layout_bench  -> one JSON line per configuration
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int D, int TILE, int STAGES, bool AOSOA>
__global__ void __launch_bounds__(256) stream_kernel(const float* __restrict__ g, int64_t n, float* out) {
  extern __shared__ __align__(128) unsigned char sm[];
  float* tile = (float*)sm;
  uint64_t* bar = (uint64_t*)(tile + (size_t)STAGES * D * TILE);
  int* cnt = (int*)(bar + STAGES);
  const int64_t ntiles_all = n / TILE;
  const int64_t per = (ntiles_all + gridDim.x - 1) / gridDim.x;
  const int64_t t0 = blockIdx.x * per, t1 = min(ntiles_all, t0 + per);
  const int nt = (int)max((int64_t)0, t1 - t0);
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
      cnt[s] = 0;
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int k) {
    const int s = k % STAGES;
    const int64_t t = t0 + k;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])),
                 "r"((uint32_t)(D * TILE * 4)) : "memory");
    if (AOSOA) {
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
                       "r"(su32(tile + (size_t)s * D * TILE)), "l"(g + t * D * TILE), "r"((uint32_t)(D * TILE * 4)),
                   "r"(su32(&bar[s])) : "memory");
    } else {
      for (int j = 0; j < D; ++j)
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
                         "r"(su32(tile + ((size_t)s * D + j) * TILE)), "l"(g + (int64_t)j * n + t * TILE),
                     "r"((uint32_t)(TILE * 4)), "r"(su32(&bar[s])) : "memory");
    }
  };
  if (threadIdx.x == 0)
    for (int k = 0; k < STAGES && k < nt; ++k) issue(k);
  float acc = 0.0f;
  for (int k = 0; k < nt; ++k) {
    const int s = k % STAGES;
    const uint32_t par = (k / STAGES) & 1;
    asm volatile("{\n\t.reg .pred p;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n\t}" ::
                     "r"(su32(&bar[s])), "r"(par) : "memory");
    const float4* tl = (const float4*)(tile + (size_t)s * D * TILE);
    for (int i = threadIdx.x; i < D * TILE / 4; i += 256) {
      const float4 v = tl[i];
      acc += v.x + v.y + v.z + v.w;
    }
    __syncwarp();
    if ((threadIdx.x & 31) == 0) {
      __threadfence_block();
      if (atomicAdd(&cnt[s], 1) == 7) {
        cnt[s] = 0;
        if (k + STAGES < nt) issue(k + STAGES);
      }
    }
  }
  if (acc == 12345.678f) out[0] = acc;
}

template <int D, int TILE, int STAGES, bool AOSOA>
void run(const float* g, int64_t n, float* out, int sms, int per_sm) {
  const size_t smem = (size_t)STAGES * D * TILE * 4 + STAGES * 12 + 64;
  if (smem * per_sm > 227 * 1024) return;
  cudaFuncSetAttribute(stream_kernel<D, TILE, STAGES, AOSOA>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  const int grid = sms * per_sm;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e30f;
  for (int r = 0; r < 8; ++r) {
    cudaEventRecord(a);
    stream_kernel<D, TILE, STAGES, AOSOA><<<grid, 256, smem>>>(g, n, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (r >= 2 && ms < best) best = ms;
  }
  const cudaError_t e = cudaGetLastError();
  const double bytes = (double)n * D * 4;
  printf("{\"d\": %d, \"tile\": %d, \"stages\": %d, \"layout\": \"%s\", \"ctas_per_sm\": %d, \"us\": %.2f, \"GBps\": %.0f, \"err\": \"%s\"}\n",
         D, TILE, STAGES, AOSOA ? "aosoa" : "soa", per_sm, best * 1e3, bytes / (best * 1e-3) / 1e9, cudaGetErrorString(e));
}

int main() {
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int64_t n = 1 << 22;
  float* g;
  float* out;
  cudaMalloc(&g, (size_t)n * 16 * 4);
  cudaMalloc(&out, 64);
  cudaMemset(g, 0, (size_t)n * 16 * 4);
#define R(D, T, S, L, P) run<D, T, S, L>(g, n, out, sms, P);
  R(10, 2048, 2, false, 1) R(10, 2048, 2, true, 1)
  R(10, 1024, 4, false, 1) R(10, 1024, 4, true, 1)
  R(10, 1024, 2, false, 2) R(10, 1024, 2, true, 2)
  R(10, 512, 4, false, 2) R(10, 512, 4, true, 2)
  R(10, 512, 8, false, 1) R(10, 512, 8, true, 1)
  R(10, 256, 8, false, 2) R(10, 256, 8, true, 2)
  R(5, 2048, 2, false, 2) R(5, 2048, 2, true, 2)
  R(5, 2048, 4, false, 1) R(5, 2048, 4, true, 1)
  return 0;
}
