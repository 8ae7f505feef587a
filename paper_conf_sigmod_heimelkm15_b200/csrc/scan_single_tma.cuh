// scan_single_tma.cuh -- single-box scan with the sample streamed through
// shared memory by TMA bulk copies (included at the end of scan.cuh).
//
// Each CTA owns a contiguous chunk of the sample and walks it in tiles of
// TILE points x d columns.  One elected thread keeps STAGES tiles in flight
// (cp.async.bulk global -> shared, completion on an mbarrier with expect_tx),
// so HBM requests are decoupled from the registers and latency of the compute
// warps: the memory system sees STAGES * TILE * 4d bytes outstanding per CTA
// while every thread computes on its points of the current tile.  A stage is
// reused after the CTA barrier that ends the tile that read it.
#pragma once

namespace kde {

template <int D, int TILE, int STAGES>
constexpr size_t single_tma_smem_bytes() {
  return (size_t)STAGES * D * TILE * sizeof(float) + STAGES * sizeof(uint64_t);
}

template <int D, bool GRAD, int MODE, int TILE, int STAGES>
__device__ __forceinline__ void scan_single_tma_body(const ScanSingleArgs& a, const float4* smc, float* tiles,
                                                     uint64_t* full, int64_t c0, int64_t c1, int ntiles) {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int PPT = TILE / kSingleThreads;  // points per thread per tile
  const int tid = threadIdx.x;
  double acc[NA];
#pragma unroll
  for (int k = 0; k < NA; ++k) acc[k] = 0.0;
  for (int k = 0; k < ntiles; ++k) {
    const int st = k % STAGES;
    mbar_wait_parity(&full[st], (uint32_t)((k / STAGES) & 1));
    const float* tl = tiles + (size_t)st * D * TILE;
    const int64_t base = c0 + (int64_t)k * TILE;
    const int64_t rem = c1 - base;
    const int npts = rem < TILE ? (int)rem : TILE;
    float s[NA];
#pragma unroll
    for (int kk = 0; kk < NA; ++kk) s[kk] = 0.0f;
    BoxDim bd[D];
    float ap[D];
#pragma unroll
    for (int j = 0; j < D; ++j) {
      const float4 c = smc[j];
      bd[j].b = make_float2(c.x, c.y);
      bd[j].hd = c.z;
      ap[j] = c.w;
    }
#pragma unroll
    for (int r = 0; r < PPT; ++r) {
      const int p = tid + r * kSingleThreads;
      const bool valid = p < npts;
      float t[D];
#pragma unroll
      for (int j = 0; j < D; ++j) t[j] = tl[j * TILE + p];
      const float c = point_box<D, GRAD, MODE>(bd, t, ap, s, valid);
      if (a.c_out && valid) __stcs(a.c_out + base + p, c);
    }
#pragma unroll
    for (int kk = 0; kk < NA; ++kk) acc[kk] += (double)s[kk];
    __syncthreads();  // every thread is done with stage st
    if (tid == 0 && k + STAGES < ntiles) {
      const int64_t nb = c0 + (int64_t)(k + STAGES) * TILE;
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_arrive_expect_tx(&full[st], (uint32_t)(D * TILE * sizeof(float)));
#pragma unroll
      for (int j = 0; j < D; ++j)
        bulk_g2s(tiles + ((size_t)st * D + j) * TILE, a.cols + (int64_t)j * a.ld + nb, (uint32_t)(TILE * sizeof(float)),
                 &full[st]);
    }
  }
  single_reduce_finalize<NA>(a, acc);
}

template <int D, bool GRAD, int TILE, int STAGES, int OCC>
__global__ void __launch_bounds__(kSingleThreads, OCC) scan_single_tma_kernel(const ScanSingleArgs a) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  float* tiles = reinterpret_cast<float*>(smem_raw);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + (size_t)STAGES * D * TILE * sizeof(float));
  __shared__ float4 smc[D];
  __shared__ int narrow_s;
  const int tid = threadIdx.x;
  // contiguous chunk of this CTA, a multiple of TILE points
  const int64_t ntile_total = (a.n + TILE - 1) / TILE;
  const int64_t tiles_per = (ntile_total + gridDim.x - 1) / gridDim.x;
  const int64_t c0 = (int64_t)blockIdx.x * tiles_per * TILE;
  const int64_t c1 = min(a.n, c0 + tiles_per * TILE);
  const int ntiles = c1 > c0 ? (int)((c1 - c0 + TILE - 1) / TILE) : 0;
  if (tid == 0) {
    narrow_s = 0;
    for (int st = 0; st < STAGES; ++st) mbar_init(&full[st], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (tid == 0) {
    for (int k = 0; k < STAGES && k < ntiles; ++k) {
      const int64_t nb = c0 + (int64_t)k * TILE;
      mbar_arrive_expect_tx(&full[k], (uint32_t)(D * TILE * sizeof(float)));
#pragma unroll
      for (int j = 0; j < D; ++j)
        bulk_g2s(tiles + ((size_t)k * D + j) * TILE, a.cols + (int64_t)j * a.ld + nb, (uint32_t)(TILE * sizeof(float)),
                 &full[k]);
    }
  }
  if (tid < D) {
    const int j = tid;
    const float ap = a.consts->ap[j];
    const bool epan = a.consts->kernel == kEpanechnikov;
    const BoxDim bd = epan ? make_boxdim<kEpanechnikov>(__ldg(a.lo + j), __ldg(a.hi + j), ap, a.consts->renc[2 * j],
                                                         a.consts->renc[2 * j + 1])
                           : make_boxdim(__ldg(a.lo + j), __ldg(a.hi + j), ap, a.consts->renc[2 * j],
                                         a.consts->renc[2 * j + 1]);
    smc[j] = make_float4(bd.b.x, bd.b.y, bd.hd, ap);
    if (!epan && bd.hd > 0.0f) atomicOr(&narrow_s, 1);
  }
  __syncthreads();
  if (a.consts->kernel == kEpanechnikov)
    scan_single_tma_body<D, GRAD, 2, TILE, STAGES>(a, smc, tiles, full, c0, c1, ntiles);
  else if (narrow_s)
    scan_single_tma_body<D, GRAD, 1, TILE, STAGES>(a, smc, tiles, full, c0, c1, ntiles);
  else
    scan_single_tma_body<D, GRAD, 0, TILE, STAGES>(a, smc, tiles, full, c0, c1, ntiles);
}

template <int D, bool GRAD, int TILE, int STAGES, int OCC>
cudaError_t launch_single_tma_variant(const ScanSingleArgs& a, int grid, cudaStream_t s) {
  constexpr size_t smem = single_tma_smem_bytes<D, TILE, STAGES>();
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(scan_single_tma_kernel<D, GRAD, TILE, STAGES, OCC>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  scan_single_tma_kernel<D, GRAD, TILE, STAGES, OCC><<<grid, kSingleThreads, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace kde
