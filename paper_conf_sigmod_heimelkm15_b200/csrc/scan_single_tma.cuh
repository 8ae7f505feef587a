// scan_single_tma.cuh -- single-box scan with the sample streamed through
// shared memory by TMA bulk copies (included at the end of scan.cuh).
//
// Warp-specialised pipeline.  Each CTA owns a contiguous chunk of the sample
// and walks it in tiles of TILE points x d columns held in a ring of STAGES
// shared-memory stages.  A ninth (producer) warp keeps the ring full: for each
// tile it waits until the stage is EMPTY (an mbarrier every compute warp
// arrives on after its last read), then issues the d cp.async.bulk copies that
// complete on the stage's FULL mbarrier (expect_tx).  The 8 compute warps only
// wait on FULL and never on each other -- there is no CTA-wide barrier in the
// tile loop, so warps drift out of phase and the FMA and MUFU pipes see a
// mixed instruction stream instead of synchronised bursts.
#pragma once

namespace kde {

constexpr int kSingleComputeWarps = kSingleThreads / 32;
constexpr int kSingleTmaThreads = kSingleThreads + 32;  // + producer warp

template <int D, int TILE, int STAGES>
constexpr size_t single_tma_smem_bytes() {
  return (size_t)STAGES * D * TILE * sizeof(float) + 2 * STAGES * sizeof(uint64_t);
}

template <int D, bool GRAD, int MODE, int TILE, int STAGES>
__device__ __forceinline__ void scan_single_tma_body(const ScanSingleArgs& a, const float4* smc, float* tiles,
                                                     uint64_t* full, uint64_t* empty, int64_t c0, int64_t c1,
                                                     int ntiles, double* acc) {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int PPT = TILE / kSingleThreads;  // points per thread per tile
  static_assert(PPT % 2 == 0, "points are processed in pairs");
  const int tid = threadIdx.x;
  BoxDim bd[D];
  float ap[D];
#pragma unroll
  for (int j = 0; j < D; ++j) {
    const float4 c = smc[j];
    bd[j].b = make_float2(c.x, c.y);
    bd[j].hd = c.z;
    ap[j] = c.w;
  }
  for (int k = 0; k < ntiles; ++k) {
    const int st = k % STAGES;
    mbar_wait_parity(&full[st], (uint32_t)((k / STAGES) & 1));
    const float* tl = tiles + (size_t)st * D * TILE;
    const int64_t base = c0 + (int64_t)k * TILE;
    const int64_t rem = c1 - base;
    const int npts = rem < TILE ? (int)rem : TILE;
    float2 s[NA];
#pragma unroll
    for (int kk = 0; kk < NA; ++kk) s[kk] = f2(0.0f);
    // point pairs (2pp, 2pp + 1), pp = tid + r * threads: one LDS.64 per column and pair
#pragma unroll
    for (int r = 0; r < PPT / 2; ++r) {
      const int pp = tid + r * kSingleThreads;
      float2 t[D];
#pragma unroll
      for (int j = 0; j < D; ++j) t[j] = *reinterpret_cast<const float2*>(tl + j * TILE + 2 * pp);
      const float2 valid = make_float2(2 * pp < npts ? 1.0f : 0.0f, 2 * pp + 1 < npts ? 1.0f : 0.0f);
      const float2 c = point_box2<D, GRAD, MODE>(bd, t, ap, s, valid);
      if (a.c_out) {
        if (2 * pp + 1 < npts)
          __stcs(reinterpret_cast<float2*>(a.c_out + base + 2 * pp), c);
        else if (2 * pp < npts)
          __stcs(a.c_out + base + 2 * pp, c.x);
      }
    }
    __syncwarp();
    if ((tid & 31) == 0) mbar_arrive(&empty[st]);  // this warp is done reading stage st
#pragma unroll
    for (int kk = 0; kk < NA; ++kk) acc[kk] += (double)s[kk].x + (double)s[kk].y;
  }
}

template <int D, bool GRAD, int TILE, int STAGES, int OCC>
__global__ void __launch_bounds__(kSingleTmaThreads, OCC) scan_single_tma_kernel(const ScanSingleArgs a) {
  constexpr int NA = GRAD ? D + 1 : 1;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  float* tiles = reinterpret_cast<float*>(smem_raw);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + (size_t)STAGES * D * TILE * sizeof(float));
  uint64_t* empty = full + STAGES;
  __shared__ float4 smc[D];
  __shared__ int narrow_s;
  const int tid = threadIdx.x;
  const bool producer = tid >= kSingleThreads;
  // contiguous chunk of this CTA, a multiple of TILE points
  const int64_t ntile_total = (a.n + TILE - 1) / TILE;
  const int64_t tiles_per = (ntile_total + gridDim.x - 1) / gridDim.x;
  const int64_t c0 = (int64_t)blockIdx.x * tiles_per * TILE;
  const int64_t c1 = min(a.n, c0 + tiles_per * TILE);
  const int ntiles = c1 > c0 ? (int)((c1 - c0 + TILE - 1) / TILE) : 0;
  if (tid == 0) {
    narrow_s = 0;
    for (int st = 0; st < STAGES; ++st) {
      mbar_init(&full[st], 1);
      mbar_init(&empty[st], kSingleComputeWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
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
  double acc[NA];
#pragma unroll
  for (int k = 0; k < NA; ++k) acc[k] = 0.0;
  if (producer) {
    if (tid == kSingleThreads) {
      for (int k = 0; k < ntiles; ++k) {
        const int st = k % STAGES;
        if (k >= STAGES) mbar_wait_parity(&empty[st], (uint32_t)((k / STAGES - 1) & 1));
        const int64_t nb = c0 + (int64_t)k * TILE;
        mbar_arrive_expect_tx(&full[st], (uint32_t)(D * TILE * sizeof(float)));
#pragma unroll
        for (int j = 0; j < D; ++j)
          bulk_g2s(tiles + ((size_t)st * D + j) * TILE, a.cols + (int64_t)j * a.ld + nb,
                   (uint32_t)(TILE * sizeof(float)), &full[st]);
      }
    }
  } else if (a.consts->kernel == kEpanechnikov) {
    scan_single_tma_body<D, GRAD, 2, TILE, STAGES>(a, smc, tiles, full, empty, c0, c1, ntiles, acc);
  } else if (narrow_s) {
    scan_single_tma_body<D, GRAD, 1, TILE, STAGES>(a, smc, tiles, full, empty, c0, c1, ntiles, acc);
  } else {
    scan_single_tma_body<D, GRAD, 0, TILE, STAGES>(a, smc, tiles, full, empty, c0, c1, ntiles, acc);
  }
  single_reduce_finalize<NA, kSingleTmaThreads>(a, acc);
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
  scan_single_tma_kernel<D, GRAD, TILE, STAGES, OCC><<<grid, kSingleTmaThreads, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace kde
