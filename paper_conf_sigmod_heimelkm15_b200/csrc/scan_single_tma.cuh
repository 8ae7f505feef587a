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
// compute warps of the culled variant (no producer warp); 16 at d = 9, 10 (one CTA per SM) measured
// slower than 8 (c5s 80.9 vs 76.5 us, profiles/r02_experiments.md)
#ifndef KDE_TUNE_CULL_WARPS
#define KDE_TUNE_CULL_WARPS(d) 8
#endif
__host__ __device__ constexpr int cull_warps(int d) { return KDE_TUNE_CULL_WARPS(d); }

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

// ---------------------------------------------------------------------------
// Tail culling (DESIGN.md §8 "culled single-box scan").  For a point t and box
// [l, u], let o_j = max(t_j - u_j, l_j - t_j, 0) sqrt(log2 e)/(sqrt2 h_j) be
// the distance OUTSIDE the box in dimension j in y' units (y'^2 = z^2 log2 e).
// Outside in dimension j, D_j <= 1/2 erfc(|z_j|) <= 1/2 e^{-z_j^2} = 2^{-o_j^2 - 1},
// so p^(i) = prod_j D_j <= 2^{-sum_j o_j^2}, and every gradient term
// |w_j| prod_{k!=j} D_k <= max(1.03, o_j) 2^{-sum_k o_k^2} <= 2^-61 once sum_k o_k^2 >= 64
// (pinned on the fp64 oracle by tests/test_oracle_pins.py::test_r15_cull_bound_against_oracle).
// A point with sum_j o_j^2 >= kCullY2 (64 + rounding slack) therefore changes p_hat
// by at most 2^-64 and each dp_hat/dh_j by at most 2^-60 * gconst_j per
// point: far below the fp32 rounding of the terms that are kept.  Such points
// are skipped (their retained p^(i) is written as 0); the others go through a
// per-warp ring of shared memory and are evaluated 64 at a time, so the
// expensive Phi evaluation (FMA + MUFU dispatch bound, §8) runs only on the
// points that can matter.  Points inside the box are never culled (o = 0), so
// the eq. (20) test (c >= the largest contribution of an outside point) sees
// every point it can flag.
constexpr int kCullRing = 128;   // queued points per warp (< 64 left + one 64-point classification chunk)
constexpr int kCullFlushChunks = 4;  // fp32 partials flushed to fp64 every 4 chunks (8 points per lane)

// st.shared.f32 under a predicate (no branch: culled lanes issue but do not store)
__device__ __forceinline__ void st_shared_if(uint32_t addr, float v, bool p) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q st.shared.f32 [%0], %1;\n\t}" ::"r"(addr), "f"(v),
      "r"((uint32_t)p)
      : "memory");
}

template <int D>
constexpr size_t cull_queue_bytes() {
  return (size_t)cull_warps(D) * kCullRing * (D + 1) * sizeof(float);
}

// d >= 9 gradient scans keep their fp64 per-thread sums in shared memory (stride kSingleThreads)
// instead of registers, so two CTAs fit per SM (register budget 96/thread at 288 x 2 threads)
#ifndef KDE_TUNE_RATIO_MIND
#define KDE_TUNE_RATIO_MIND 17  // from this d on: point_box2_ratio + smem sums (off: measured no gain at one CTA per SM)
#endif
template <int D, bool GRAD, bool CULL>
__host__ __device__ constexpr bool acc_in_smem() {
  return CULL && GRAD && D >= KDE_TUNE_RATIO_MIND;
}

template <int D, int TILE, int STAGES, bool CULL, bool GRAD = false>
constexpr size_t single_tma_kernel_smem() {
  return single_tma_smem_bytes<D, TILE, STAGES>() + (CULL ? cull_queue_bytes<D>() : 0) +
         (acc_in_smem<D, GRAD, CULL>() ? (size_t)(D + 1) * 32 * cull_warps(D) * sizeof(double) : 0);
}

template <int D, bool GRAD, int MODE, int TILE, int STAGES, typename Release>
__device__ __forceinline__ void scan_single_cull_body(const ScanSingleArgs& a, const float4* smc, const float2* scb,
                                                      float* tiles, uint64_t* full, Release& release, float* queue,
                                                      int64_t c0, int64_t c1, int ntiles, double* acc, bool keep_all) {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int NT = 32 * cull_warps(D);
  constexpr int AS = acc_in_smem<D, GRAD, true>() ? NT : 1;  // stride of acc (shared memory or registers)
  constexpr int PPT = TILE / NT;  // points per thread per tile
  static_assert(PPT % 2 == 0, "points are classified in pairs");
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  float* qt = queue + (size_t)warp * kCullRing * (D + 1);  // [D][kCullRing] coordinates
  int* qi = reinterpret_cast<int*>(qt + D * kCullRing);     // [kCullRing] point offset from c0
  // d >= 9: the box constants (5 d floats) are re-read from shared memory (broadcast) where they are
  // used instead of living in registers for the whole scan, which keeps wide gradient scans at two
  // CTAs per SM; narrower boxes keep them in registers.
#ifndef KDE_TUNE_RELOAD_MIND
#define KDE_TUNE_RELOAD_MIND 13  // from this d on: box constants re-read from shared memory (register budget)
#endif
  constexpr bool kReload = D >= KDE_TUNE_RELOAD_MIND;
  constexpr bool kRatio = D >= KDE_TUNE_RATIO_MIND;  // few-register gradient form (point_box2_ratio)
  BoxDim bd[D];
  float ap[D];
  float2 cb[D];  // (c ap, hw' ap) of the clamped box, for the classification
  auto load_box = [&]() {
#pragma unroll
    for (int j = 0; j < D; ++j) {
      const float4 c = smc[j];
      bd[j].b = make_float2(c.x, c.y);
      bd[j].hd = c.z;
      ap[j] = c.w;
    }
  };
  auto load_cb = [&]() {
#pragma unroll
    for (int j = 0; j < D; ++j) {
      cb[j] = scb[j];
      ap[j] = smc[j].w;
    }
  };
  if (!kReload) {
    load_box();
    load_cb();
  }
  const unsigned lt = (1u << lane) - 1u;
#if KDE_TUNE_L2KEEP
  const uint64_t pol_keep = l2_policy_evict_last();  // retained p^(i): read by the karma pass next
#endif
  unsigned head = 0, tail = 0;  // warp-uniform ring positions (head is a multiple of 64)
  int nproc = 0;
  float2 s[NA];
#pragma unroll
  for (int kk = 0; kk < NA; ++kk) s[kk] = f2(0.0f);

  // evaluate ring entries head + [0, 64): lane takes entries 2 lane, 2 lane + 1 (one LDS.64 per column)
  auto process = [&](int cnt) {
    if (kReload) load_box();
    const int e = (int)(head & (kCullRing - 1)) + 2 * lane;
    const bool v0 = 2 * lane < cnt, v1 = 2 * lane + 1 < cnt;
    float2 t[D];
#pragma unroll
    for (int j = 0; j < D; ++j) {
      const float2 q = *reinterpret_cast<const float2*>(qt + j * kCullRing + e);
      // stale ring slots may hold any bit pattern: replace them by a finite coordinate
      t[j] = make_float2(v0 ? q.x : bd[j].b.y, v1 ? q.y : bd[j].b.y);
    }
    const float2 vv = make_float2(v0 ? 1.0f : 0.0f, v1 ? 1.0f : 0.0f);
    float2 c;
    if constexpr (GRAD && kRatio)
      c = point_box2_ratio<D, MODE>(bd, t, ap, s, vv);
    else
      c = point_box2<D, GRAD, MODE>(bd, t, ap, s, vv);
    if (a.c_out) {
      const int2 ix = *reinterpret_cast<const int2*>(qi + e);
#if KDE_TUNE_L2KEEP
      if (v0) st_keep_f1(a.c_out + c0 + ix.x, c.x, pol_keep);
      if (v1) st_keep_f1(a.c_out + c0 + ix.y, c.y, pol_keep);
#else
      if (v0) __stcs(a.c_out + c0 + ix.x, c.x);
      if (v1) __stcs(a.c_out + c0 + ix.y, c.y);
#endif
    }
    head += 64;
    if (++nproc == kCullFlushChunks) {
#pragma unroll
      for (int kk = 0; kk < NA; ++kk) {
        acc[kk * AS] += (double)s[kk].x + (double)s[kk].y;
        s[kk] = f2(0.0f);
      }
      nproc = 0;
    }
  };

  for (int k = 0; k < ntiles; ++k) {
    const int st = k % STAGES;
    mbar_wait_parity(&full[st], (uint32_t)((k / STAGES) & 1));
    const float* tl = tiles + (size_t)st * D * TILE;
    const int64_t base = c0 + (int64_t)k * TILE;
    const int64_t rem = c1 - base;
    const int npts = rem < TILE ? (int)rem : TILE;
#pragma unroll 1
    for (int r = 0; r < PPT / 2; ++r) {
      const int pp = tid + r * NT;
      float2 t[D];
#pragma unroll
      for (int j = 0; j < D; ++j) t[j] = *reinterpret_cast<const float2*>(tl + j * TILE + 2 * pp);
      if (kReload) load_cb();
      // classification in scaled coordinates (make_cullbox / cull_score, phi.cuh)
      const float2 o2 = cull_score<D, MODE == 2>(t, ap, cb);
      const bool val0 = 2 * pp < npts, val1 = 2 * pp + 1 < npts;
      const bool al0 = val0 && (keep_all || o2.x < cull_limit<MODE == 2>()),
                 al1 = val1 && (keep_all || o2.y < cull_limit<MODE == 2>());
      if (a.c_out) {  // culled points retain 0; kept points are overwritten after evaluation (same warp, synced)
#if KDE_TUNE_L2KEEP
        if (val1)
          st_keep_f2(a.c_out + base + 2 * pp, f2(0.0f), pol_keep);
        else if (val0)
          st_keep_f1(a.c_out + base + 2 * pp, 0.0f, pol_keep);
#else
        if (val1)
          __stcs(reinterpret_cast<float2*>(a.c_out + base + 2 * pp), f2(0.0f));
        else if (val0)
          __stcs(a.c_out + base + 2 * pp, 0.0f);
#endif
      }
      __syncwarp();  // the previous chunk's ring reads are done before these writes
      // Branch-free compaction of the 64 candidates: the kept ones go to [tail, tail + nkeep)
      // (x halves, then y halves, in lane order) with predicated shared stores.
      const unsigned m0 = __ballot_sync(0xffffffffu, al0), m1 = __ballot_sync(0xffffffffu, al1);
      const int n0 = __popc(m0), nkeep = n0 + __popc(m1);
      const int off = (int)(base - c0) + 2 * pp;
      const uint32_t a0 = smem_u32(qt + ((tail + (unsigned)__popc(m0 & lt)) & (kCullRing - 1)));
      const uint32_t a1 = smem_u32(qt + ((tail + (unsigned)(n0 + __popc(m1 & lt))) & (kCullRing - 1)));
#pragma unroll
      for (int j = 0; j < D; ++j) {
        st_shared_if(a0 + j * kCullRing * 4, t[j].x, al0);
        st_shared_if(a1 + j * kCullRing * 4, t[j].y, al1);
      }
      if (a.c_out) {
        st_shared_if(a0 + D * kCullRing * 4, __int_as_float(off), al0);
        st_shared_if(a1 + D * kCullRing * 4, __int_as_float(off + 1), al1);
      }
      tail += (unsigned)nkeep;
      __syncwarp();
      while (tail - head >= 64u) process(64);
    }
    release(k);  // this warp is done reading stage st (the ring holds copies of the kept points)
  }
  if (tail != head) process((int)(tail - head));
#pragma unroll
  for (int kk = 0; kk < NA; ++kk) acc[kk * AS] += (double)s[kk].x + (double)s[kk].y;
}

// Culled variant: no producer warp -- the LAST compute warp to finish a tile's classification
// issues that stage's next TMA copies (per-stage arrival counters), so all 8 warps compute and
// the CTA's register budget allows two CTAs per SM at d >= 9.
template <int D, bool CULL>
__host__ __device__ constexpr int single_tma_threads() {
  return CULL ? 32 * cull_warps(D) : kSingleTmaThreads;
}

template <int D, bool GRAD, int TILE, int STAGES, int OCC, bool CULL>
__global__ void __launch_bounds__(single_tma_threads<D, CULL>(), OCC) scan_single_tma_kernel(const ScanSingleArgs a) {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int NT = single_tma_threads<D, CULL>();
  constexpr int NW = CULL ? cull_warps(D) : kSingleComputeWarps;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  float* tiles = reinterpret_cast<float*>(smem_raw);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + (size_t)STAGES * D * TILE * sizeof(float));
  uint64_t* empty = full + STAGES;
  float* queue = reinterpret_cast<float*>(smem_raw + single_tma_smem_bytes<D, TILE, STAGES>());
  __shared__ float4 smc[D];
  __shared__ float2 scb[D];
  __shared__ int narrow_s, nocull_s;
  __shared__ int rcnt[STAGES];  // culled variant: warps done with each stage
  const int tid = threadIdx.x;
  const bool producer = !CULL && tid >= kSingleThreads;
  // contiguous chunk of this CTA, a multiple of TILE points
  const int64_t ntile_total = (a.n + TILE - 1) / TILE;
  const int64_t tiles_per = (ntile_total + gridDim.x - 1) / gridDim.x;
  const int64_t c0 = (int64_t)blockIdx.x * tiles_per * TILE;
  const int64_t c1 = min(a.n, c0 + tiles_per * TILE);
  const int ntiles = c1 > c0 ? (int)((c1 - c0 + TILE - 1) / TILE) : 0;
  if (tid == 0) {
    narrow_s = 0;
    nocull_s = 0;
    for (int st = 0; st < STAGES; ++st) {
      mbar_init(&full[st], 1);
      mbar_init(&empty[st], kSingleComputeWarps);
      rcnt[st] = 0;
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int k) {  // tile k -> stage k % STAGES, completing on full[stage]
    const int st = k % STAGES;
    const int64_t nb = c0 + (int64_t)k * TILE;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    mbar_arrive_expect_tx(&full[st], (uint32_t)(D * TILE * sizeof(float)));
#if KDE_TUNE_L2KEEP
    if (a.c_out) {  // streaming step: the sample must not displace K and p^(i) from L2
      const uint64_t pol = l2_policy_evict_first();
#pragma unroll
      for (int j = 0; j < D; ++j)
        bulk_g2s_hint(tiles + ((size_t)st * D + j) * TILE, a.cols + (int64_t)j * a.ld + nb,
                      (uint32_t)(TILE * sizeof(float)), &full[st], pol);
      return;
    }
#endif
#pragma unroll
    for (int j = 0; j < D; ++j)
      bulk_g2s(tiles + ((size_t)st * D + j) * TILE, a.cols + (int64_t)j * a.ld + nb, (uint32_t)(TILE * sizeof(float)),
               &full[st]);
  };
  if (CULL && tid == 0)
    for (int k = 0; k < STAGES && k < ntiles; ++k) issue(k);
  auto release = [&](int k) {  // last warp out of tile k refills its stage with tile k + STAGES
    __syncwarp();
    if ((tid & 31) == 0) {
      const int st = k % STAGES;
      __threadfence_block();
      if (atomicAdd(&rcnt[st], 1) == NW - 1) {
        rcnt[st] = 0;
        if (k + STAGES < ntiles) issue(k + STAGES);
      }
    }
  };
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
    if (CULL) {
      scb[j] = make_cullbox(__ldg(a.lo + j), __ldg(a.hi + j), ap, a.consts->renc[2 * j], a.consts->renc[2 * j + 1]);
      if (!cullbox_ok(scb[j])) atomicOr(&nocull_s, 1);
    }
  }
  __syncthreads();
  double acc[NA];
#pragma unroll
  for (int k = 0; k < NA; ++k) acc[k] = 0.0;
  constexpr bool kAccSh = acc_in_smem<D, GRAD, CULL>();
  double* accsh = reinterpret_cast<double*>(smem_raw + single_tma_smem_bytes<D, TILE, STAGES>() +
                                            (CULL ? cull_queue_bytes<D>() : 0)) + tid;
  if (kAccSh && !producer)
#pragma unroll
    for (int k = 0; k < NA; ++k) accsh[k * NT] = 0.0;
  double* accp = (kAccSh && !producer) ? accsh : acc;
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
  } else if (CULL && a.consts->kernel == kEpanechnikov) {
    scan_single_cull_body<D, GRAD, 2, TILE, STAGES>(a, smc, scb, tiles, full, release, queue, c0, c1, ntiles, accp,
                                                    nocull_s != 0);
  } else if (a.consts->kernel == kEpanechnikov) {
    scan_single_tma_body<D, GRAD, 2, TILE, STAGES>(a, smc, tiles, full, empty, c0, c1, ntiles, acc);
  } else if (CULL) {
    if (narrow_s)
      scan_single_cull_body<D, GRAD, 1, TILE, STAGES>(a, smc, scb, tiles, full, release, queue, c0, c1, ntiles, accp,
                                                      nocull_s != 0);
    else
      scan_single_cull_body<D, GRAD, 0, TILE, STAGES>(a, smc, scb, tiles, full, release, queue, c0, c1, ntiles, accp,
                                                      nocull_s != 0);
  } else if (narrow_s) {
    scan_single_tma_body<D, GRAD, 1, TILE, STAGES>(a, smc, tiles, full, empty, c0, c1, ntiles, acc);
  } else {
    scan_single_tma_body<D, GRAD, 0, TILE, STAGES>(a, smc, tiles, full, empty, c0, c1, ntiles, acc);
  }
  if (kAccSh && !producer)
#pragma unroll
    for (int k = 0; k < NA; ++k) acc[k] = accsh[k * NT];
  single_reduce_finalize<NA, NT>(a, acc);
}

template <int D, bool GRAD, int TILE, int STAGES, int OCC, bool CULL>
cudaError_t launch_single_tma_variant(const ScanSingleArgs& a, int grid, cudaStream_t s) {
  constexpr size_t smem = single_tma_kernel_smem<D, TILE, STAGES, CULL, GRAD>();
  static_assert(smem + 1024 <= 227 * 1024, "single-box scan shared memory");
  // the attribute belongs to the device context: set it once per device (bit per ordinal)
  static std::atomic<unsigned long long> attr_set{0ull};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const unsigned long long bit = 1ull << (dev & 63);
  if (!(attr_set.load(std::memory_order_acquire) & bit)) {
    e = cudaFuncSetAttribute(scan_single_tma_kernel<D, GRAD, TILE, STAGES, OCC, CULL>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set.fetch_or(bit, std::memory_order_acq_rel);
  }
  scan_single_tma_kernel<D, GRAD, TILE, STAGES, OCC, CULL><<<grid, single_tma_threads<D, CULL>(), smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace kde
