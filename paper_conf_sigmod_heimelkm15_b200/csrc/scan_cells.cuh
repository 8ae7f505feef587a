// scan_cells.cuh -- the culled batched scan over the spatially ordered copy of the sample
// (reading R17; included by scan.cuh, which provides the TMA / mbarrier helpers, point_box2 and
// the cull helpers of phi.cuh).
//
// Per box the scan computes the same sums as scan_batched_kernel (eq. 2 + 13 and the eq. 17 terms,
// P:L98), skipping (point, box) pairs whose contribution is provably below 2^-64
// (reading R15).  The work is organised the other way round from the unordered batched scan: the
// LANES of a warp are points, the warp holds one box at a time.
//
//  * cells (cells.cu): kCellPts consecutive points of the Morton-ordered copy with their bounding
//    box.  Per cell and box one test on the bounding box classifies the pair as
//      skip    -- every point of the cell is >= 8 scaled bandwidths outside the box (R15 holds for
//                 each of them: the cell is not touched at all),
//      full    -- every point lies inside the kept region: all points are evaluated, no
//                 per-point classification,
//      partial -- per-point classification (cull_score, as the other scans), then the kept points
//                 are evaluated -- compacted into a per-warp index list when few, masked when many.
//  * grid: (nsplit, ngroups).  Group g owns the boxes at probe-sorted positions g, g + ngroups, ...
//    (dealt, so every group and every warp gets a similar mix of cheap and expensive boxes); the
//    CTA streams the cells split, split + nsplit, ... (strided over the whole curve, so every CTA
//    sees every region of the data) through a TMA ring, as the batched scan.
//  * ownership: slot i of the group belongs to warp i mod 8, so one warp adds every contribution
//    of a box, in cell order: per (cell, box) item the lanes' fp32 sums (<= 8 points each) are
//    reduced by a fixed butterfly and added into the box's fp64 accumulator in shared memory.
//    Results are therefore deterministic (bitwise repeatable), independent of scheduling.
//  * the (split, box) accumulators go to partials[split][comp][q] and are summed in split order
//    by reduce_splits_kernel (kernels.cu), exactly as for the unordered batched scan.
#pragma once

namespace kde {

static_assert(kCellPts == kTilePts, "cells are the batched scan's tiles");
constexpr int kCellsThreads = 256;
constexpr int kCellsWarps = kCellsThreads / 32;

template <int D>
struct CellsK {  // boxes per lane of a warp's slot set (QG = 256 K boxes per CTA)
#ifdef KDE_TUNE_CELLS_K
  static constexpr int value = KDE_TUNE_CELLS_K;
#else
  static constexpr int value = 1;
#endif
};
template <int D>
struct CellsMinB {
#ifdef KDE_TUNE_CELLS_MINB
  static constexpr int value = KDE_TUNE_CELLS_MINB;
#else
  static constexpr int value = D <= 6 ? 4 : (D <= 12 ? 2 : 1);
#endif
};
__host__ __device__ constexpr int cells_stages(int d) {
#ifdef KDE_TUNE_CELLS_STAGES
  return (void)d, KDE_TUNE_CELLS_STAGES;
#else
  return d <= 8 ? 3 : 2;
#endif
}
// CTAs per resident slot (waves): several smaller CTAs per SM slot even out the work of the
// strided cell sets and box groups (the hardware starts a new CTA where one finished)
#ifndef KDE_TUNE_CELLS_WAVES
#define KDE_TUNE_CELLS_WAVES 32
#endif
// point pairs per lane and iteration of a full item (kCellPts / 64 must be a multiple)
#ifndef KDE_TUNE_CELLS_PU
#define KDE_TUNE_CELLS_PU 1
#endif
// an item with more kept points than this is evaluated masked (no compaction)
#ifndef KDE_TUNE_CELLS_DENSE
#define KDE_TUNE_CELLS_DENSE 160
#endif
template <int D>
__host__ __device__ constexpr int cells_qg() {
  return kCellsThreads * CellsK<D>::value;
}

template <int D, bool GRAD>
constexpr size_t cells_smem_bytes() {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int QG = cells_qg<D>();
  return (size_t)cells_stages(D) * D * kCellPts * sizeof(float)  // tile ring
         + (size_t)QG * D * sizeof(float4)                     // (b.x, b.y, cb.x, cb.y) per box and dim
         + (size_t)QG * NA * sizeof(double)                    // fp64 accumulators
         + (size_t)cells_stages(D) * (sizeof(uint64_t) + sizeof(int))  // full barriers, arrival counters
         + (size_t)QG * sizeof(unsigned)                       // per-box flags
         + (size_t)kCellsWarps * kCellPts;                     // per-warp kept-point lists (uint8)
}

constexpr unsigned kCellsKeepAll = 1u << 31;  // box not representable in scaled fp32: no culling
constexpr unsigned kCellsEmpty = 1u << 30;    // slot beyond q

// Sum NA per-lane values over the warp and add component k to acc[k]: a reduce-scatter butterfly
// (P = NA rounded up to a power of two; at the level with offset o a lane keeps the half of its
// values selected by lane bit o and receives the partner's copy of that half), P - 1 + 5 - log2 P
// shuffles instead of 5 NA.  Afterwards lane k << (5 - log2 P) holds component k.  Fixed order.
template <int NA>
__device__ __forceinline__ void warp_sum_scatter(const float (&v)[NA], double* acc, int lane) {
  constexpr int P = NA <= 1 ? 1 : NA <= 2 ? 2 : NA <= 4 ? 4 : NA <= 8 ? 8 : NA <= 16 ? 16 : 32;
  constexpr int LP = P == 1 ? 0 : P == 2 ? 1 : P == 4 ? 2 : P == 8 ? 3 : P == 16 ? 4 : 5;
  static_assert(NA <= 32, "at most 32 components");
  float w[P];
#pragma unroll
  for (int k = 0; k < P; ++k) w[k] = k < NA ? v[k] : 0.0f;
#pragma unroll
  for (int lev = 0; lev < LP; ++lev) {
    const int half = P >> (lev + 1);
    const int o = 16 >> lev;
    const bool up = (lane & o) != 0;
#pragma unroll
    for (int i = 0; i < half; ++i) {
      const float send = up ? w[i] : w[i + half];
      const float keep = up ? w[i + half] : w[i];
      w[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
    }
  }
  float r = w[0];
#pragma unroll
  for (int o = 16 >> LP; o > 0; o >>= 1) r += __shfl_xor_sync(0xffffffffu, r, o);
  const int k = lane >> (5 - LP);
  if ((lane & ((1 << (5 - LP)) - 1)) == 0 && k < NA) acc[k] += (double)r;
}

// Shared-memory loads the compiler may not hoist out of the item's loops: the box constants are
// re-read (broadcast) where they are used instead of occupying D x 5 registers across the item.
#ifndef KDE_TUNE_CELLS_RELOAD
#define KDE_TUNE_CELLS_RELOAD 1
#endif
__device__ __forceinline__ float4 cells_lds4(const float4* p) {
#if KDE_TUNE_CELLS_RELOAD
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "r"(static_cast<uint32_t>(__cvta_generic_to_shared(p))));
  return v;
#else
  return *p;
#endif
}
__device__ __forceinline__ float cells_lds1(const float* p) {
#if KDE_TUNE_CELLS_RELOAD
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(static_cast<uint32_t>(__cvta_generic_to_shared(p))));
  return v;
#else
  return *p;
#endif
}
// Box table entry per dimension: (b.x, b.y, cb.x, cb.y).  A narrow dimension (MODE 1, bit j of nm)
// has b = (l, l) and keeps its half-width hd in the .y slot; an Epanechnikov dimension (MODE 2)
// recomputes Delta = (b.x - b.y) ap -- the same fp32 operations as make_boxdim when the bounds are
// not clamped, and unused by phi_epan2 when they are (every point is then >= 2h outside the
// clamped bound, so |v| > 1 and the clamped difference is taken).
template <int D, int MODE>
__device__ __forceinline__ void cells_boxdims(const float4* tb, const float (&ap)[D], unsigned nm, BoxDim (&bd)[D]) {
#pragma unroll
  for (int j = 0; j < D; ++j) {
    const float4 v = cells_lds4(tb + j);
    if (MODE == 1 && ((nm >> j) & 1u)) {
      bd[j].b = make_float2(v.x, v.x);
      bd[j].hd = v.y;
    } else {
      bd[j].b = make_float2(v.x, v.y);
      bd[j].hd = MODE == 2 ? (v.x - v.y) * ap[j] : 0.0f;
    }
  }
}

// One (box, cell) item: the lanes hold point pairs.  Adds the item's sums into acc[0..NA) and
// returns the number of points evaluated (all of a full cell, the kept ones of a partial cell).
template <int D, bool GRAD, int MODE>
__device__ __forceinline__ int cells_item(const float* tl, int npts, bool full, const float4* tb,
                                           unsigned nm, const float (&ap)[D], double* acc, unsigned char* list,
                                           int lane) {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr bool EPAN = MODE == 2;
  float2 s[NA];
#pragma unroll
  for (int k = 0; k < NA; ++k) s[k] = f2(0.0f);
  constexpr int kRounds = kCellPts / 64;  // point pairs per lane
  const int rounds = (npts + 63) >> 6;
  int ev = npts;
  if (full) {
    for (int r = 0; r < rounds; r += KDE_TUNE_CELLS_PU) {  // PU independent pairs per iteration (ILP)
#pragma unroll
      for (int u = 0; u < KDE_TUNE_CELLS_PU; ++u) {
        const int p = 64 * (r + u) + 2 * lane;  // p < kCellPts always: the padding is finite (zeros)
        float2 t[D];
#pragma unroll
        for (int j = 0; j < D; ++j) t[j] = *reinterpret_cast<const float2*>(tl + j * kCellPts + p);
        BoxDim bd[D];
        cells_boxdims<D, MODE>(tb, ap, nm, bd);
        point_box2<D, GRAD, MODE>(bd, t, ap, s, make_float2(p < npts ? 1.0f : 0.0f, p + 1 < npts ? 1.0f : 0.0f));
      }
    }
  } else {
    // classification: bit 2r (2r + 1) of kb = point 64 r + 2 lane (+ 1) is kept
    unsigned kb = 0u;
#pragma unroll
    for (int r = 0; r < kRounds; ++r) {
      if (r < rounds) {
        const int p = 64 * r + 2 * lane;
        float2 t[D];
#pragma unroll
        for (int j = 0; j < D; ++j) t[j] = *reinterpret_cast<const float2*>(tl + j * kCellPts + p);
        float2 cb[D];
#pragma unroll
        for (int j = 0; j < D; ++j) {
          const float4 v = cells_lds4(tb + j);
          cb[j] = make_float2(v.z, v.w);
        }
        const float2 u = __fadd2_rn(cull_score<D, EPAN>(t, ap, cb), f2(-cull_limit<EPAN>()));
        kb |= ((__float_as_uint(u.x) >> 31) & (p < npts ? 1u : 0u)) << (2 * r);
        kb |= ((__float_as_uint(u.y) >> 31) & (p + 1 < npts ? 1u : 0u)) << (2 * r + 1);
      }
    }
    const int m = (int)__reduce_add_sync(0xffffffffu, (unsigned)__popc(kb));
    if (m == 0) return 0;
    ev = m;
    if (m > KDE_TUNE_CELLS_DENSE) {  // many kept: masked evaluation of the rounds that hold any
      for (int r = 0; r < rounds; ++r) {
        const unsigned v = (kb >> (2 * r)) & 3u;
        if (!__any_sync(0xffffffffu, v != 0u)) continue;
        const int p = 64 * r + 2 * lane;
        float2 t[D];
#pragma unroll
        for (int j = 0; j < D; ++j) t[j] = *reinterpret_cast<const float2*>(tl + j * kCellPts + p);
        BoxDim bd[D];
        cells_boxdims<D, MODE>(tb, ap, nm, bd);
        point_box2<D, GRAD, MODE>(bd, t, ap, s, make_float2((float)(v & 1u), (float)(v >> 1)));
      }
    } else {  // few kept: compact their indices (round-major, lane order), evaluate 64 at a time
      const unsigned lt = (1u << lane) - 1u;
      int base = 0;
#pragma unroll
      for (int r = 0; r < kRounds; ++r) {
        const unsigned k0 = (kb >> (2 * r)) & 1u, k1 = (kb >> (2 * r + 1)) & 1u;
        const unsigned b0 = __ballot_sync(0xffffffffu, k0), b1 = __ballot_sync(0xffffffffu, k1);
        const int pos = base + __popc(b0 & lt) + __popc(b1 & lt);
        if (k0) list[pos] = (unsigned char)(64 * r + 2 * lane);
        if (k1) list[pos + (int)k0] = (unsigned char)(64 * r + 2 * lane + 1);
        base += __popc(b0) + __popc(b1);
      }
      __syncwarp();
      for (int g0 = 0; g0 < m; g0 += 64) {
        const int e0 = g0 + 2 * lane;
        const bool v0 = e0 < m, v1 = e0 + 1 < m;
        const int i0 = v0 ? list[e0] : 0, i1 = v1 ? list[e0 + 1] : i0;
        float2 t[D];
#pragma unroll
        for (int j = 0; j < D; ++j) t[j] = make_float2(tl[j * kCellPts + i0], tl[j * kCellPts + i1]);
        BoxDim bd[D];
        cells_boxdims<D, MODE>(tb, ap, nm, bd);
        point_box2<D, GRAD, MODE>(bd, t, ap, s, make_float2(v0 ? 1.0f : 0.0f, v1 ? 1.0f : 0.0f));
      }
      __syncwarp();  // the list is rewritten by the next item
    }
  }
  // fixed reduce-scatter over the lanes, then one fp64 add per component (deterministic)
  float v[NA];
#pragma unroll
  for (int k = 0; k < NA; ++k) v[k] = s[k].x + s[k].y;
  warp_sum_scatter<NA>(v, acc, lane);
  return ev;
}

template <int D, bool GRAD>
__global__ void __launch_bounds__(kCellsThreads, CellsMinB<D>::value) scan_cells_kernel(const ScanCellsArgs a) {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int K = CellsK<D>::value;
  constexpr int QG = cells_qg<D>();
  constexpr int S = cells_stages(D);
  extern __shared__ __align__(16) unsigned char smem_raw[];
  float* tile = reinterpret_cast<float*>(smem_raw);                           // [S][D][kCellPts]
  float4* tab = reinterpret_cast<float4*>(tile + (size_t)S * D * kCellPts);  // [QG][D]
  double* acc = reinterpret_cast<double*>(tab + (size_t)QG * D);             // [QG][NA]
  uint64_t* bar = reinterpret_cast<uint64_t*>(acc + (size_t)QG * NA);       // [S]
  int* cnt = reinterpret_cast<int*>(bar + S);                                // [S]
  unsigned* flags = reinterpret_cast<unsigned*>(cnt + S);                    // [QG]
  unsigned char* lists = reinterpret_cast<unsigned char*>(flags + QG);       // [warps][kCellPts]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // x = box group, y = cell set: the groups of one cell set are launched together and share its
  // tiles through L2 (the sample is read from HBM about once, not once per group)
  const int g = blockIdx.x, ngroups = gridDim.x;
  const int split = blockIdx.y, nsplit = gridDim.y;

  float ap[D];
#pragma unroll
  for (int j = 0; j < D; ++j) ap[j] = a.consts->ap[j];
  const bool epan = a.consts->kernel == kEpanechnikov;

  // box setup: slot i <-> probe-sorted position g + ngroups * i
  for (int i = tid; i < QG; i += kCellsThreads) {
    const int64_t pos = (int64_t)g + (int64_t)ngroups * i;
    unsigned f = 0u;
    if (pos < a.q) {
      const int64_t qi = a.perm ? a.perm[pos] : pos;
#pragma unroll
      for (int j = 0; j < D; ++j) {
        const float l = __ldg(a.lo + qi * D + j), u = __ldg(a.hi + qi * D + j);
        const unsigned rmin = a.consts->renc[2 * j], rmax = a.consts->renc[2 * j + 1];
        const BoxDim bd = epan ? make_boxdim<kEpanechnikov>(l, u, ap[j], rmin, rmax) : make_boxdim(l, u, ap[j], rmin, rmax);
        const float2 cb = make_cullbox(l, u, ap[j], rmin, rmax);
        const bool nar = !epan && bd.hd > 0.0f;
        tab[i * D + j] = make_float4(bd.b.x, nar ? bd.hd : bd.b.y, cb.x, cb.y);  // see cells_boxdims
        if (nar) f |= 1u << j;
        if (!cullbox_ok(cb)) f |= kCellsKeepAll;
      }
    } else {
      f = kCellsEmpty;
    }
    flags[i] = f;
#pragma unroll
    for (int k = 0; k < NA; ++k) acc[(size_t)i * NA + k] = 0.0;
  }

  const int ntiles = split < a.ncells ? (int)((a.ncells - 1 - split) / nsplit + 1) : 0;
  if (tid == 0) {
    for (int st = 0; st < S; ++st) {
      mbar_init(&bar[st], 1);
      cnt[st] = 0;
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int k) {
    const int buf = k % S;
    const int64_t cell = split + (int64_t)k * nsplit;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    mbar_arrive_expect_tx(&bar[buf], (uint32_t)(D * kCellPts * sizeof(float)));
#pragma unroll
    for (int j = 0; j < D; ++j)
      bulk_g2s(tile + ((size_t)buf * D + j) * kCellPts, a.ccols + (int64_t)j * a.ld + cell * kCellPts,
               (uint32_t)(kCellPts * sizeof(float)), &bar[buf]);
  };
  if (tid == 0)
    for (int k = 0; k < S && k < ntiles; ++k) issue(k);

  unsigned char* list = lists + warp * kCellPts;
  constexpr float kEps = 1.0f / (1 << 20);  // rounding margin of the scaled bounding-box test
  float apj = ap[0];  // lane j < D: dimension j's scale
#pragma unroll
  for (int j = 1; j < D; ++j) apj = lane == j ? ap[j] : apj;
  const float2* cbb2 = reinterpret_cast<const float2*>(a.cbb);
  float2 bbn = make_float2(0.0f, 0.0f);  // the next cell's bounding box (lane j: dimension j), prefetched
  if (lane < D && ntiles > 0) bbn = __ldg(cbb2 + (int64_t)split * D + lane);
  __shared__ unsigned long long wstats[4 * kCellsWarps];  // a.stats (profiling)
  if (lane < 4) wstats[4 * warp + lane] = 0ull;
  __syncwarp();
  for (int k = 0; k < ntiles; ++k) {
    const int st = k % S;
    const int64_t cell = split + (int64_t)k * nsplit;
    const int npts = (int)min((int64_t)kCellPts, a.n - cell * kCellPts);
    // the cell's bounding box in scaled coordinates: centre cc, half-width chw (lane j holds dim j)
    const float2 bb = bbn;
    if (lane < D && k + 1 < ntiles) bbn = __ldg(cbb2 + (cell + nsplit) * D + lane);
    const float ccj = fmaf(0.5f, bb.x, 0.5f * bb.y) * apj;  // no overflow of bb.x + bb.y
    const float chwj = (0.5f * bb.y - 0.5f * bb.x) * apj;
    float cc[D], chw[D];
#pragma unroll
    for (int j = 0; j < D; ++j) {
      cc[j] = __shfl_sync(0xffffffffu, ccj, j);
      chw[j] = __shfl_sync(0xffffffffu, chwj, j);
    }
    // classify this warp's boxes against the cell (lane owns slots warp + 8 (lane + 32 kk))
    unsigned alive[K], fullm[K];
#pragma unroll
    for (int kk = 0; kk < K; ++kk) {
      const int slot = warp + kCellsWarps * (lane + 32 * kk);
      const unsigned f = flags[slot];
      float o2 = 0.0f, O2 = 0.0f;
#pragma unroll
      for (int j = 0; j < D; ++j) {
        const float4 tb = tab[slot * D + j];
        const float dc = fabsf(cc[j] - tb.z);
        const float err = kEps * (fabsf(cc[j]) + chw[j] + fabsf(tb.z) + tb.w);
        const float near = dc - chw[j] - tb.w - err;  // <= the smallest distance outside the box
        const float far = dc + chw[j] - tb.w;         // ~ the largest distance outside the box
        if (epan) {
          o2 = fmaxf(o2, near);
          O2 = fmaxf(O2, far);
        } else {
          const float nr = fmaxf(near, 0.0f), fr = fmaxf(far, 0.0f);
          o2 = fmaf(nr, nr, o2);
          O2 = fmaf(fr, fr, O2);
        }
      }
      const bool keep_all = (f & kCellsKeepAll) != 0u;
      const bool skip = (f & kCellsEmpty) != 0u || (!keep_all && (epan ? o2 >= 1.0f : o2 >= kCullY2));
      const bool isfull = !skip && (keep_all || (epan ? O2 < 1.0f : O2 < kCullY2));  // every point kept
      alive[kk] = __ballot_sync(0xffffffffu, !skip);
      fullm[kk] = __ballot_sync(0xffffffffu, isfull);
    }
    mbar_wait_parity_suspend(&bar[st], (uint32_t)((k / S) & 1));
    const float* tl = tile + (size_t)st * D * kCellPts;
#pragma unroll
    for (int kk = 0; kk < K; ++kk) {
      unsigned al = alive[kk];
      while (al) {
        const int b = __ffs(al) - 1;
        al &= al - 1u;
        const int slot = warp + kCellsWarps * (b + 32 * kk);
        const bool fl = (fullm[kk] >> b) & 1u;
        const unsigned f = flags[slot];
        const float4* tb = tab + slot * D;
        double* ac = acc + (size_t)slot * NA;
        int ev;
        if (epan)
          ev = cells_item<D, GRAD, 2>(tl, npts, fl, tb, f, ap, ac, list, lane);
        else if (f & ((1u << D) - 1u))
          ev = cells_item<D, GRAD, 1>(tl, npts, fl, tb, f, ap, ac, list, lane);
        else
          ev = cells_item<D, GRAD, 0>(tl, npts, fl, tb, f, ap, ac, list, lane);
        if (a.stats && lane == 0) {  // per-warp counters in shared memory (no registers held)
          unsigned long long* c4 = wstats + 4 * warp;
          c4[0] += 1;
          c4[1] += fl ? 1 : 0;
          c4[2] += (unsigned long long)ev;
          c4[3] += fl ? 0 : (unsigned long long)npts;
        }
      }
    }
    __syncwarp();
    if (lane == 0) {
      __threadfence_block();  // this warp's reads of the stage precede its arrival
      if (atomicAdd(&cnt[st], 1) == kCellsWarps - 1) {
        cnt[st] = 0;
        if (k + S < ntiles) issue(k + S);
      }
    }
  }
  if (a.stats && lane < 4) atomicAdd(a.stats + lane, wstats[4 * warp + lane]);  // per-warp totals
  __syncthreads();
  // partials row entry g * QG + slot: consecutive threads write consecutive doubles (the reduction
  // maps entries back to boxes, reduce_splits_mapped)
  for (int i = tid; i < QG; i += kCellsThreads) {
    const int64_t pos = (int64_t)g + (int64_t)ngroups * i;
    if (pos >= a.q) continue;
#pragma unroll
    for (int k = 0; k < NA; ++k)
      a.partials[((int64_t)split * NA + k) * a.qpad + (int64_t)g * QG + i] = acc[(size_t)i * NA + k];
  }
}

template <int D, bool GRAD>
cudaError_t launch_cells_tg(const ScanCellsArgs& a, dim3 grid, cudaStream_t s) {
  constexpr size_t smem = cells_smem_bytes<D, GRAD>();
  static_assert(smem <= 227 * 1024, "scan_cells_kernel shared memory");
  static std::atomic<unsigned long long> attr_set{0ull};  // per device ordinal
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const unsigned long long bit = 1ull << (dev & 63);
  if (!(attr_set.load(std::memory_order_acquire) & bit)) {
    e = cudaFuncSetAttribute(scan_cells_kernel<D, GRAD>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set.fetch_or(bit, std::memory_order_acq_rel);
  }
  scan_cells_kernel<D, GRAD><<<grid, kCellsThreads, smem, s>>>(a);
  return cudaGetLastError();
}

// grid: ngroups = ceil(q / QG) box groups x nsplit strided cell sets, KDE_TUNE_CELLS_WAVES waves of MINB CTAs per SM
template <int D>
cudaError_t launch_cells_t(bool grad, const ScanCellsArgs& a, int num_sms, int* splits_out, cudaStream_t s,
                           bool dry_run) {
  constexpr int QG = cells_qg<D>();
  const int64_t ngroups = (a.q + QG - 1) / QG;
  if (ngroups > 0x7fffffff) return cudaErrorInvalidValue;
  int64_t nsplit = ((int64_t)num_sms * CellsMinB<D>::value * KDE_TUNE_CELLS_WAVES + ngroups - 1) / ngroups;
  if (nsplit > a.ncells) nsplit = a.ncells;
  if (nsplit < 1) nsplit = 1;
  if (nsplit > 65535) nsplit = 65535;  // grid y
  if (splits_out) *splits_out = (int)nsplit;
  if (dry_run) return cudaSuccess;
  dim3 grid((unsigned)ngroups, (unsigned)nsplit);
  return grad ? launch_cells_tg<D, true>(a, grid, s) : launch_cells_tg<D, false>(a, grid, s);
}

// ---------------------------------------------------------------- one box (q == 1, no retain)
// The same cell test for a single box.  Warp gw owns the cells gw, gw + W, ... (W = all warps of the
// grid; at most 32 per warp for the sizes the grid is chosen for, else in batches of 32): one
// batched test (lane k: candidate k) gives the warp its touched cells, which it then streams
// through two per-warp shared-memory buffers with cp.async (the next touched cell loads while the
// current one is evaluated).  A skipped cell is never read.  Each touched cell is one cells_item
// (full / classified, compacted or masked) added into the warp's fp64 accumulator; the warps'
// accumulators are summed in warp order, then the block reduction + deterministic last-block pass
// of the other single-box scans (single_reduce_finalize).
#ifndef KDE_TUNE_CELLS1_OCC
#define KDE_TUNE_CELLS1_OCC(d) ((d) <= 5 ? 2 : 1)
#endif
#ifndef KDE_TUNE_CELLS1_NBUF
#define KDE_TUNE_CELLS1_NBUF(d) ((d) <= 12 ? 2 : 1)
#endif
__host__ __device__ constexpr int cells_single_occ(int d) { return KDE_TUNE_CELLS1_OCC(d); }
template <int D>
__host__ __device__ constexpr int cells_single_nbuf() { return KDE_TUNE_CELLS1_NBUF(D); }  // shared-memory budget
template <int D>
__host__ __device__ constexpr size_t cells_single_smem() {
  return (size_t)(kCellsThreads / 32) * cells_single_nbuf<D>() * D * kCellPts * sizeof(float);  // per-warp buffers
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(dst))),
               "l"(src)
               : "memory");
}

template <int D, bool GRAD, int MODE>
__device__ __forceinline__ void cells_single_body(const ScanSingleArgs& a, const float4* tab, unsigned nm, bool keep_all,
                                                  const float (&ap)[D], float* wbuf, unsigned char* list, double* wacc,
                                                  unsigned long long* wst) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t W = (int64_t)gridDim.x * (kCellsThreads / 32);
  const int64_t gw = (int64_t)blockIdx.x * (kCellsThreads / 32) + warp;
  constexpr bool EPAN = MODE == 2;
  constexpr float kEps = 1.0f / (1 << 20);
  const float2* cbb2 = reinterpret_cast<const float2*>(a.cbb);
  for (int64_t base = gw; base < a.ncells; base += 32 * W) {  // batches of 32 candidate cells
    // lane k tests candidate base + k W against the box (all dimensions)
    const int64_t cand = base + (int64_t)lane * W;
    float nr = 0.0f, fr = 0.0f;  // EPAN: max_j; Gaussian: sum_j relu^2
    if (cand < a.ncells) {
      if (EPAN) nr = fr = -INFINITY;
#pragma unroll
      for (int j = 0; j < D; ++j) {
        const float2 bb = __ldg(cbb2 + cand * D + j);
        const float4 tb = tab[j];
        const float cc = fmaf(0.5f, bb.x, 0.5f * bb.y) * ap[j], chw = (0.5f * bb.y - 0.5f * bb.x) * ap[j];
        const float dc = fabsf(cc - tb.z);
        const float err = kEps * (fabsf(cc) + chw + fabsf(tb.z) + tb.w);
        const float near = dc - chw - tb.w - err, far = dc + chw - tb.w;
        if (EPAN) {
          nr = fmaxf(nr, near);
          fr = fmaxf(fr, far);
        } else {
          const float n2 = fmaxf(near, 0.0f), f2v = fmaxf(far, 0.0f);
          nr = fmaf(n2, n2, nr);
          fr = fmaf(f2v, f2v, fr);
        }
      }
    }
    const bool touched = cand < a.ncells && (keep_all || (EPAN ? nr < 1.0f : nr < kCullY2));
    const bool isfull = touched && (keep_all || (EPAN ? fr < 1.0f : fr < kCullY2));
    unsigned tm = __ballot_sync(0xffffffffu, touched);
    const unsigned fm = __ballot_sync(0xffffffffu, isfull);
    auto load = [&](int k, int buf) {  // cell base + k W -> buffer buf (cp.async, one group)
      const float* src = a.ccols + (base + (int64_t)k * W) * kCellPts;
      float* dst = wbuf + (size_t)buf * D * kCellPts;
#pragma unroll
      for (int j = 0; j < D; ++j)
#pragma unroll
        for (int h = 0; h < kCellPts / 128; ++h)
          cp_async16(dst + j * kCellPts + 128 * h + 4 * lane, src + (int64_t)j * a.ld + 128 * h + 4 * lane);
      asm volatile("cp.async.commit_group;" ::: "memory");
    };
    int cur = tm ? __ffs(tm) - 1 : -1;
    if (cur >= 0) {
      tm &= tm - 1u;
      load(cur, 0);
    }
    constexpr int NB = cells_single_nbuf<D>();
    int buf = 0;
    while (cur >= 0) {
      const int nxt = tm ? __ffs(tm) - 1 : -1;
      if (nxt >= 0) tm &= tm - 1u;
      if (NB == 2 && nxt >= 0) {
        load(nxt, buf ^ 1);
        asm volatile("cp.async.wait_group 1;" ::: "memory");
      } else {
        asm volatile("cp.async.wait_group 0;" ::: "memory");
      }
      __syncwarp();
      const int64_t cell = base + (int64_t)cur * W;
      const int npts = (int)min((int64_t)kCellPts, a.n - cell * kCellPts);
      const bool fl = (fm >> cur) & 1u;
      const int ev = cells_item<D, GRAD, MODE>(wbuf + (size_t)buf * D * kCellPts, npts, fl, tab, nm, ap, wacc, list, lane);
      if (a.stats && lane == 0) {
        unsigned long long* c4 = wst + 4 * warp;
        c4[0] += 1;
        c4[1] += fl ? 1 : 0;
        c4[2] += (unsigned long long)ev;
        c4[3] += fl ? 0ull : (unsigned long long)npts;
      }
      __syncwarp();  // the buffer is refilled NB cells later
      if (NB == 2) {
        buf ^= 1;
      } else if (nxt >= 0) {
        load(nxt, 0);
      }
      cur = nxt;
    }
  }
}

template <int D, bool GRAD>
__global__ void __launch_bounds__(kCellsThreads, cells_single_occ(D)) scan_cells_single_kernel(const ScanSingleArgs a) {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int NW = kCellsThreads / 32;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  float* wbufs = reinterpret_cast<float*>(smem_raw);  // [NW][2][D][kCellPts]
  __shared__ float4 tab[D];                           // cells_boxdims encoding (b.x, b.y | hd, cb.x, cb.y)
  __shared__ unsigned nm_s, nocull_s;
  __shared__ double wacc[NW][NA];
  __shared__ unsigned long long wst[4 * NW];
  __shared__ __align__(16) unsigned char lists[NW][kCellPts];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    nm_s = 0u;
    nocull_s = 0u;
  }
  if (tid < NW * NA) wacc[tid / NA][tid % NA] = 0.0;
  if (tid < 4 * NW) wst[tid] = 0ull;
  __syncthreads();
  const bool epan = a.consts->kernel == kEpanechnikov;
  if (tid < D) {
    const int j = tid;
    const float apj = a.consts->ap[j];
    const float l = __ldg(a.lo + j), u = __ldg(a.hi + j);
    const unsigned rmin = a.consts->renc[2 * j], rmax = a.consts->renc[2 * j + 1];
    const BoxDim bd = epan ? make_boxdim<kEpanechnikov>(l, u, apj, rmin, rmax) : make_boxdim(l, u, apj, rmin, rmax);
    const float2 cb = make_cullbox(l, u, apj, rmin, rmax);
    const bool nar = !epan && bd.hd > 0.0f;
    tab[j] = make_float4(bd.b.x, nar ? bd.hd : bd.b.y, cb.x, cb.y);
    if (nar) atomicOr(&nm_s, 1u << j);
    if (!cullbox_ok(cb)) atomicOr(&nocull_s, 1u);
  }
  __syncthreads();
  float ap[D];
#pragma unroll
  for (int j = 0; j < D; ++j) ap[j] = a.consts->ap[j];
  const unsigned nm = nm_s;
  const bool keep_all = nocull_s != 0u;
  float* wbuf = wbufs + (size_t)warp * cells_single_nbuf<D>() * D * kCellPts;
  if (epan)
    cells_single_body<D, GRAD, 2>(a, tab, nm, keep_all, ap, wbuf, lists[warp], wacc[warp], wst);
  else if (nm)
    cells_single_body<D, GRAD, 1>(a, tab, nm, keep_all, ap, wbuf, lists[warp], wacc[warp], wst);
  else
    cells_single_body<D, GRAD, 0>(a, tab, nm, keep_all, ap, wbuf, lists[warp], wacc[warp], wst);
  __syncthreads();
  double acc[NA];
#pragma unroll
  for (int k = 0; k < NA; ++k) {
    double t = 0.0;
    if (tid == 0)
      for (int w = 0; w < NW; ++w) t += wacc[w][k];  // warp order: deterministic
    acc[k] = t;
  }
  if (a.stats && tid < 4) {
    unsigned long long t = 0ull;
    for (int w = 0; w < NW; ++w) t += wst[4 * w + tid];
    atomicAdd(a.stats + tid, t);
  }
  (void)lane;
  single_reduce_finalize<NA, kCellsThreads>(a, acc);
}

template <int D>
cudaError_t launch_cells_single_t(bool grad, const ScanSingleArgs& a, int grid, cudaStream_t s) {
  constexpr size_t smem = cells_single_smem<D>();
  static_assert(smem + 8 * 1024 <= 227 * 1024, "single-box cells scan shared memory");
  static std::atomic<unsigned long long> attr_set{0ull};  // per device ordinal
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const unsigned long long bit = 1ull << (dev & 63);
  if (!(attr_set.load(std::memory_order_acquire) & bit)) {
    e = cudaFuncSetAttribute(scan_cells_single_kernel<D, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(scan_cells_single_kernel<D, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set.fetch_or(bit, std::memory_order_acq_rel);
  }
  if (grad)
    scan_cells_single_kernel<D, true><<<grid, kCellsThreads, smem, s>>>(a);
  else
    scan_cells_single_kernel<D, false><<<grid, kCellsThreads, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace kde
