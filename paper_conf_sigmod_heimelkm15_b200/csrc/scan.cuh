// scan.cuh -- the hot path: one pass over the sample computing, per box,
//   S_0   = sum_i p^(i)(Omega)                         eq. (2)+(13)
//   S_j   = sum_i w_ij prod_{k!=j} D_ik                eq. (17), P:L545 (d p^(i)/d h_j = gconst_j S_j-term)
// and optionally the retained per-point contributions p^(i).
//
// q == 1 with culling (default): scan_single_tma_kernel<..., CULL=1> (scan_single_tma.cuh).
// scan_single_kernel  (q == 1, cull off, d > 8): HBM-streaming reduction.  Each thread owns
//   float4 chunks of the SoA columns (coalesced 128-bit loads, streaming cache
//   hint), fp32 math per point, fp32 sums over 8 points flushed to fp64,
//   warp-shuffle + block reduction, and a deterministic last-block second pass
//   (fixed order) that also finalises p_hat and dp_hat/dh.
// scan_batched_kernel (q > 1): FP32/SFU-bound.  A CTA owns QB <= 256 boxes
//   (bounds in registers; 256/QB threads share a box and split its points)
//   and one contiguous split of the sample; sample
//   tiles of 256 points x d columns are staged into shared memory by TMA bulk
//   copies (cp.async.bulk + mbarrier, a 4-stage ring refilled by the last warp
//   out, no CTA barrier) and read as broadcasts.  Batches that fill 256-box CTAs
//   are culled (reading R15): boxes ordered by a probed kept count (cull_order.cu)
//   and re-sorted in the CTA, per-tile alive masks, lane-local alive walks.
//   fp32 sums over 32 points are flushed into per-thread fp64 accumulators in
//   shared memory; per-(split, box) partials go to global memory and are
//   reduced in fixed split order by reduce_splits_kernel (kernels.cu).
#pragma once
#include <atomic>
#include <cstdint>
#include <cuda_runtime.h>

#include "common.cuh"
#include "peer.cuh"
#include "phi.cuh"

namespace kde {

// boxes per thread (QT) and resident CTAs per SM (MINB) of the batched scan
// (measured on B200 by tools/tune_batched.cu, gpurun_out/tune1.jsonl)
template <int D>
struct QT_for {
  static constexpr int value = 1;
};
// (KDE_TUNE_* macros override the measured defaults for tuning builds: tools/kbench.cu)
template <int D>
struct PU_for {  // point pairs per inner iteration
#ifdef KDE_TUNE_PU
  static constexpr int value = KDE_TUNE_PU;
#else
  static constexpr int value = 2;
#endif
};
template <int D>
struct MINB_for {
#ifdef KDE_TUNE_MINB
  static constexpr int value = KDE_TUNE_MINB;
#else
  static constexpr int value = D <= 6 ? 4 : (D <= 12 ? 2 : 1);
#endif
};
// single-box TMA scan: points per tile, tiles in flight, resident CTAs per SM
// (measured on B200 with tools/kbench.cu, profiles/r01_tune_single_ws.jsonl:
// 2048-point tiles; 2 stages x 2 CTAs up to d = 5, 3 stages x 1 CTA above)
#ifndef KDE_TUNE_SINGLE_TILE
#define KDE_TUNE_SINGLE_TILE 2048
#endif
constexpr int kSingleTile = KDE_TUNE_SINGLE_TILE;
static_assert(kColAlign % kSingleTile == 0, "TMA tiles of the single-box scan must not cross the padded column end");
__host__ __device__ constexpr int single_stages(int d) {
#ifdef KDE_TUNE_SINGLE_STAGES
  return (void)d, KDE_TUNE_SINGLE_STAGES;
#else
  return d <= 5 ? 2 : 3;
#endif
}
__host__ __device__ constexpr int single_tma_occ(int d) {
#ifdef KDE_TUNE_SINGLE_OCC
  return (void)d, KDE_TUNE_SINGLE_OCC;
#else
  return d <= 5 ? 2 : 1;
#endif
}

constexpr int kSingleThreads = 256;
constexpr int kBatchedThreads = 256;
constexpr int kTilePts = 256;  // points per shared-memory tile
constexpr int kFlushPts = 32;  // fp32 partial sums are flushed to fp64 every kFlushPts points
constexpr int kSingleFlushPts = 16;  // single-box scan: fp32 partials flushed every 16 points

// resident 256-thread CTAs per SM for the single-box scan (register budget)
// (measured on B200 by tools/tune_single.cu, profiles/r01_tune_single*.jsonl)
#ifndef KDE_TUNE_SINGLE_TMA_MAXD
#define KDE_TUNE_SINGLE_TMA_MAXD 8
#endif
__host__ __device__ constexpr bool single_uses_tma(int d) { return d <= KDE_TUNE_SINGLE_TMA_MAXD; }
__host__ __device__ constexpr int single_occ(int d, bool grad) {
  return grad ? (d <= 3 ? 4 : (d <= 10 ? 3 : 1)) : (d <= 10 ? 4 : (d <= 14 ? 2 : 1));
}

__device__ __forceinline__ float f4c(const float4& v, int p) {
  return p == 0 ? v.x : (p == 1 ? v.y : (p == 2 ? v.z : v.w));
}

// All d factors of eq. (13) for one point and one box, the product p^(i), and
// (GRAD) the d gradient terms w_j prod_{k!=j} D_k, added into s[0..D].
// Returns p^(i).  `valid` masks padding points (contributes exactly 0).
// MODE: 0 = Gaussian, no narrow dimension; 1 = Gaussian, general (narrow
// dimensions on the Gauss-Legendre path); 2 = Epanechnikov product kernel.
template <int D, bool GRAD, int MODE>
__device__ __forceinline__ float point_box(const BoxDim (&bd)[D], const float (&t)[D], const float (&ap)[D],
                                           float* s, bool valid) {
  float Dv[D], wv[D];
#pragma unroll
  for (int j = 0; j < D; ++j)
    Dv[j] = MODE == 2 ? phi_epan<GRAD>(bd[j], t[j], ap[j], wv[j]) : phi_diff<GRAD, MODE == 1>(bd[j], t[j], ap[j], wv[j]);
  float pre[D + 1];
  pre[0] = 1.0f;
#pragma unroll
  for (int j = 0; j < D; ++j) pre[j + 1] = pre[j] * Dv[j];
  const float c = valid ? pre[D] : 0.0f;
  s[0] += c;
  if (GRAD) {
    float suf = valid ? 1.0f : 0.0f;
#pragma unroll
    for (int j = D - 1; j >= 0; --j) {
      s[1 + j] = fmaf(wv[j], pre[j] * suf, s[1 + j]);
      suf *= Dv[j];
    }
  }
  return c;
}

// point_box for two points at once (float2 lanes = points, see phi_diff2):
// s2[k] holds per-lane fp32 partial sums; `valid` is 1 or 0 per point and
// enters as the first factor of the product, so a padding point contributes
// exactly 0 to every sum.  Returns (p^(i0), p^(i1)).
template <int D, bool GRAD, int MODE>
__device__ __forceinline__ float2 point_box2(const BoxDim (&bd)[D], const float2 (&t)[D], const float (&ap)[D],
                                             float2* s2, const float2 valid) {
  float2 Dv[D], wv[D];
#pragma unroll
  for (int j = 0; j < D; ++j) {
    if (MODE == 2) {
      Dv[j] = phi_epan2<GRAD>(bd[j], t[j], ap[j], wv[j]);
    } else {
      Dv[j] = phi_diff2<GRAD, MODE == 1>(bd[j], t[j], ap[j], wv[j]);
    }
  }
  float2 pre[D + 1];
  pre[0] = valid;
#pragma unroll
  for (int j = 0; j < D; ++j) pre[j + 1] = __fmul2_rn(pre[j], Dv[j]);
  s2[0] = __fadd2_rn(s2[0], pre[D]);
  if (GRAD) {
    float2 suf = f2(1.0f);
#pragma unroll
    for (int j = D - 1; j >= 0; --j) {
      s2[1 + j] = __ffma2_rn(wv[j], j == D - 1 ? pre[j] : __fmul2_rn(pre[j], suf), s2[1 + j]);
      if (j > 0) suf = j == D - 1 ? Dv[j] : __fmul2_rn(suf, Dv[j]);
    }
  }
  return pre[D];
}

// GRAD variant of point_box2 with few live registers (the culled single-box scan at d >= 9):
// the gradient term of dimension j is written w_j * p / D_j instead of w_j * prefix_j * suffix_j,
// so only the d ratios r_j = w_j / D_j and the running product p are live, not the d factors,
// d terms and d + 1 prefixes.  D_j == 0 (a factor flushed to zero) drops that term: then
// |w_j| <= |y'| e^{-z^2} < 2^-120 as well, far below the culling floor (reading R15).
template <int D, int MODE>
__device__ __forceinline__ float2 point_box2_ratio(const BoxDim (&bd)[D], const float2 (&t)[D], const float (&ap)[D],
                                                   float2* s2, const float2 valid) {
  float2 r[D];
  float2 p = valid;
#pragma unroll
  for (int j = 0; j < D; ++j) {
    float2 w;
    const float2 Dj = MODE == 2 ? phi_epan2<true>(bd[j], t[j], ap[j], w) : phi_diff2<true, MODE == 1>(bd[j], t[j], ap[j], w);
    p = __fmul2_rn(p, Dj);
    const float2 inv = make_float2(Dj.x != 0.0f ? rcp_approx(Dj.x) : 0.0f, Dj.y != 0.0f ? rcp_approx(Dj.y) : 0.0f);
    r[j] = __fmul2_rn(w, inv);
  }
  s2[0] = __fadd2_rn(s2[0], p);
#pragma unroll
  for (int j = 0; j < D; ++j) s2[1 + j] = __ffma2_rn(r[j], p, s2[1 + j]);
  return p;
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Block reduction of the per-thread fp64 sums (fixed order), one fp64 partial
// per block, and a deterministic second pass by the last block to finish
// (fixed strided order + fixed tree) that also finalises p_hat, dp_hat/dh.
template <int NA, int NT = kSingleThreads>
__device__ __forceinline__ void single_reduce_finalize(const ScanSingleArgs& a, const double (&acc)[NA]) {
  __shared__ double red[NT / 32][NA];
  __shared__ bool am_last;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int k = 0; k < NA; ++k) {
    const double r = warp_sum(acc[k]);
    if (lane == 0) red[warp][k] = r;
  }
  __syncthreads();
  if (threadIdx.x < NA) {
    double t = 0.0;
#pragma unroll
    for (int w = 0; w < NT / 32; ++w) t += red[w][threadIdx.x];
    a.block_partials[(int64_t)blockIdx.x * NA + threadIdx.x] = t;
    __threadfence();
  }
  __syncthreads();
  if (threadIdx.x == 0) am_last = (atomicAdd(a.counter, 1u) == gridDim.x - 1);
  __syncthreads();
  if (!am_last) return;
  __threadfence();
  // fused exchange (sharded model, peer transport): the final sums go straight into every rank's
  // window slot of this epoch, then this rank's flag is released (peer.cuh)
  const uint64_t pe = a.peer ? peer_next_epoch(*a.peer) : 0;
  // deterministic second pass over the block partials (fixed strided order + fixed tree)
  for (int k = 0; k < NA; ++k) {
    double t = 0.0;
    for (int b = threadIdx.x; b < (int)gridDim.x; b += NT) t += __ldcg(a.block_partials + (int64_t)b * NA + k);
    t = warp_sum(t);
    __syncthreads();
    if (lane == 0) red[warp][0] = t;
    __syncthreads();
    if (threadIdx.x == 0) {
      double tot = 0.0;
#pragma unroll
      for (int w = 0; w < NT / 32; ++w) tot += red[w][0];
      a.sums_out[k] = tot;
      if (a.peer) peer_store(*a.peer, pe, k, tot);
      const double fin = k == 0 ? tot / a.n_global : tot * a.consts->gconst[k - 1] / a.n_global;
      if (a.fin_out) a.fin_out[k] = fin;
      if (k == 0 && a.est_out) *a.est_out = fin;
      if (k > 0 && a.dpdh_out) a.dpdh_out[k - 1] = fin;
    }
  }
  if (threadIdx.x == 0) {
    if (a.peer) peer_release(*a.peer, pe);
    *a.counter = 0u;
  }
}

// ---------------------------------------------------------------- single box
// The box is uniform over the CTA: its per-dimension setup (b1, b2, hd, ap)
// lives in shared memory and is re-read (broadcast LDS.128) per point group.
// Each thread processes VW consecutive points per column load (VW-wide
// vector loads, coalesced across the warp).
template <int D, bool GRAD>
struct SingleVW {
#ifdef KDE_TUNE_SINGLE_VW
  static constexpr int value = KDE_TUNE_SINGLE_VW;
#else
  static constexpr int value = 2;
#endif
};
template <int D, bool GRAD>
struct SinglePF {  // register double-buffered prefetch: spills, measured slower (tools/tune_single.cu)
#ifdef KDE_TUNE_SINGLE_PF
  static constexpr bool value = KDE_TUNE_SINGLE_PF;
#else
  static constexpr bool value = false;
#endif
};

template <int VW>
struct VecT;
template <>
struct VecT<1> {
  using type = float;
};
template <>
struct VecT<2> {
  using type = float2;
};
template <>
struct VecT<4> {
  using type = float4;
};

__device__ __forceinline__ float vcomp(const float& v, int) { return v; }
__device__ __forceinline__ float vcomp(const float2& v, int p) { return p == 0 ? v.x : v.y; }
__device__ __forceinline__ float ldcs_v(const float* p) { return __ldcs(p); }
__device__ __forceinline__ void stcs_v(float* p, const float* c) { __stcs(p, c[0]); }
__device__ __forceinline__ float vcomp(const float4& v, int p) { return f4c(v, p); }
__device__ __forceinline__ float2 ldcs_v(const float2* p) { return __ldcs(p); }
__device__ __forceinline__ float4 ldcs_v(const float4* p) { return __ldcs(p); }
__device__ __forceinline__ void stcs_v(float2* p, const float* c) { __stcs(p, make_float2(c[0], c[1])); }
__device__ __forceinline__ void stcs_v(float4* p, const float* c) { __stcs(p, make_float4(c[0], c[1], c[2], c[3])); }

template <int D, bool GRAD, int MODE, int VW>
__device__ __forceinline__ void single_group(const typename VecT<VW>::type (&tv)[D], const float4* __restrict__ smc,
                                             float2* s2, float* c_out, int64_t v, int valid) {
  static_assert(VW == 2 || VW == 4, "points are processed in pairs");
  BoxDim bd[D];
  float ap[D];
#pragma unroll
  for (int j = 0; j < D; ++j) {
    const float4 c = smc[j];
    bd[j].b = make_float2(c.x, c.y);
    bd[j].hd = c.z;
    ap[j] = c.w;
  }
  float cs[VW];
#pragma unroll
  for (int p = 0; p < VW; p += 2) {
    float2 t[D];
#pragma unroll
    for (int j = 0; j < D; ++j) t[j] = make_float2(vcomp(tv[j], p), vcomp(tv[j], p + 1));
    const float2 c = point_box2<D, GRAD, MODE>(bd, t, ap, s2,
                                               make_float2(p < valid ? 1.0f : 0.0f, p + 1 < valid ? 1.0f : 0.0f));
    cs[p] = c.x;
    cs[p + 1] = c.y;
  }
  if (c_out) stcs_v(reinterpret_cast<typename VecT<VW>::type*>(c_out) + v, cs);
}

template <int D, bool GRAD, int MODE, int VW, bool PF>
__device__ __forceinline__ void scan_single_body(const ScanSingleArgs& a, const float4* smc);

template <int D, bool GRAD, int VW = SingleVW<D, GRAD>::value, int OCC = single_occ(D, GRAD),
          bool PF = SinglePF<D, GRAD>::value>
__global__ void __launch_bounds__(kSingleThreads, OCC) scan_single_kernel(const ScanSingleArgs a) {
  __shared__ float4 smc[D];
  __shared__ int narrow_s;
  if (threadIdx.x == 0) narrow_s = 0;
  __syncthreads();
  if (threadIdx.x < D) {
    const int j = threadIdx.x;
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
    scan_single_body<D, GRAD, 2, VW, PF>(a, smc);
  else if (narrow_s)
    scan_single_body<D, GRAD, 1, VW, PF>(a, smc);
  else
    scan_single_body<D, GRAD, 0, VW, PF>(a, smc);
}

template <int D, bool GRAD, int MODE, int VW, bool PF>
__device__ __forceinline__ void scan_single_body(const ScanSingleArgs& a, const float4* smc) {
  constexpr int NA = GRAD ? D + 1 : 1;
  using V = typename VecT<VW>::type;
  double acc[NA];
#pragma unroll
  for (int k = 0; k < NA; ++k) acc[k] = 0.0;

  const V* col = reinterpret_cast<const V*>(a.cols);
  const int64_t ldv = a.ld / VW;
  const int64_t nfull = a.n / VW;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  // fp32 partial sums over up to kSingleFlushPts points, then flushed into
  // fp64.  The next group's column loads are issued before the current group
  // is computed (register double buffer), so each warp keeps d loads in flight.
  constexpr int kGroups = kSingleFlushPts / VW;
  if (PF) {
    V cur[D], nxt[D];
    if (v < nfull) {
#pragma unroll
      for (int j = 0; j < D; ++j) cur[j] = ldcs_v(col + j * ldv + v);
    }
    while (v < nfull) {
      float2 s[NA];
#pragma unroll
      for (int k = 0; k < NA; ++k) s[k] = f2(0.0f);
#pragma unroll 1
      for (int u = 0; u < kGroups && v < nfull; u += 2) {
        int64_t vn = v + stride;
        if (vn < nfull) {
#pragma unroll
          for (int j = 0; j < D; ++j) nxt[j] = ldcs_v(col + j * ldv + vn);
        }
        single_group<D, GRAD, MODE, VW>(cur, smc, s, a.c_out, v, VW);
        v = vn;
        if (v >= nfull) break;
        vn = v + stride;
        if (vn < nfull) {
#pragma unroll
          for (int j = 0; j < D; ++j) cur[j] = ldcs_v(col + j * ldv + vn);
        }
        single_group<D, GRAD, MODE, VW>(nxt, smc, s, a.c_out, v, VW);
        v = vn;
      }
#pragma unroll
      for (int k = 0; k < NA; ++k) acc[k] += (double)s[k].x + (double)s[k].y;
    }
  } else {
    while (v < nfull) {
      float2 s[NA];
#pragma unroll
      for (int k = 0; k < NA; ++k) s[k] = f2(0.0f);
#pragma unroll 1
      for (int u = 0; u < kGroups && v < nfull; ++u, v += stride) {
        V t0[D];
#pragma unroll
        for (int j = 0; j < D; ++j) t0[j] = ldcs_v(col + j * ldv + v);
        single_group<D, GRAD, MODE, VW>(t0, smc, s, a.c_out, v, VW);
      }
#pragma unroll
      for (int k = 0; k < NA; ++k) acc[k] += (double)s[k].x + (double)s[k].y;
    }
  }
  // the ragged tail group (n % VW points) belongs to the thread that reaches v == nfull
  if (v == nfull && a.n > (int64_t)VW * nfull) {
    const int valid = (int)(a.n - (int64_t)VW * nfull);
    V t0[D];
#pragma unroll
    for (int j = 0; j < D; ++j) t0[j] = ldcs_v(col + j * ldv + v);
    float2 s[NA];
#pragma unroll
    for (int k = 0; k < NA; ++k) s[k] = f2(0.0f);
    single_group<D, GRAD, MODE, VW>(t0, smc, s, a.c_out, v, valid);
#pragma unroll
    for (int k = 0; k < NA; ++k) acc[k] += (double)s[k].x + (double)s[k].y;
  }

  single_reduce_finalize<NA>(a, acc);
}

// ---------------------------------------------------------------- many boxes
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait_parity(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "KDE_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra KDE_WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// bulk copy with an L2 eviction policy (createpolicy), for streams that should not displace others
__device__ __forceinline__ void bulk_g2s_hint(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
#ifndef KDE_TUNE_SUSPEND_NS
#define KDE_TUNE_SUSPEND_NS 1000000
#endif
// as mbar_wait_parity, but a waiting warp is suspended (up to the hint, woken early by the phase
// flip) instead of spinning on issue slots that the computing warps of the SM need
__device__ __forceinline__ void mbar_wait_parity_suspend(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "KDE_WAITS_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
      "@!p bra KDE_WAITS_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity), "r"((uint32_t)KDE_TUNE_SUSPEND_NS)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// Accumulate every point of one shared-memory tile against the thread's QT
// boxes.  The thread takes point PAIRS (2pp, 2pp + 1), pp = phase, phase + R,
// ... (one LDS.64 per column and pair; see point_box2).  No barriers inside,
// so the GENERAL (narrow-dimension) and fast variants can be chosen per warp.
template <int D, bool GRAD, int MODE, int QT, int PU>
__device__ __forceinline__ void batched_tile_compute(const float* tl, int npts, int phase, int R, double* accsh,
                                                     const BoxDim (&bd)[QT][D], const float (&ap)[D]) {
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int kFlushPairs = kFlushPts / 2;
  const int tid = threadIdx.x;
  const int npairs = (npts + 1) >> 1;
  const int mine = npairs > phase ? (npairs - phase + R - 1) / R : 0;
  for (int m0 = 0; m0 < mine; m0 += kFlushPairs) {
    const int me = min(m0 + kFlushPairs, mine);
    float2 s[QT][NA];
#pragma unroll
    for (int qq = 0; qq < QT; ++qq)
#pragma unroll
      for (int kk = 0; kk < NA; ++kk) s[qq][kk] = f2(0.0f);
    int m = m0;
    for (; m + PU <= me; m += PU) {  // PU pairs per iteration: more independent chains per warp
#pragma unroll
      for (int u = 0; u < PU; ++u) {
        const int pp = phase + (m + u) * R;
        float2 t[D];
#pragma unroll
        for (int j = 0; j < D; ++j) t[j] = *reinterpret_cast<const float2*>(tl + j * kTilePts + 2 * pp);
        const float2 valid = make_float2(1.0f, 2 * pp + 1 < npts ? 1.0f : 0.0f);
#pragma unroll
        for (int qq = 0; qq < QT; ++qq) point_box2<D, GRAD, MODE>(bd[qq], t, ap, s[qq], valid);
      }
    }
    for (; m < me; ++m) {
      const int pp = phase + m * R;
      float2 t[D];
#pragma unroll
      for (int j = 0; j < D; ++j) t[j] = *reinterpret_cast<const float2*>(tl + j * kTilePts + 2 * pp);
      const float2 valid = make_float2(1.0f, 2 * pp + 1 < npts ? 1.0f : 0.0f);
#pragma unroll
      for (int qq = 0; qq < QT; ++qq) point_box2<D, GRAD, MODE>(bd[qq], t, ap, s[qq], valid);
    }
#pragma unroll
    for (int qq = 0; qq < QT; ++qq)
#pragma unroll
      for (int kk = 0; kk < NA; ++kk)
        accsh[(qq * NA + kk) * kBatchedThreads + tid] += (double)s[qq][kk].x + (double)s[qq][kk].y;
  }
}

// Culled tile compute (reading R15, one box per thread, QB == 256): the thread
// classifies all kTilePts points of the tile against its box (cull_o2, 3 packed
// FMA-pipe + 2 ALU instructions per point pair and dimension, broadcast LDS.64),
// keeping a 256-bit alive mask in registers, then walks its own alive points two at a
// time (the warp iterates max over its lanes -- boxes are sorted by their kept
// fraction within the CTA, see the kernel) with lane-varying LDS gathers from the tile.
constexpr int kTileWords = kTilePts / 32;
#ifndef KDE_TUNE_BATCHED_LINF
#define KDE_TUNE_BATCHED_LINF 0
#endif

// phase / R: with R threads per box (small batches) the thread owns the words w = phase (mod R)
template <int D, bool EPAN>
__device__ __forceinline__ void cull_tile_mask(const float* tl, int npts, const float (&ap)[D], const float2 (&cb)[D],
                                               unsigned (&mk)[kTileWords], int phase = 0, int R = 1,
                                               bool keep_all = false) {
#pragma unroll
  for (int w = 0; w < kTileWords; ++w) {
    mk[w] = 0u;
    if ((w & (R - 1)) != phase) continue;  // warp-uniform: a warp holds one phase (QB >= 32)
    unsigned m = 0u;
#pragma unroll 4
    for (int q = 0; q < 16; ++q) {
      const int pp = 16 * w + q;
      float2 t[D];
#pragma unroll
      for (int j = 0; j < D; ++j) t[j] = *reinterpret_cast<const float2*>(tl + j * kTilePts + 2 * pp);
      // kept <=> score - limit < 0: the sign bits are the mask bits (finite scores, exact sign)
      // KDE_TUNE_BATCHED_LINF: Gaussian classification by max_j o_j >= sqrt(64.5) (sound: it implies
      // sum_j o_j^2 >= 64.5) -- 2 FMA-pipe + 1 ALU op per pair-dimension instead of 4 FMA-pipe ops,
      // at the price of evaluating points the L2 test would cull (A/B experiment)
      constexpr bool kMax = EPAN || KDE_TUNE_BATCHED_LINF;
      const float lim = EPAN ? cull_limit<true>() : (KDE_TUNE_BATCHED_LINF ? 8.0311892f : cull_limit<false>());
      const float2 u = __fadd2_rn(cull_score<D, kMax>(t, ap, cb), f2(-lim));
      m |= (__float_as_uint(u.x) >> 31) << (2 * q);
      m |= (__float_as_uint(u.y) >> 31) << (2 * q + 1);
    }
    if (keep_all) m = 0xffffffffu;  // box not representable in fp32 scaled coordinates: no culling
    const int v = npts - 32 * w;  // valid points in this word
    mk[w] = v >= 32 ? m : (v > 0 ? m & ((1u << v) - 1u) : 0u);
  }
}

__device__ __forceinline__ unsigned sel_word(const unsigned (&mk)[kTileWords], int w) {
  unsigned r = mk[0];
#pragma unroll
  for (int i = 1; i < kTileWords; ++i) r = w == i ? mk[i] : r;
  return r;
}

template <int D, bool GRAD, int MODE>
__device__ __forceinline__ void batched_tile_cull(const float* tl, int npts, double* accsh, const BoxDim (&bd)[D],
                                                  const float (&ap)[D], const float2 (&cb)[D], int phase, int R) {
  bool keep_all = false;
#pragma unroll
  for (int j = 0; j < D; ++j) keep_all |= !cullbox_ok(cb[j]);
  constexpr int NA = GRAD ? D + 1 : 1;
  constexpr int kFlushPairs = kFlushPts / 2;
  const int tid = threadIdx.x;
  unsigned mk[kTileWords];
  cull_tile_mask<D, MODE == 2>(tl, npts, ap, cb, mk, phase, R, keep_all);
  int w = 0;
  unsigned m = mk[0];
  auto next = [&]() -> int {  // next alive point of this lane, -1 when exhausted
    while (m == 0u && w < kTileWords - 1) m = sel_word(mk, ++w);
    if (m == 0u) return -1;
    const int b = __ffs(m) - 1;
    m &= m - 1u;
    return 32 * w + b;
  };
  float2 s[NA];
#pragma unroll
  for (int kk = 0; kk < NA; ++kk) s[kk] = f2(0.0f);
  int it = 0;
  while (true) {
    const int p0 = next(), p1 = next();
    if (!__any_sync(0xffffffffu, p0 >= 0)) break;
    float2 t[D];
#pragma unroll
    for (int j = 0; j < D; ++j)  // masked points take a finite coordinate (the box bound)
      t[j] = make_float2(p0 >= 0 ? tl[j * kTilePts + p0] : bd[j].b.y, p1 >= 0 ? tl[j * kTilePts + p1] : bd[j].b.y);
    point_box2<D, GRAD, MODE>(bd, t, ap, s, make_float2(p0 >= 0 ? 1.0f : 0.0f, p1 >= 0 ? 1.0f : 0.0f));
    if (++it == kFlushPairs) {
#pragma unroll
      for (int kk = 0; kk < NA; ++kk) {
        accsh[kk * kBatchedThreads + tid] += (double)s[kk].x + (double)s[kk].y;
        s[kk] = f2(0.0f);
      }
      it = 0;
    }
  }
#pragma unroll
  for (int kk = 0; kk < NA; ++kk) accsh[kk * kBatchedThreads + tid] += (double)s[kk].x + (double)s[kk].y;
}

// The tile loop of the batched scan: a ring of kBatchedStages tile buffers
// filled by TMA bulk copies (completing on full[stage]).  No CTA barrier:
// each warp arrives on the stage's counter after its last read, and the
// LAST warp out issues the copies of tile k + kBatchedStages into it, so warps
// with less work (culling: boxes sorted by kept fraction) run ahead by up to
// kBatchedStages - 1 tiles instead of waiting at every tile.
#ifndef KDE_TUNE_BATCHED_STAGES
#define KDE_TUNE_BATCHED_STAGES 4
#endif
constexpr int kBatchedStages = KDE_TUNE_BATCHED_STAGES;

template <int D, bool GRAD, int QT, int PU, typename Issue>
__device__ __forceinline__ void batched_tiles(const ScanBatchedArgs& a, const float* tile, uint64_t* full, int* cnt,
                                              double* accsh, const BoxDim (&bd)[QT][D], const float (&ap)[D],
                                              const float2 (&cb)[D], bool cull, int64_t s0, int64_t s1,
                                              int ntiles, int mode, int phase, int R, Issue& issue) {
  const int tid = threadIdx.x;
  for (int k = 0; k < ntiles; ++k) {
    const int st = k % kBatchedStages;
    mbar_wait_parity(&full[st], (uint32_t)((k / kBatchedStages) & 1));
    const float* tl = tile + st * D * kTilePts;
    const int64_t rem = s1 - (s0 + (int64_t)k * kTilePts);
    const int npts = rem < kTilePts ? (int)rem : kTilePts;
    if (cull && mode == 2)
      batched_tile_cull<D, GRAD, 2>(tl, npts, accsh, bd[0], ap, cb, phase, R);
    else if (cull && mode == 1)
      batched_tile_cull<D, GRAD, 1>(tl, npts, accsh, bd[0], ap, cb, phase, R);
    else if (cull)
      batched_tile_cull<D, GRAD, 0>(tl, npts, accsh, bd[0], ap, cb, phase, R);
    else if (mode == 2)
      batched_tile_compute<D, GRAD, 2, QT, PU>(tl, npts, phase, R, accsh, bd, ap);
    else if (mode == 1)
      batched_tile_compute<D, GRAD, 1, QT, PU>(tl, npts, phase, R, accsh, bd, ap);
    else
      batched_tile_compute<D, GRAD, 0, QT, PU>(tl, npts, phase, R, accsh, bd, ap);
    __syncwarp();
    if ((tid & 31) == 0) {
      __threadfence_block();  // this warp's reads of the stage precede its arrival
      if (atomicAdd(&cnt[st], 1) == kBatchedThreads / 32 - 1) {
        cnt[st] = 0;
        if (k + kBatchedStages < ntiles) issue(k + kBatchedStages);
      }
    }
  }
}

template <int D, bool GRAD, int QT = QT_for<D>::value>
constexpr size_t batched_smem_bytes() {
  constexpr int NA = GRAD ? D + 1 : 1;
  return (size_t)kBatchedStages * D * kTilePts * sizeof(float) + (size_t)QT * NA * kBatchedThreads * sizeof(double) +
         kBatchedStages * (sizeof(uint64_t) + sizeof(int));
}

template <int D, bool GRAD, int QT = QT_for<D>::value, int MINB = MINB_for<D>::value, int PU = PU_for<D>::value>
__global__ void __launch_bounds__(kBatchedThreads, MINB) scan_batched_kernel(const ScanBatchedArgs a) {
  constexpr int NA = GRAD ? D + 1 : 1;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  float* tile = reinterpret_cast<float*>(smem_raw);  // [kBatchedStages][D][kTilePts]
  double* accsh = reinterpret_cast<double*>(smem_raw + (size_t)kBatchedStages * D * kTilePts * sizeof(float));
  uint64_t* bar = reinterpret_cast<uint64_t*>(reinterpret_cast<unsigned char*>(accsh) +
                                              (size_t)QT * NA * kBatchedThreads * sizeof(double));  // full[stages]
  int* cnt = reinterpret_cast<int*>(bar + kBatchedStages);                                     // [stages]
  const int tid = threadIdx.x;

  // This CTA's QB boxes (slots 0..QB-1, box qbase + slot).  With QB < 256 each
  // box is handled by R = 256/QB threads ("phases") that split the points of
  // every tile, so small batches (e.g. the ~100-box training sets of batch
  // optimisation) still keep all threads busy.  Boxes with a
  // narrow dimension need the general Phi path; a CTA-local stable partition
  // puts them into the last slots so at most one warp mixes both kinds.
  static_assert(QT == 1, "the phase mapping assumes one box per thread");
  const int QB = a.qb;
  const int R = kBatchedThreads / QB;
  const int slot = tid % QB, phase = tid / QB;
  const int64_t qbase = (int64_t)blockIdx.x * QB;
  __shared__ int perm_s[kBatchedThreads];
  __shared__ int base_s[2 * (kBatchedThreads / 32) + 1];
  const int lane = tid & 31, warp = tid >> 5;
  float ap[D];
#pragma unroll
  for (int j = 0; j < D; ++j) ap[j] = a.consts->ap[j];
  const bool epan = a.consts->kernel == kEpanechnikov;
  bool nar = false;
  if (tid < QB && !epan) {
    int64_t qi = qbase + tid;
    if (qi >= a.q) qi = a.q - 1;  // duplicate a valid box; its partial is never written
    if (a.perm) qi = a.perm[qi];
#pragma unroll
    for (int j = 0; j < D; ++j) {
      const float l = __ldg(a.lo + qi * D + j), u = __ldg(a.hi + qi * D + j);
      const float dy = (u - l) * ap[j];
      nar |= dy > 0.0f && dy < kNarrowY;
    }
  }
  const unsigned live = __ballot_sync(0xffffffffu, tid < QB);
  const unsigned nmask = __ballot_sync(0xffffffffu, nar);
  if (lane == 0) {
    base_s[2 * warp] = __popc(live & ~nmask);  // normal count
    base_s[2 * warp + 1] = __popc(nmask);      // narrow count
  }
  __syncthreads();
  if (tid == 0) {  // exclusive prefixes in slot order: normals first, then narrows
    constexpr int G = kBatchedThreads / 32;
    int tn = 0;
    for (int g = 0; g < G; ++g) tn += base_s[2 * g];
    int rn = 0, rw = tn;
    for (int g = 0; g < G; ++g) {
      const int cn = base_s[2 * g], cw = base_s[2 * g + 1];
      base_s[2 * g] = rn;
      base_s[2 * g + 1] = rw;
      rn += cn;
      rw += cw;
    }
  }
  __syncthreads();
  if (tid < QB) {
    const unsigned lt = (1u << lane) - 1u;
    const int pos = nar ? base_s[2 * warp + 1] + __popc(nmask & lt) : base_s[2 * warp] + __popc(live & ~nmask & lt);
    perm_s[pos] = tid;
  }
  __syncthreads();
  BoxDim bd[QT][D];
  bool narrow[QT];
  {
    int64_t qi = qbase + perm_s[slot];
    if (qi >= a.q) qi = a.q - 1;
    if (a.perm) qi = a.perm[qi];
    narrow[0] = false;
#pragma unroll
    for (int j = 0; j < D; ++j) {
      if (epan) {
        bd[0][j] = make_boxdim<kEpanechnikov>(__ldg(a.lo + qi * D + j), __ldg(a.hi + qi * D + j), ap[j],
                                              a.consts->renc[2 * j], a.consts->renc[2 * j + 1]);
      } else {
        bd[0][j] = make_boxdim(__ldg(a.lo + qi * D + j), __ldg(a.hi + qi * D + j), ap[j], a.consts->renc[2 * j],
                               a.consts->renc[2 * j + 1]);
        narrow[0] |= bd[0][j].hd > 0.0f;
      }
    }
  }
#pragma unroll
  for (int k = 0; k < QT * NA; ++k) accsh[k * kBatchedThreads + tid] = 0.0;

  const int64_t s0 = (int64_t)blockIdx.y * a.split_len;
  const int64_t s1 = min(a.n, s0 + a.split_len);
  const int ntiles = (int)((s1 - s0 + kTilePts - 1) / kTilePts);
  if (tid == 0) {
    for (int st = 0; st < kBatchedStages; ++st) {
      mbar_init(&bar[st], 1);
      cnt[st] = 0;
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int k) {
    const int buf = k % kBatchedStages;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    mbar_arrive_expect_tx(&bar[buf], (uint32_t)(D * kTilePts * sizeof(float)));
#pragma unroll
    for (int j = 0; j < D; ++j)
      bulk_g2s(tile + (buf * D + j) * kTilePts, a.cols + (int64_t)j * a.ld + s0 + (int64_t)k * kTilePts,
               (uint32_t)(kTilePts * sizeof(float)), &bar[buf]);
  };
  if (tid == 0)
    for (int k = 0; k < kBatchedStages && k < ntiles; ++k) issue(k);

  // Culling (reading R15, large batches): sort the CTA's boxes by their kept fraction on the
  // split's first tile (narrow-dimension boxes last), so that the lanes of a warp walk alive
  // lists of similar length; each thread then takes the box perm_s[tid].
  // culling with R > 1 threads per box (phases own alternate mask words) is supported, but measured
  // no faster than the unculled small-batch path, so the host enables it for full CTAs only
  const bool cull = a.cull && QB >= 32;  // R <= kTileWords threads per box
  float2 cb[D];
  if (cull && R > 1) {  // small batches: the narrow/normal partition order, no re-sort
    int64_t qi = qbase + perm_s[slot];
    if (qi >= a.q) qi = a.q - 1;
    if (a.perm) qi = a.perm[qi];
#pragma unroll
    for (int j = 0; j < D; ++j)
      cb[j] = make_cullbox(__ldg(a.lo + qi * D + j), __ldg(a.hi + qi * D + j), ap[j], a.consts->renc[2 * j],
                           a.consts->renc[2 * j + 1]);
  }
  if (cull && R == 1) {
    __shared__ int key_s[kBatchedThreads];
    int64_t q0 = min(qbase + tid, a.q - 1);
    if (a.perm) q0 = a.perm[q0];
#pragma unroll
    for (int j = 0; j < D; ++j)
      cb[j] = make_cullbox(__ldg(a.lo + q0 * D + j), __ldg(a.hi + q0 * D + j), ap[j], a.consts->renc[2 * j],
                           a.consts->renc[2 * j + 1]);
    int cnt = 0;
    if (ntiles > 0) {
      mbar_wait_parity(&bar[0], 0u);
      const int64_t rem = s1 - s0;
      unsigned mk[kTileWords];
      if (epan)
        cull_tile_mask<D, true>(tile, rem < kTilePts ? (int)rem : kTilePts, ap, cb, mk);
      else
        cull_tile_mask<D, false>(tile, rem < kTilePts ? (int)rem : kTilePts, ap, cb, mk);
#pragma unroll
      for (int w = 0; w < kTileWords; ++w) cnt += __popc(mk[w]);
    }
    bool nar0 = false;
#pragma unroll
    for (int j = 0; j < D; ++j) {
      const float dy = (__ldg(a.hi + q0 * D + j) - __ldg(a.lo + q0 * D + j)) * ap[j];
      nar0 |= !epan && dy > 0.0f && dy < kNarrowY;
    }
    key_s[tid] = ((nar0 ? 512 : 0) + cnt) * kBatchedThreads + tid;  // unique keys: a deterministic order
    __syncthreads();
    for (int k = 2; k <= kBatchedThreads; k <<= 1)  // bitonic sort, ascending
      for (int jj = k >> 1; jj > 0; jj >>= 1) {
        const int ix = tid ^ jj;
        if (ix > tid) {
          const int x = key_s[tid], y = key_s[ix];
          if (((tid & k) == 0) == (x > y)) {
            key_s[tid] = y;
            key_s[ix] = x;
          }
        }
        __syncthreads();
      }
    const int sl = key_s[tid] % kBatchedThreads;
    perm_s[tid] = sl;
    int64_t qi = qbase + sl;
    if (qi >= a.q) qi = a.q - 1;
    if (a.perm) qi = a.perm[qi];
    narrow[0] = false;
#pragma unroll
    for (int j = 0; j < D; ++j) {
      const float l = __ldg(a.lo + qi * D + j), u = __ldg(a.hi + qi * D + j);
      if (epan) {
        bd[0][j] = make_boxdim<kEpanechnikov>(l, u, ap[j], a.consts->renc[2 * j], a.consts->renc[2 * j + 1]);
      } else {
        bd[0][j] = make_boxdim(l, u, ap[j], a.consts->renc[2 * j], a.consts->renc[2 * j + 1]);
        narrow[0] |= bd[0][j].hd > 0.0f;
      }
      cb[j] = make_cullbox(l, u, ap[j], a.consts->renc[2 * j], a.consts->renc[2 * j + 1]);
    }
    __syncthreads();
  }

  // One warp-uniform variant for the whole split: boxes with a narrow
  // dimension (rare) switch the warp to the general per-dimension path, so
  // the common path stays branch-free and the QT boxes interleave for ILP.
  bool my_narrow = false;
#pragma unroll
  for (int qq = 0; qq < QT; ++qq) my_narrow |= narrow[qq];
  const int mode = epan ? 2 : (__any_sync(0xffffffffu, my_narrow) ? 1 : 0);
  batched_tiles<D, GRAD, QT, PU>(a, tile, bar, cnt, accsh, bd, ap, cb, cull, s0, s1, ntiles, mode, phase, R, issue);

  // combine the R phases of each box in phase order, then
  // partials[(split*(NA) + comp) * q + qi]
  if (R > 1) __syncthreads();
  if (tid < QB) {
    const int64_t qs = qbase + perm_s[tid];
    if (qs < a.q) {
      const int64_t qi = a.perm ? a.perm[qs] : qs;
#pragma unroll
      for (int kk = 0; kk < NA; ++kk) {
        double t = 0.0;
        for (int ph = 0; ph < R; ++ph) t += accsh[kk * kBatchedThreads + ph * QB + tid];
        a.partials[((int64_t)blockIdx.y * NA + kk) * a.q + qi] = t;
      }
    }
  }
}

// ---------------------------------------------------------------- launchers
// forward declarations (scan_single_tma.cuh, scan_cells.cuh, included below)
template <int D>
cudaError_t launch_cells_single_t(bool grad, const ScanSingleArgs& a, int grid, cudaStream_t s);
template <int D, bool GRAD, int TILE, int STAGES, int OCC, bool CULL>
cudaError_t launch_single_tma_variant(const ScanSingleArgs& a, int grid, cudaStream_t s);

// culled single-box scan (every d): TMA tiles + a per-warp ring of kept points.
// Two stages; 2048-point tiles up to d = 10 (8 KB bulk copies per column: 4 KB / 2 KB copies
// measured 0.43 / 0.39 of HBM at d = 10 against 0.47, profiles/r02_experiments.md), 1024 / 512
// above (shared-memory budget); two CTAs per SM up to d = 5.
#ifndef KDE_TUNE_CULL_TILE
#define KDE_TUNE_CULL_TILE(d) ((d) <= 10 ? 2048 : ((d) <= 12 ? 1024 : 512))
#endif
#ifndef KDE_TUNE_CULL_STAGES
#define KDE_TUNE_CULL_STAGES(d) 2
#endif
#ifndef KDE_TUNE_CULL_OCC
#define KDE_TUNE_CULL_OCC(d) ((d) <= 5 ? 2 : 1)
#endif
__host__ __device__ constexpr int cull_tile(int d) { return KDE_TUNE_CULL_TILE(d); }
__host__ __device__ constexpr int cull_stages(int d) { return (void)d, KDE_TUNE_CULL_STAGES(d); }
__host__ __device__ constexpr int cull_occ(int d) { return KDE_TUNE_CULL_OCC(d); }

// cull on: the culled TMA variant;
// d <= 8: TMA-pipelined, warp-specialised variant (kSingleTile-point tiles, single_stages(d) stages,
// single_tma_occ(d) CTAs/SM);
// d > 8: register-streaming variant (measured faster or equal there).
template <int D>
cudaError_t launch_single_t(bool grad, const ScanSingleArgs& a, int grid, cudaStream_t s) {
  if (a.cull && a.ccols && !a.c_out) return launch_cells_single_t<D>(grad, a, grid, s);  // scan_cells.cuh
  if (a.cull) {
    return grad ? launch_single_tma_variant<D, true, cull_tile(D), cull_stages(D), cull_occ(D), true>(a, grid, s)
                : launch_single_tma_variant<D, false, cull_tile(D), cull_stages(D), cull_occ(D), true>(a, grid, s);
  }
  if constexpr (single_uses_tma(D)) {
    return grad
               ? launch_single_tma_variant<D, true, kSingleTile, single_stages(D), single_tma_occ(D), false>(a, grid, s)
               : launch_single_tma_variant<D, false, kSingleTile, single_stages(D), single_tma_occ(D), false>(a, grid,
                                                                                                              s);
  }
  if (grad)
    scan_single_kernel<D, true><<<grid, kSingleThreads, 0, s>>>(a);
  else
    scan_single_kernel<D, false><<<grid, kSingleThreads, 0, s>>>(a);
  return cudaGetLastError();
}

// tuning entry point (tools/tune_single.cu)
template <int D, bool GRAD, int VW, int OCC, bool PF>
cudaError_t launch_single_variant(const ScanSingleArgs& a, int grid, cudaStream_t s) {
  scan_single_kernel<D, GRAD, VW, OCC, PF><<<grid, kSingleThreads, 0, s>>>(a);
  return cudaGetLastError();
}

template <int D, bool GRAD, int QT = QT_for<D>::value, int MINB = MINB_for<D>::value, int PU = PU_for<D>::value>
cudaError_t launch_batched_tg(const ScanBatchedArgs& a, dim3 grid, cudaStream_t s) {
  constexpr size_t smem = batched_smem_bytes<D, GRAD, QT>();
  // the attribute belongs to the device context: set it once per device (bit per ordinal)
  static std::atomic<unsigned long long> attr_set{0ull};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const unsigned long long bit = 1ull << (dev & 63);
  if (!(attr_set.load(std::memory_order_acquire) & bit)) {
    e = cudaFuncSetAttribute(scan_batched_kernel<D, GRAD, QT, MINB, PU>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr_set.fetch_or(bit, std::memory_order_acq_rel);
  }
  scan_batched_kernel<D, GRAD, QT, MINB, PU><<<grid, kBatchedThreads, smem, s>>>(a);
  return cudaGetLastError();
}

// Grid for the batched scan: query tiles (256*QT boxes) x sample splits,
// about `waves` x MINB CTAs per SM; split_len is a tile multiple.
// boxes per CTA: the power of two QB in [16, 256] minimising the padded
// work ceil(q/QB)*QB, with a 3% penalty per halving (smaller QB re-reads the
// sample tiles for fewer boxes); 256 for large batches.
inline int batched_qb(int64_t q) {
  int best = kBatchedThreads;
  double best_cost = -1.0;
  double pen = 1.0;
  for (int qb = kBatchedThreads; qb >= 16; qb >>= 1, pen *= 1.03) {
    const double cost = (double)((q + qb - 1) / qb * qb) * pen;
    if (best_cost < 0.0 || cost < best_cost) {
      best = qb;
      best_cost = cost;
    }
  }
  return best;
}

inline void batched_grid(int64_t q, int64_t n, int qb, int minb, int num_sms, int waves, int64_t* qtiles,
                         int64_t* splits, int64_t* split_len) {
  *qtiles = (q + qb - 1) / qb;
  const int64_t ntile_pts = (n + kTilePts - 1) / kTilePts;
  const int64_t target = (int64_t)num_sms * minb * waves;
  int64_t sp = (target + *qtiles - 1) / *qtiles;
  if (sp > ntile_pts) sp = ntile_pts;
  if (sp < 1) sp = 1;
  int64_t len = ((n + sp - 1) / sp + kTilePts - 1) / kTilePts * kTilePts;
  if (len < kTilePts) len = kTilePts;
  sp = (n + len - 1) / len;
  if (sp < 1) sp = 1;
  *splits = sp;
  *split_len = len;
}

template <int D>
cudaError_t launch_batched_t(bool grad, const ScanBatchedArgs& a_in, int num_sms, int* splits_out, cudaStream_t s,
                             bool dry_run) {
  constexpr int QT = QT_for<D>::value;
  constexpr int MINB = MINB_for<D>::value;
  ScanBatchedArgs a = a_in;
  int64_t qtiles, splits, split_len;
  a.qb = batched_qb(a.q) * QT;
  batched_grid(a.q, a.n, a.qb, MINB, num_sms, 4, &qtiles, &splits, &split_len);
  if (splits_out) *splits_out = (int)splits;
  if (dry_run) return cudaSuccess;
  a.split_len = split_len;
  dim3 grid((unsigned)qtiles, (unsigned)splits);
  return grad ? launch_batched_tg<D, true>(a, grid, s) : launch_batched_tg<D, false>(a, grid, s);
}

}  // namespace kde

#include "scan_single_tma.cuh"
#include "scan_cells.cuh"

#define KDE_INSTANTIATE_SCAN(D)                                                                              \
  namespace kde {                                                                                            \
  template cudaError_t launch_single_t<D>(bool, const ScanSingleArgs&, int, cudaStream_t);                   \
  template cudaError_t launch_batched_t<D>(bool, const ScanBatchedArgs&, int, int*, cudaStream_t, bool);     \
  template cudaError_t launch_cells_t<D>(bool, const ScanCellsArgs&, int, int*, cudaStream_t, bool);         \
  }
