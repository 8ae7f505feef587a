// kernels.cu -- everything on the path except the scan itself:
//   sample layout (row-major -> SoA), Scott moments (eq. 3), constant
//   derivation, split / rank reduction + finalisation, loss epilogue (eq. 5,
//   14, 18, C.1), karma pass + ordered compaction (eq. 6-8, 19-20),
//   row replacement, the on-device Listing 1 step (Section 4.1)
//   and the harness box counter.
// All reductions use a fixed order, so results are bitwise reproducible.
#include <cooperative_groups.h>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>
#include <math_constants.h>

#include "common.cuh"
#include "kernels.cuh"
#include "peer.cuh"

namespace kde {
namespace cg = cooperative_groups;

// ------------------------------------------------------------ layout
// rows: device row-major [n][d]; cols: [d][ld].  Flags non-finite values.
__global__ void rows_to_cols_kernel(const float* __restrict__ rows, int64_t n, int d, float* __restrict__ cols,
                                    int64_t ld, int* bad) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  for (int j = 0; j < d; ++j) {
    const float x = rows[i * d + j];
    if (!isfinite(x)) *bad = 1;
    cols[(int64_t)j * ld + i] = x;
  }
}

// rows[r][j] -> cols[j][idx_local[r]], karma[idx_local[r]] = k_init
__global__ void scatter_rows_kernel(const int64_t* __restrict__ idx_local, const float* __restrict__ rows, int64_t k,
                                    int d, float* __restrict__ cols, int64_t ld, double* __restrict__ karma,
                                    double k_init) {
  const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= k) return;
  const int64_t i = idx_local[r];
  for (int j = 0; j < d; ++j) cols[(int64_t)j * ld + i] = rows[r * d + j];
  karma[i] = k_init;
}

__global__ void cols_to_rows_kernel(const float* __restrict__ cols, int64_t ld, int64_t n, int d,
                                    float* __restrict__ rows) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  for (int j = 0; j < d; ++j) rows[i * d + j] = cols[(int64_t)j * ld + i];
}

// ------------------------------------------------------------ column ranges
#define fenc fenc_range
#define fdec fdec_range

// enc[2j] = min, enc[2j+1] = max of column j over points [0, n) (accumulating)
__global__ void col_range_kernel(const float* __restrict__ cols, int64_t ld, int64_t n, unsigned* enc) {
  const int j = blockIdx.y;
  float lo = CUDART_INF_F, hi = -CUDART_INF_F;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const float x = cols[(int64_t)j * ld + i];
    lo = fminf(lo, x);
    hi = fmaxf(hi, x);
  }
  for (int o = 16; o > 0; o >>= 1) {
    lo = fminf(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = fmaxf(hi, __shfl_xor_sync(0xffffffffu, hi, o));
  }
  if ((threadIdx.x & 31) == 0) {
    atomicMin(enc + 2 * j, fenc(lo));
    atomicMax(enc + 2 * j + 1, fenc(hi));
  }
}

// widen the ranges by k host-supplied rows (row-major, device): a block reduces its rows in
// shared memory first, then one atomic per (block, column) -- not one per element
__global__ void row_range_kernel(const float* __restrict__ rows, int64_t k, int d, unsigned* enc) {
  __shared__ unsigned smin[kMaxDim], smax[kMaxDim];
  if (threadIdx.x < kMaxDim) {
    smin[threadIdx.x] = 0xFFFFFFFFu;
    smax[threadIdx.x] = 0u;
  }
  __syncthreads();
  unsigned lmin[kMaxDim], lmax[kMaxDim];
#pragma unroll
  for (int j = 0; j < kMaxDim; ++j) {
    lmin[j] = 0xFFFFFFFFu;
    lmax[j] = 0u;
  }
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < k; r += (int64_t)gridDim.x * blockDim.x) {
#pragma unroll
    for (int j = 0; j < kMaxDim; ++j)
      if (j < d) {
        const unsigned v = fenc(rows[r * d + j]);
        lmin[j] = min(lmin[j], v);
        lmax[j] = max(lmax[j], v);
      }
  }
#pragma unroll
  for (int j = 0; j < kMaxDim; ++j)
    if (j < d) {
      atomicMin(smin + j, lmin[j]);
      atomicMax(smax + j, lmax[j]);
    }
  __syncthreads();
  if (threadIdx.x < d) {
    atomicMin(enc + 2 * threadIdx.x, smin[threadIdx.x]);
    atomicMax(enc + 2 * threadIdx.x + 1, smax[threadIdx.x]);
  }
}


// device-resident replacement: the first min(*d_k, cap) GLOBAL indices of
// idx_global (e.g. the karma compaction output) receive rows[0..], karma reset.
// Indices outside this shard [row_offset, row_offset + n) are skipped.
__global__ void scatter_rows_dev_kernel(const int64_t* __restrict__ idx_global, const float* __restrict__ rows,
                                        const int64_t* __restrict__ d_k, int64_t cap, int d, float* __restrict__ cols,
                                        int64_t ld, int64_t n, int64_t row_offset, double* __restrict__ karma,
                                        double k_init, unsigned* __restrict__ enc) {
  const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t k = min(*d_k, cap);
  if (r >= k) return;
  const int64_t i = idx_global[r] - row_offset;
  if (i < 0 || i >= n) return;
  for (int j = 0; j < d; ++j) {
    const float x = rows[r * d + j];
    cols[(int64_t)j * ld + i] = x;
    atomicMin(enc + 2 * j, fenc(x));
    atomicMax(enc + 2 * j + 1, fenc(x));
  }
  karma[i] = k_init;
}

// ------------------------------------------------------------ Scott moments
// Per (block, column) fp64 Welford over a contiguous chunk, Chan merge in a
// fixed tree inside the block.  out[(j*nb + b)*3 + {0,1,2}] = (count, mean, M2).
__device__ __forceinline__ void chan_merge(double& na, double& ma, double& m2a, double nb, double mb, double m2b) {
  if (nb == 0.0) return;
  if (na == 0.0) {
    na = nb; ma = mb; m2a = m2b;
    return;
  }
  const double n = na + nb;
  const double delta = mb - ma;
  ma = ma + delta * (nb / n);
  m2a = m2a + m2b + delta * delta * (na * nb / n);
  na = n;
}

__global__ void moments_partial_kernel(const float* __restrict__ cols, int64_t ld, int64_t n, int64_t chunk,
                                       double* __restrict__ out) {
  const int j = blockIdx.y, b = blockIdx.x, nb = gridDim.x;
  const int64_t a0 = (int64_t)b * chunk;
  const int64_t a1 = min(n, a0 + chunk);
  double cnt = 0.0, mean = 0.0, m2 = 0.0;
  for (int64_t i = a0 + threadIdx.x; i < a1; i += blockDim.x) {
    const double x = (double)cols[(int64_t)j * ld + i];
    cnt += 1.0;
    const double delta = x - mean;
    mean += delta / cnt;
    m2 += delta * (x - mean);
  }
  __shared__ double sc[256], sm[256], s2[256];
  sc[threadIdx.x] = cnt; sm[threadIdx.x] = mean; s2[threadIdx.x] = m2;
  __syncthreads();
  for (int o = blockDim.x / 2; o > 0; o >>= 1) {
    if (threadIdx.x < o) {
      double na = sc[threadIdx.x], ma = sm[threadIdx.x], m2a = s2[threadIdx.x];
      chan_merge(na, ma, m2a, sc[threadIdx.x + o], sm[threadIdx.x + o], s2[threadIdx.x + o]);
      sc[threadIdx.x] = na; sm[threadIdx.x] = ma; s2[threadIdx.x] = m2a;
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    double* o = out + ((int64_t)j * nb + b) * 3;
    o[0] = sc[0]; o[1] = sm[0]; o[2] = s2[0];
  }
}

// Sequential Chan merge of np partials per column (fixed order) -> mom[j*3..].
__global__ void moments_merge_kernel(const double* __restrict__ part, int np, int d, double* __restrict__ mom) {
  const int j = threadIdx.x;
  if (j >= d) return;
  double na = 0.0, ma = 0.0, m2a = 0.0;
  for (int b = 0; b < np; ++b) {
    const double* p = part + ((int64_t)j * np + b) * 3;
    chan_merge(na, ma, m2a, p[0], p[1], p[2]);
  }
  mom[j * 3 + 0] = na; mom[j * 3 + 1] = ma; mom[j * 3 + 2] = m2a;
}

// Merge per-rank moments gathered as [rank][d][3] in rank order.
__global__ void moments_merge_ranks_kernel(const double* __restrict__ g, int world, int d, double* __restrict__ mom) {
  const int j = threadIdx.x;
  if (j >= d) return;
  double na = 0.0, ma = 0.0, m2a = 0.0;
  for (int r = 0; r < world; ++r) {
    const double* p = g + ((int64_t)r * d + j) * 3;
    chan_merge(na, ma, m2a, p[0], p[1], p[2]);
  }
  mom[j * 3 + 0] = na; mom[j * 3 + 1] = ma; mom[j * 3 + 2] = m2a;
}

__device__ void set_consts_dev(DevConsts* c, int j, double h) {
  const double kSqrtLog2e = 1.2011224087864498;  // sqrt(log2 e)
  const double kSqrtPi = 1.7724538509055160273;
  const double kSqrt2 = 1.4142135623730950488;
  c->h[j] = h;
  if (c->kernel == kEpanechnikov) {  // reading R14: v = (b - t)/h, dD/dh = -(3/(4h)) Delta (1 - S)
    c->ap[j] = (float)(1.0 / h);
    c->gconst[j] = -0.75 / h;
  } else {
    c->ap[j] = (float)(kSqrtLog2e / (kSqrt2 * h));
    c->gconst[j] = 1.0 / (kSqrtPi * kSqrtLog2e * h);
  }
}

__global__ void set_kernel_type_kernel(int kernel, int d, DevConsts* c) {
  if (threadIdx.x == 0) c->kernel = kernel;
  __syncthreads();
  const int j = threadIdx.x;
  if (j < d) set_consts_dev(c, j, c->h[j]);
}

// eq. (3): h_j = s^(-1/(d+4)) sigma_j, population sigma.
__global__ void scott_kernel(const double* __restrict__ mom, int d, DevConsts* c, int* bad) {
  const int j = threadIdx.x;
  if (j >= d) return;
  const double n = mom[j * 3 + 0];
  const double sigma = sqrt(mom[j * 3 + 2] / n);
  const double h = pow(n, -1.0 / (d + 4.0)) * sigma;
  if (!(h >= 1e-30 && h <= 1e30)) *bad = 1;  // e.g. a constant column
  set_consts_dev(c, j, h);
}

__global__ void set_consts_kernel(HVec hv, int d, DevConsts* c) {
  const int j = threadIdx.x;
  if (j < d) set_consts_dev(c, j, hv.v[j]);
}

// ------------------------------------------------------------ reductions
// sums[qi][k] = sum_{s in split order} partials[(s*NA + k)*q + qi]; with
// finalisation (world == 1): est[qi] = S_0/N, dpdh[qi][j] = S_j gconst_j / N.
__global__ void reduce_splits_kernel(const double* __restrict__ partials, int splits, int64_t q, int na,
                                     double* __restrict__ sums, const PeerArgs* __restrict__ peer) {
  const int64_t qi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t pe = peer ? peer_next_epoch(*peer) : 0;
  if (qi < q)
    for (int k = 0; k < na; ++k) {
      double t = 0.0;
      for (int s = 0; s < splits; ++s) t += partials[((int64_t)s * na + k) * q + qi];
      if (peer)
        peer_store(*peer, pe, qi * na + k, t);  // fused exchange: straight into every rank's window
      else
        sums[qi * na + k] = t;
    }
  if (!peer) return;
  __shared__ bool last_s;
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) last_s = atomicAdd(peer->count + 2, 1u) == gridDim.x - 1;
  __syncthreads();
  if (last_s && threadIdx.x == 0) {  // every block's stores are fenced: flags up
    peer->count[2] = 0u;
    peer_release(*peer, pe);
  }
}

// The same sums for few outputs and many splits (small batches over the cells scan: q x na outputs,
// thousands of splits): one warp per output, lane l sums the splits s = l (mod 32) in increasing order,
// then a fixed butterfly -- deterministic, and ~32x shorter dependent load chains than a thread per
// output.
__global__ void reduce_splits_wide_kernel(const double* __restrict__ partials, int splits, int64_t q, int na,
                                          double* __restrict__ sums, const PeerArgs* __restrict__ peer) {
  const int64_t o = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;  // output = qi * na + k
  const int lane = threadIdx.x & 31;
  const uint64_t pe = peer ? peer_next_epoch(*peer) : 0;
  if (o < q * na) {  // warp-uniform
    const int64_t qi = o / na;
    const int k = (int)(o % na);
    double t = 0.0;
    for (int s = lane; s < splits; s += 32) t += partials[((int64_t)s * na + k) * q + qi];
#pragma unroll
    for (int w = 16; w > 0; w >>= 1) t += __shfl_xor_sync(0xffffffffu, t, w);
    if (lane == 0) {
      if (peer)
        peer_store(*peer, pe, qi * na + k, t);
      else
        sums[qi * na + k] = t;
    }
  }
  if (!peer) return;
  __shared__ bool last_s;
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) last_s = atomicAdd(peer->count + 2, 1u) == gridDim.x - 1;
  __syncthreads();
  if (last_s && threadIdx.x == 0) {
    peer->count[2] = 0u;
    peer_release(*peer, pe);
  }
}

// The cells scan's partials: row entry r = g * QG + i holds the box at probe-sorted position
// pos = g + ngroups * i (perm[pos], or pos itself); entries with pos >= q are padding.
__device__ __forceinline__ int64_t cells_entry_box(int64_t r, int qg, int ngroups, int64_t q, const int* perm) {
  const int64_t g = r / qg, i = r % qg;
  const int64_t pos = g + (int64_t)ngroups * i;
  if (pos >= q) return -1;
  return perm ? (int64_t)perm[pos] : pos;
}
__global__ void reduce_splits_mapped_kernel(const double* __restrict__ partials, int splits, int64_t qpad, int64_t q,
                                            int na, int qg, int ngroups, const int* __restrict__ perm,
                                            double* __restrict__ sums, const PeerArgs* __restrict__ peer, int wide) {
  const uint64_t pe = peer ? peer_next_epoch(*peer) : 0;
  if (wide) {  // a warp per (entry, component): lanes over splits, fixed butterfly
    const int64_t o = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (o < qpad * na) {
      const int64_t r = o / na;
      const int k = (int)(o % na);
      const int64_t qi = cells_entry_box(r, qg, ngroups, q, perm);
      if (qi >= 0) {  // warp-uniform
        double t = 0.0;
        for (int s = lane; s < splits; s += 32) t += partials[((int64_t)s * na + k) * qpad + r];
#pragma unroll
        for (int w = 16; w > 0; w >>= 1) t += __shfl_xor_sync(0xffffffffu, t, w);
        if (lane == 0) {
          if (peer)
            peer_store(*peer, pe, qi * na + k, t);
          else
            sums[qi * na + k] = t;
        }
      }
    }
  } else {  // a thread per entry (coalesced across entries)
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t qi = r < qpad ? cells_entry_box(r, qg, ngroups, q, perm) : -1;
    if (qi >= 0)
      for (int k = 0; k < na; ++k) {
        double t = 0.0;
        for (int s = 0; s < splits; ++s) t += partials[((int64_t)s * na + k) * qpad + r];
        if (peer)
          peer_store(*peer, pe, qi * na + k, t);
        else
          sums[qi * na + k] = t;
      }
  }
  if (!peer) return;
  __shared__ bool last_s;
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) last_s = atomicAdd(peer->count + 2, 1u) == gridDim.x - 1;
  __syncthreads();
  if (last_s && threadIdx.x == 0) {
    peer->count[2] = 0u;
    peer_release(*peer, pe);
  }
}

// gathered[r][q][na] summed in rank order -> sums[q][na]
__global__ void combine_ranks_kernel(const double* __restrict__ gathered, int world, int64_t q, int na,
                                     double* __restrict__ sums) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= q * na) return;
  double t = 0.0;
  for (int r = 0; r < world; ++r) t += gathered[(int64_t)r * q * na + e];
  sums[e] = t;
}

__global__ void finalize_kernel(const double* __restrict__ sums, int64_t q, int d, int na, const DevConsts* c,
                                double n_global, double* __restrict__ est, double* __restrict__ dpdh) {
  const int64_t qi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (qi >= q) return;
  est[qi] = sums[qi * na] / n_global;
  if (dpdh && na > 1)
    for (int j = 0; j < d; ++j) dpdh[qi * d + j] = sums[qi * na + 1 + j] * c->gconst[j] / n_global;
}

// ------------------------------------------------------------ losses (Appendix C.1)
__device__ __forceinline__ double sgn3(double a, double b) { return a < b ? -1.0 : (a > b ? 1.0 : 0.0); }

__device__ void loss_eval(int kind, double lambda, double phat, double p, double* L, double* dL) {
  switch (kind) {
    case 0: *L = (phat - p) * (phat - p); *dL = 2.0 * (phat - p); break;
    case 1: *L = fabs(phat - p); *dL = sgn3(phat, p); break;
    case 2: *L = fabs(phat - p) / (lambda + p); *dL = sgn3(phat, p) / (lambda + p); break;
    case 3: {
      const double r = (phat - p) / (lambda + p);
      *L = r * r;
      *dL = 2.0 * r / (lambda + p);  // reading R7: true derivative of the printed loss
    } break;
    default: {
      const double r = log(lambda + phat) - log(lambda + p);
      *L = r * r;
      *dL = 2.0 * r / (lambda + phat);
    }
  }
}

// eq. (5): loss = (1/q) sum L_k; eq. (14): grad_j = (1/q) sum L'_k dp_k/dh_j;
// eq. (18): x h_j in log mode.  One block, fixed strided order + fixed tree.
__global__ void loss_epilogue_kernel(const double* __restrict__ est, const double* __restrict__ dpdh,
                                     const double* __restrict__ true_sel, int64_t q, int d, int kind, double lambda,
                                     int log_bw, const DevConsts* c, double* __restrict__ loss_out,
                                     double* __restrict__ grad_out) {
  constexpr int T = 512;
  __shared__ double red[T / 32][kMaxDim + 1];
  double acc[kMaxDim + 1];
  for (int k = 0; k <= d; ++k) acc[k] = 0.0;
  for (int64_t qi = threadIdx.x; qi < q; qi += T) {
    double L, dL;
    loss_eval(kind, lambda, est[qi], true_sel[qi], &L, &dL);
    acc[0] += L;
    for (int j = 0; j < d; ++j) acc[1 + j] += dL * dpdh[qi * d + j];
  }
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int k = 0; k <= d; ++k) {
    double v = acc[k];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (lane == 0) red[warp][k] = v;
  }
  __syncthreads();
  if (threadIdx.x <= d) {
    double t = 0.0;
    for (int w = 0; w < T / 32; ++w) t += red[w][threadIdx.x];
    t /= (double)q;
    if (threadIdx.x == 0) {
      *loss_out = t;
    } else {
      const int j = threadIdx.x - 1;
      grad_out[j] = log_bw ? t * c->h[j] : t;
    }
  }
}

// ------------------------------------------------------------ karma
// Each block owns a contiguous range of kKarmaPts points, visited in ascending
// order (pass-major, thread-minor), so the flag bitmap words are in index order.
// eq. (19)-(20) threshold computed per block in fp64 from (lo, hi, h).
__device__ double epan_cdf_dev(double v) {
  if (v <= -1.0) return 0.0;
  if (v >= 1.0) return 1.0;
  return (2.0 + 3.0 * v - v * v * v) / 4.0;
}

// eq. (19)-(20): p_max = prod_j M_j(centre), thr = max_j p_max M_j(face) / M_j(centre)
// (Gaussian: M(centre) = erf(w / (2 sqrt2 h)), M(face) = erf(w / (sqrt2 h)) / 2;
//  Epanechnikov: the same derivation with its CDF).
__device__ double thr20_dev(const float* lo, const float* hi, int d, const DevConsts* c) {
  const double kSqrt2 = 1.4142135623730950488;
  double pmax = 1.0, best = 0.0;
  for (int j = 0; j < d; ++j) {
    const double w = (double)hi[j] - (double)lo[j];
    if (!(w > 0.0)) return CUDART_INF;  // zero width: shortcut disabled (reading R5)
    double centre, face;
    if (c->kernel == kEpanechnikov) {
      centre = isinf(w) ? 1.0 : epan_cdf_dev(w / (2.0 * c->h[j])) - epan_cdf_dev(-w / (2.0 * c->h[j]));
      face = isinf(w) ? 0.5 : epan_cdf_dev(w / c->h[j]) - 0.5;
    } else {
      centre = erf(w / (2.0 * kSqrt2 * c->h[j]));
      face = isinf(w) ? 0.5 : 0.5 * erf(w / (kSqrt2 * c->h[j]));
    }
    pmax *= centre;
    best = fmax(best, face / centre);
  }
  if (!(pmax > 0.0)) return CUDART_INF;
  return pmax * best;
}

#ifndef KDE_TUNE_KARMA_MINB
#define KDE_TUNE_KARMA_MINB 4  // 64 registers, 4 blocks per SM
#endif
// Each block owns kKarmaPts contiguous points; a thread takes KV = 4 consecutive points per pass
// (one float4 of p^(i), two double2 of K: 128-bit loads and stores, the karma array is padded to
// the column length), all passes' loads issued before any arithmetic.  Flag bits are assembled
// into index-order bitmap words with three shuffles (8 lanes x 4 points = one word).  The last
// block to finish turns the per-block counts into exclusive offsets (one O(nb) scan), so the
// compaction needs no prefix of its own.
constexpr int kKarmaKV = 4;
__global__ void __launch_bounds__(kKarmaThreads, KDE_TUNE_KARMA_MINB)
    karma_kernel(const float* __restrict__ cvals, double* __restrict__ karma, int64_t n, double n_global,
                 const double* __restrict__ phat_ptr, const double* __restrict__ p_ptr, KarmaParamsDev kp,
                 const float* lo, const float* hi, int d, const DevConsts* c, uint32_t* __restrict__ bitmap,
                 int32_t* __restrict__ block_counts, int64_t* __restrict__ block_offsets, unsigned* __restrict__ kdone,
                 int nb) {
  __shared__ double thr_s;
  __shared__ int32_t wcount[kKarmaThreads / 32];
  __shared__ bool last_s;
  const double p = *p_ptr;
  if (threadIdx.x == 0) thr_s = (kp.empty_region && p == 0.0) ? thr20_dev(lo, hi, d, c) : CUDART_INF;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  __syncthreads();
  const double phat = *phat_ptr;
  double L_full, dummy;
  loss_eval(kp.loss, kp.lambda, phat, p, &L_full, &dummy);
  const double thr = thr_s;
  const int64_t base = (int64_t)blockIdx.x * kKarmaPts;
  constexpr int PASSES = kKarmaPts / (kKarmaThreads * kKarmaKV);
#ifndef KDE_TUNE_KARMA_PB
#define KDE_TUNE_KARMA_PB 2
#endif
  constexpr int PB = KDE_TUNE_KARMA_PB;  // passes per load batch
  static_assert(PASSES % PB == 0, "karma load batches");
  const double inv_nm1 = 1.0 / (n_global - 1.0);
  int32_t my = 0;
#pragma unroll 1
  for (int r0 = 0; r0 < PASSES; r0 += PB) {
    float4 cv[PB];
    double2 kv[PB][2];
#pragma unroll
    for (int r = 0; r < PB; ++r) {
      const int64_t i = base + ((int64_t)(r0 + r) * kKarmaThreads + threadIdx.x) * kKarmaKV;
      if (i < n) {  // i is a multiple of 4; c and K are padded past n
        cv[r] = __ldcs(reinterpret_cast<const float4*>(cvals + i));
        kv[r][0] = __ldcs(reinterpret_cast<const double2*>(karma + i));
        kv[r][1] = __ldcs(reinterpret_cast<const double2*>(karma + i + 2));
      } else {
        cv[r] = make_float4(0.f, 0.f, 0.f, 0.f);
        kv[r][0] = kv[r][1] = make_double2(0.0, 0.0);
      }
    }
#pragma unroll
    for (int r = 0; r < PB; ++r) {
      const int64_t i = base + ((int64_t)(r0 + r) * kKarmaThreads + threadIdx.x) * kKarmaKV;
      const float cc[4] = {cv[r].x, cv[r].y, cv[r].z, cv[r].w};
      double kk[4] = {kv[r][0].x, kv[r][0].y, kv[r][1].x, kv[r][1].y};
      unsigned nib = 0u;
#pragma unroll
      for (int v = 0; v < kKarmaKV; ++v) {
        if (i + v < n) {
          const double ci = (double)cc[v];
          const double p_minus = (phat * n_global - ci) * inv_nm1;  // eq. (6)
          double L_minus;
          loss_eval(kp.loss, kp.lambda, p_minus, p, &L_minus, &dummy);
          kk[v] = fmin(kk[v] + (L_minus - L_full), kp.k_max);  // eq. (7)-(8)
          const bool flag = (kk[v] < kp.threshold) || (ci >= thr);
          nib |= (unsigned)flag << v;
        }
      }
      if (i < n) {
        __stcs(reinterpret_cast<double2*>(karma + i), make_double2(kk[0], kk[1]));
        __stcs(reinterpret_cast<double2*>(karma + i + 2), make_double2(kk[2], kk[3]));
      }
      // word w of this warp's 128 points = nibbles of lanes 8w .. 8w+7
      unsigned word = nib << (4 * (lane & 7));
      word |= __shfl_xor_sync(0xffffffffu, word, 1);
      word |= __shfl_xor_sync(0xffffffffu, word, 2);
      word |= __shfl_xor_sync(0xffffffffu, word, 4);
      if ((lane & 7) == 0) {
        const int64_t w0 = (base + ((int64_t)(r0 + r) * kKarmaThreads + warp * 32) * kKarmaKV) / 32;
        bitmap[w0 + (lane >> 3)] = word;
        my += __popc(word);
      }
    }
  }
  for (int o = 8; o < 32; o <<= 1) my += __shfl_xor_sync(0xffffffffu, my, o);
  if (lane == 0) wcount[warp] = my;
  __syncthreads();
  if (threadIdx.x == 0) {
    int32_t t = 0;
    for (int w = 0; w < kKarmaThreads / 32; ++w) t += wcount[w];
    block_counts[blockIdx.x] = t;
    __threadfence();
    last_s = atomicAdd(kdone, 1u) == (unsigned)nb - 1;
  }
  __syncthreads();
  if (!last_s) return;
  __threadfence();
  // last block: exclusive offsets of the nb block counts, fixed order (each thread a contiguous run)
  __shared__ int64_t run_s[kKarmaThreads];
  const int per = (nb + kKarmaThreads - 1) / kKarmaThreads;
  const int b0 = min(nb, (int)threadIdx.x * per), b1 = min(nb, b0 + per);
  int64_t t = 0;
  for (int b = b0; b < b1; ++b) t += __ldcg(block_counts + b);
  run_s[threadIdx.x] = t;
  __syncthreads();
  if (threadIdx.x == 0) {
    int64_t acc = 0;
    for (int k = 0; k < kKarmaThreads; ++k) {
      const int64_t v = run_s[k];
      run_s[k] = acc;
      acc += v;
    }
    block_offsets[nb] = acc;  // total
    *kdone = 0u;
  }
  __syncthreads();
  int64_t o = run_s[threadIdx.x];
  for (int b = b0; b < b1; ++b) {
    block_offsets[b] = o;
    o += __ldcg(block_counts + b);
  }
}

__device__ __noinline__ void online_update_body(const double* __restrict__ ret, const double* __restrict__ p_ptr,
                                   const OnlineParamsDev& op, int d, OnlineState* st, DevConsts* c);

// Ordered compaction of the karma flags: block b writes the ascending GLOBAL
// indices of its flagged points at offset sum_{b' < b} count[b'] (computed by
// the block itself -- no separate scan pass); at most cap are written.  The
// last block to finish writes the total and runs the optional tail of a
// device-resident streaming step: the Listing 1 bandwidth update and the
// replacement of the first min(total, cap) flagged points by tail.rows.
#ifndef KDE_TUNE_COMPACT_MINB
#define KDE_TUNE_COMPACT_MINB 8
#endif
__global__ void __launch_bounds__(kKarmaThreads, KDE_TUNE_COMPACT_MINB) compact_fused_kernel(const uint32_t* __restrict__ bitmap, int64_t n, const int64_t* __restrict__ block_offsets,
                                     int nb, int64_t row_offset, int64_t* __restrict__ idx_out, int64_t cap,
                                     int64_t* __restrict__ total_out, unsigned* __restrict__ done, StreamTail tail) {
  constexpr int W = kKarmaPts / 32;  // bitmap words per block
  constexpr int WPL = W / 32;
  __shared__ int32_t wpre[W];
  __shared__ uint32_t wbits[W];  // the block's bitmap words, read once by warp 0
  __shared__ int64_t off_s;
  __shared__ bool last_s;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) off_s = __ldg(block_offsets + blockIdx.x);  // exclusive offset (karma_kernel's last block)
  const int64_t wbase = (int64_t)blockIdx.x * W;
  const int64_t nwords = (n + 31) / 32;
  if (tid < 32) {  // exclusive prefix of the block's word popcounts
    int c[WPL], tot = 0;
#pragma unroll
    for (int k = 0; k < WPL; ++k) {
      const int64_t w = wbase + WPL * lane + k;
      const uint32_t word = w < nwords ? bitmap[w] : 0u;
      wbits[WPL * lane + k] = word;
      c[k] = __popc(word);
      tot += c[k];
    }
    int incl = tot;
#pragma unroll
    for (int k = 1; k < 32; k <<= 1) {
      const int v = __shfl_up_sync(0xffffffffu, incl, k);
      if (lane >= k) incl += v;
    }
    int run = incl - tot;
#pragma unroll
    for (int k = 0; k < WPL; ++k) {
      wpre[WPL * lane + k] = run;
      run += c[k];
    }
  }
  __syncthreads();
  const int64_t off = off_s;
#pragma unroll 4
  for (int w = warp; w < W; w += kKarmaThreads / 32) {
    const uint32_t word = wbits[w];  // 0 past the end of the bitmap
    if (word & (1u << lane)) {
      const int64_t pos = off + wpre[w] + __popc(word & ((1u << lane) - 1u));
      if (pos < cap) idx_out[pos] = row_offset + (wbase + w) * 32 + lane;
    }
  }
  // last block: total + optional streaming tail
  __threadfence();
  __syncthreads();
  if (tid == 0) last_s = atomicAdd(done, 1u) == (unsigned)nb - 1;
  __syncthreads();
  if (!last_s) return;
  __threadfence();
  if (tid == 0) {
    const int64_t tot = __ldg(block_offsets + nb);
    off_s = tot;
    if (total_out) *total_out = tot;
    *done = 0u;
  }
  __syncthreads();
  if (tail.online) online_update_body(tail.ret, tail.p, tail.op, tail.d, tail.st, tail.c);
  if (tail.rows) {
    __shared__ unsigned rmin[kMaxDim], rmax[kMaxDim];
    if (tid < kMaxDim) {
      rmin[tid] = 0xFFFFFFFFu;
      rmax[tid] = 0u;
    }
    __syncthreads();
    const int64_t k = min(off_s, cap);
    const float* __restrict__ rows = tail.rows;
    float* __restrict__ cols = tail.cols;
    // one flagged point per thread: its index and all d coordinates are loaded before any
    // store, so the block waits for ~2 memory latencies instead of 2 per (point, dim) pass
    for (int64_t r = tid; r < k; r += kKarmaThreads) {
      const int64_t i = __ldcg(idx_out + r) - row_offset;
      float x[kMaxDim];
#pragma unroll
      for (int j = 0; j < kMaxDim; ++j) x[j] = j < tail.d ? rows[r * tail.d + j] : 0.0f;
#pragma unroll
      for (int j = 0; j < kMaxDim; ++j) {
        if (j < tail.d) {
          cols[(int64_t)j * tail.ld + i] = x[j];
          atomicMin(rmin + j, fenc(x[j]));  // shared-memory range of the new rows
          atomicMax(rmax + j, fenc(x[j]));
        }
      }
      tail.karma[i] = tail.k_init;
    }
    __syncthreads();
    if (tid < tail.d && k > 0) {
      atomicMin(tail.c->renc + 2 * tid, rmin[tid]);
      atomicMax(tail.c->renc + 2 * tid + 1, rmax[tid]);
    }
  }
}

// ------------------------------------------------------------ online bandwidth (Listing 1, reconstructed)
// ret: [1+d] = (p_hat, dp/dh_j) of the retained query.  Adds L' dp/dh (x h in
// log mode, eq. 18) to the mini-batch; every `minibatch` queries applies the
// RMSprop / Rprop step of P:L179-183 and re-derives the constants.
// One Listing 1 step, executed by one whole block (thread j < d owns dimension j).  Not inlined:
// the standalone kernel and the fused streaming step run the same machine code, so their
// bandwidths stay bit-identical (inlined copies may contract log/exp differently).
__device__ __noinline__ void online_update_body(const double* __restrict__ ret, const double* __restrict__ p_ptr,
                                   const OnlineParamsDev& op, int d, OnlineState* st, DevConsts* c) {
  const int j = threadIdx.x;
  const double p = *p_ptr;
  double L, dL;
  loss_eval(op.loss, op.lambda, ret[0], p, &L, &dL);
  const int count = st->count + 1;
  const bool apply = count >= op.minibatch;
  __syncthreads();  // every thread has read st->count
  if (j < d) {
    double g = dL * ret[1 + j];
    if (op.log_bw) g *= c->h[j];
    const double acc = st->acc[j] + g;
    if (!apply) {
      st->acc[j] = acc;
    } else {
      const double gm = acc / (double)op.minibatch;                        // line 12
      const double ms = op.alpha * st->ms[j] + (1.0 - op.alpha) * gm * gm;  // line 14
      double lr = st->lr[j];
      if (gm * st->gprev[j] > 0.0) lr = fmin(lr * op.lr_inc, op.lr_max);  // lines 15-16
      else if (gm * st->gprev[j] < 0.0) lr = fmax(lr * op.lr_dec, op.lr_min);
      double step = ms > 0.0 ? lr * gm / sqrt(ms) : 0.0;  // line 17
      double h = c->h[j];
      if (op.log_bw) {
        h = exp(log(h) - step);
      } else {
        if (step > h / 2.0) step = h / 2.0;  // positivity safeguard
        h = h - step;
      }
      set_consts_dev(c, j, h);
      st->ms[j] = ms;
      st->lr[j] = lr;
      st->gprev[j] = gm;
      st->acc[j] = 0.0;
    }
  }
  if (j == 0) {
    st->count = apply ? 0 : count;
    st->updated = apply ? 1 : 0;
  }
  __syncthreads();
}

__global__ void online_update_kernel(const double* __restrict__ ret, const double* __restrict__ p_ptr,
                                     OnlineParamsDev op, int d, OnlineState* st, DevConsts* c) {
  online_update_body(ret, p_ptr, op, d, st, c);
}

// ------------------------------------------------------------ karma pass, one cooperative kernel
// The whole feedback tail of a query in ONE persistent launch (cooperative: all CTAs co-resident,
// grid-wide barriers).  The points are cut into passes of 1024 (256 threads x 4 consecutive points);
// CTA b owns the contiguous passes [b P / G, (b + 1) P / G) -- balanced to one pass.
//   phase 1  karma (eq. 6-8) and flags (R4, eq. 20): 128-bit loads of p^(i) and K, index-order
//            bitmap words (8 lanes x 4 points per word), a per-CTA flag count;
//   barrier  -> the CTA's offset is the sum of the counts of the CTAs before it;
//   phase 2  ordered compaction of its bitmap words into ascending GLOBAL indices (128 words per
//            step: warp 0 forms the popcount prefix, all warps write);
//   barrier  -> phase 3 (streaming step only): CTA 0 runs the Listing 1 step, all CTAs replace the
//            first min(total, cap) flagged points by tail.rows.
#ifndef KDE_TUNE_COOP_THREADS
#define KDE_TUNE_COOP_THREADS 256
#endif
#ifndef KDE_TUNE_COOP_MINB
#define KDE_TUNE_COOP_MINB 2  // 128 registers, 2 CTAs per SM (room for PB = 4)
#endif
constexpr int kCoopThreads = KDE_TUNE_COOP_THREADS;
constexpr int kCoopPass = kCoopThreads * kKarmaKV;  // points per pass (kCoopThreads / 8 bitmap words)

struct KarmaCoopArgs {
  const float* cvals;
  double* karma;
  int64_t n;
  double n_global;
  const double* phat;
  const double* p;
  KarmaParamsDev kp;
  const float* lo;
  const float* hi;
  int d;
  const DevConsts* c;
  uint32_t* bitmap;
  int32_t* cta_counts;  // [grid]
  int64_t row_offset;
  int64_t* idx_out;
  int64_t cap;
  int64_t* total_out;
  StreamTail tail;
};

__global__ void __launch_bounds__(kCoopThreads, KDE_TUNE_COOP_MINB) karma_coop_kernel(const KarmaCoopArgs a) {
  cg::grid_group grid = cg::this_grid();
  constexpr int W = 128;  // bitmap words per compaction step
  constexpr int WPL = W / 32;
  __shared__ double thr_s;
  __shared__ int64_t red_s[2][kCoopThreads / 32];
  __shared__ int32_t wpre[W];
  __shared__ uint32_t wbits[W];
  __shared__ int32_t segtot_s;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int G = gridDim.x, b = blockIdx.x;
  const int64_t n = a.n;
  const int64_t P = (n + kCoopPass - 1) / kCoopPass;
  const int64_t p0 = (int64_t)b * P / G, p1 = (int64_t)(b + 1) * P / G;
  const KarmaParamsDev kp = a.kp;
  const double p = *a.p;
  if (tid == 0) thr_s = (kp.empty_region && p == 0.0) ? thr20_dev(a.lo, a.hi, a.d, a.c) : CUDART_INF;
  __syncthreads();
  const double phat = *a.phat;
  double L_full, dummy;
  loss_eval(kp.loss, kp.lambda, phat, p, &L_full, &dummy);
  const double thr = thr_s;
  const double inv_nm1 = 1.0 / (a.n_global - 1.0);
  // ---------------- phase 1: karma + flags
  int32_t my = 0;
#ifndef KDE_TUNE_COOP_PB
#define KDE_TUNE_COOP_PB 4  // 4 passes of loads in flight (ncu: 25.3 vs 27.6 us at 2^22 with 2, profiles/r02_experiments.md)
#endif
  constexpr int PB = KDE_TUNE_COOP_PB;  // passes whose loads are in flight together
#if KDE_TUNE_L2KEEP
  const uint64_t pol_keep = l2_policy_evict_last();  // K and p^(i) stay in L2 across queries
#endif
#pragma unroll 1
  for (int64_t q0 = p0; q0 < p1; q0 += PB) {
    float4 cv[PB];
    double2 kv[PB][2];
#pragma unroll
    for (int r = 0; r < PB; ++r) {
      const int64_t i = (q0 + r) * kCoopPass + (int64_t)tid * kKarmaKV;
      if (q0 + r < p1 && i < n) {  // i is a multiple of 4; c and K are padded past n
#if KDE_TUNE_L2KEEP
        cv[r] = ld_keep_f4(a.cvals + i, pol_keep);
        kv[r][0] = ld_keep_d2(a.karma + i, pol_keep);
        kv[r][1] = ld_keep_d2(a.karma + i + 2, pol_keep);
#else
        cv[r] = __ldcs(reinterpret_cast<const float4*>(a.cvals + i));
        kv[r][0] = __ldcs(reinterpret_cast<const double2*>(a.karma + i));
        kv[r][1] = __ldcs(reinterpret_cast<const double2*>(a.karma + i + 2));
#endif
      } else {
        cv[r] = make_float4(0.f, 0.f, 0.f, 0.f);
        kv[r][0] = kv[r][1] = make_double2(0.0, 0.0);
      }
    }
#pragma unroll
    for (int r = 0; r < PB; ++r) {
      if (q0 + r >= p1) break;  // CTA-uniform
      const int64_t i = (q0 + r) * kCoopPass + (int64_t)tid * kKarmaKV;
      const float cc[4] = {cv[r].x, cv[r].y, cv[r].z, cv[r].w};
      double kk[4] = {kv[r][0].x, kv[r][0].y, kv[r][1].x, kv[r][1].y};
      unsigned nib = 0u;
#pragma unroll
      for (int v = 0; v < kKarmaKV; ++v) {
        if (i + v < n) {
          const double ci = (double)cc[v];
          const double p_minus = (phat * a.n_global - ci) * inv_nm1;  // eq. (6)
          double L_minus;
          loss_eval(kp.loss, kp.lambda, p_minus, p, &L_minus, &dummy);
          kk[v] = fmin(kk[v] + (L_minus - L_full), kp.k_max);  // eq. (7)-(8)
          nib |= (unsigned)((kk[v] < kp.threshold) || (ci >= thr)) << v;
        }
      }
      if (i < n) {
#if KDE_TUNE_L2KEEP
        st_keep_d2(a.karma + i, make_double2(kk[0], kk[1]), pol_keep);
        st_keep_d2(a.karma + i + 2, make_double2(kk[2], kk[3]), pol_keep);
#else
        __stcs(reinterpret_cast<double2*>(a.karma + i), make_double2(kk[0], kk[1]));
        __stcs(reinterpret_cast<double2*>(a.karma + i + 2), make_double2(kk[2], kk[3]));
#endif
      }
      unsigned word = nib << (4 * (lane & 7));  // word of 32 points = nibbles of 8 lanes
      word |= __shfl_xor_sync(0xffffffffu, word, 1);
      word |= __shfl_xor_sync(0xffffffffu, word, 2);
      word |= __shfl_xor_sync(0xffffffffu, word, 4);
      if ((lane & 7) == 0) {
        a.bitmap[(q0 + r) * (kCoopPass / 32) + warp * 4 + (lane >> 3)] = word;
        my += __popc(word);
      }
    }
  }
  for (int o = 8; o < 32; o <<= 1) my += __shfl_xor_sync(0xffffffffu, my, o);
  if (lane == 0) red_s[0][warp] = my;
  __syncthreads();
  if (tid == 0) {
    int32_t t = 0;
    for (int w = 0; w < kCoopThreads / 32; ++w) t += (int32_t)red_s[0][w];
    a.cta_counts[b] = t;
  }
  grid.sync();
  // ---------------- phase 2: this CTA's offset (fixed-order integer sums), ordered compaction
  int64_t before = 0, total = 0;
  for (int c = tid; c < G; c += kCoopThreads) {
    const int64_t v = __ldcg(a.cta_counts + c);
    total += v;
    if (c < b) before += v;
  }
  for (int o = 16; o > 0; o >>= 1) {
    before += __shfl_xor_sync(0xffffffffu, before, o);
    total += __shfl_xor_sync(0xffffffffu, total, o);
  }
  __syncthreads();
  if (lane == 0) {
    red_s[0][warp] = before;
    red_s[1][warp] = total;
  }
  __syncthreads();
  before = total = 0;
  for (int w = 0; w < kCoopThreads / 32; ++w) {
    before += red_s[0][w];
    total += red_s[1][w];
  }
  if (total > 0) {  // nothing flagged anywhere: no bitmap to walk
    const int64_t nwords = (n + 31) / 32;
    const int64_t w1 = min(p1 * (kCoopPass / 32), nwords);
    int64_t run = before;
    for (int64_t wb = p0 * (kCoopPass / 32); wb < w1; wb += W) {
      if (warp == 0) {  // the step's words, their exclusive popcount prefix
        int cnt[WPL], tot = 0;
#pragma unroll
        for (int k = 0; k < WPL; ++k) {
          const int64_t w = wb + WPL * lane + k;
          const uint32_t word = w < w1 ? __ldcg(a.bitmap + w) : 0u;
          wbits[WPL * lane + k] = word;
          cnt[k] = __popc(word);
          tot += cnt[k];
        }
        int incl = tot;
#pragma unroll
        for (int k = 1; k < 32; k <<= 1) {
          const int v = __shfl_up_sync(0xffffffffu, incl, k);
          if (lane >= k) incl += v;
        }
        int rr = incl - tot;
#pragma unroll
        for (int k = 0; k < WPL; ++k) {
          wpre[WPL * lane + k] = rr;
          rr += cnt[k];
        }
        if (lane == 31) segtot_s = incl;
      }
      __syncthreads();
#pragma unroll 4
      for (int w = warp; w < W; w += kCoopThreads / 32) {
        const uint32_t word = wbits[w];
        if (word & (1u << lane)) {
          const int64_t pos = run + wpre[w] + __popc(word & ((1u << lane) - 1u));
          if (pos < a.cap) a.idx_out[pos] = a.row_offset + (wb + w) * 32 + lane;
        }
      }
      run += segtot_s;
      __syncthreads();
    }
  }
  if (b == 0 && tid == 0 && a.total_out) *a.total_out = total;
  const StreamTail& tail = a.tail;
  if (!tail.online && !tail.rows) return;
  grid.sync();
  // ---------------- phase 3: the streaming step's tail
  if (tail.online && b == 0) online_update_body(tail.ret, tail.p, tail.op, tail.d, tail.st, tail.c);
  if (tail.rows) {
    __shared__ unsigned rmin[kMaxDim], rmax[kMaxDim];
    if (tid < kMaxDim) {
      rmin[tid] = 0xFFFFFFFFu;
      rmax[tid] = 0u;
    }
    __syncthreads();
    const int64_t k = min(total, a.cap);
    const float* __restrict__ rows = tail.rows;
    float* __restrict__ cols = tail.cols;
    for (int64_t r = (int64_t)b * kCoopThreads + tid; r < k; r += (int64_t)G * kCoopThreads) {
      const int64_t i = __ldcg(a.idx_out + r) - a.row_offset;
      float x[kMaxDim];
#pragma unroll
      for (int j = 0; j < kMaxDim; ++j) x[j] = j < tail.d ? rows[r * tail.d + j] : 0.0f;
#pragma unroll
      for (int j = 0; j < kMaxDim; ++j) {
        if (j < tail.d) {
          cols[(int64_t)j * tail.ld + i] = x[j];
          atomicMin(rmin + j, fenc(x[j]));
          atomicMax(rmax + j, fenc(x[j]));
        }
      }
      tail.karma[i] = tail.k_init;
    }
    __syncthreads();
    if (tid < tail.d && (int64_t)b * kCoopThreads < k) {
      atomicMin(tail.c->renc + 2 * tid, rmin[tid]);
      atomicMax(tail.c->renc + 2 * tid + 1, rmax[tid]);
    }
  }
}

// ------------------------------------------------------------ harness: exact box counts
// counts[k] = |{r : l_kj < R_rj < u_kj for all j}|, open box as in P:L45.
__global__ void count_in_box_kernel(const float* __restrict__ rows, int64_t n, int d, const float* __restrict__ lo,
                                    const float* __restrict__ hi, int64_t q, int64_t rows_per_block,
                                    unsigned long long* __restrict__ counts) {
  const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t r0 = (int64_t)blockIdx.y * rows_per_block;
  const int64_t r1 = min(n, r0 + rows_per_block);
  __shared__ float tile[256 * kMaxDim];
  float l[kMaxDim], u[kMaxDim];
  const int64_t kk = k < q ? k : q - 1;
  for (int j = 0; j < d; ++j) {
    l[j] = lo[kk * d + j];
    u[j] = hi[kk * d + j];
  }
  unsigned long long cnt = 0;
  for (int64_t t0 = r0; t0 < r1; t0 += 256) {
    const int m = (r1 - t0) < 256 ? (int)(r1 - t0) : 256;
    __syncthreads();
    for (int e = threadIdx.x; e < m * d; e += blockDim.x) tile[e] = rows[t0 * d + e];
    __syncthreads();
    for (int r = 0; r < m; ++r) {
      bool in = true;
      for (int j = 0; j < d; ++j) {
        const float x = tile[r * d + j];
        in = in && (x > l[j]) && (x < u[j]);
      }
      cnt += in ? 1ull : 0ull;
    }
  }
  if (k < q && cnt) atomicAdd(counts + k, cnt);
}

// ------------------------------------------------------------ launchers
#define KDE_LAUNCH_CHECK() return cudaGetLastError()

cudaError_t launch_rows_to_cols(const float* rows, int64_t n, int d, float* cols, int64_t ld, int* bad,
                                cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  rows_to_cols_kernel<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(rows, n, d, cols, ld, bad);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_cols_to_rows(const float* cols, int64_t ld, int64_t n, int d, float* rows, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  cols_to_rows_kernel<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(cols, ld, n, d, rows);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_col_range(const float* cols, int64_t ld, int64_t n, int d, unsigned* enc, DevConsts* c,
                             cudaStream_t s) {
  int64_t nb = (n + 255) / 256;
  if (nb > 1024) nb = 1024;
  if (nb < 1) nb = 1;
  col_range_kernel<<<dim3((unsigned)nb, d), 256, 0, s>>>(cols, ld, n, enc);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_row_range(const float* rows, int64_t k, int d, unsigned* enc, DevConsts* c, cudaStream_t s) {
  if (k == 0) return cudaSuccess;
  int64_t nb = (k + 255) / 256;
  if (nb > 296) nb = 296;
  row_range_kernel<<<(unsigned)nb, 256, 0, s>>>(rows, k, d, enc);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_scatter_rows_dev(const int64_t* idx_global, const float* rows, const int64_t* d_k, int64_t cap, int d,
                                    float* cols, int64_t ld, int64_t n, int64_t row_offset, double* karma, double k_init,
                                    unsigned* enc, DevConsts* c, cudaStream_t s) {
  if (cap == 0) return cudaSuccess;
  scatter_rows_dev_kernel<<<(unsigned)((cap + 255) / 256), 256, 0, s>>>(idx_global, rows, d_k, cap, d, cols, ld, n,
                                                                         row_offset, karma, k_init, enc);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_scatter_rows(const int64_t* idx_local, const float* rows, int64_t k, int d, float* cols,
                                int64_t ld, double* karma, double k_init, cudaStream_t s) {
  if (k == 0) return cudaSuccess;
  scatter_rows_kernel<<<(unsigned)((k + 255) / 256), 256, 0, s>>>(idx_local, rows, k, d, cols, ld, karma, k_init);
  KDE_LAUNCH_CHECK();
}
int moments_blocks(int64_t n) {
  int64_t nb = (n + 65535) / 65536;
  if (nb < 1) nb = 1;
  if (nb > 1024) nb = 1024;
  return (int)nb;
}
cudaError_t launch_moments(const float* cols, int64_t ld, int64_t n, int d, double* part, double* mom,
                           cudaStream_t s) {
  const int nb = moments_blocks(n);
  const int64_t chunk = (n + nb - 1) / nb;
  moments_partial_kernel<<<dim3(nb, d), 256, 0, s>>>(cols, ld, n, chunk, part);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  moments_merge_kernel<<<1, 32, 0, s>>>(part, nb, d, mom);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_moments_merge_ranks(const double* g, int world, int d, double* mom, cudaStream_t s) {
  moments_merge_ranks_kernel<<<1, 32, 0, s>>>(g, world, d, mom);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_scott(const double* mom, int d, DevConsts* c, int* bad, cudaStream_t s) {
  scott_kernel<<<1, 32, 0, s>>>(mom, d, c, bad);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_set_kernel_type(int kernel, int d, DevConsts* c, cudaStream_t s) {
  set_kernel_type_kernel<<<1, 32, 0, s>>>(kernel, d, c);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_set_consts(const double* h, int d, DevConsts* c, cudaStream_t s) {
  HVec hv;
  for (int j = 0; j < d; ++j) hv.v[j] = h[j];
  set_consts_kernel<<<1, 32, 0, s>>>(hv, d, c);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_reduce_splits(const double* partials, int splits, int64_t q, int na, double* sums,
                                 const PeerArgs* peer, cudaStream_t s) {
  if (splits >= 64 && q * na <= 65536) {  // few outputs, long chains: a warp per output
    const int64_t threads = q * na * 32;
    reduce_splits_wide_kernel<<<(unsigned)((threads + 255) / 256), 256, 0, s>>>(partials, splits, q, na, sums, peer);
  } else {
    reduce_splits_kernel<<<(unsigned)((q + 255) / 256), 256, 0, s>>>(partials, splits, q, na, sums, peer);
  }
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_reduce_splits_mapped(const double* partials, int splits, int64_t qpad, int64_t q, int na, int qg,
                                        int ngroups, const int* perm, double* sums, const PeerArgs* peer,
                                        cudaStream_t s) {
  const int wide = (splits >= 64 && qpad * na <= 65536) ? 1 : 0;
  const int64_t threads = wide ? qpad * na * 32 : qpad;
  reduce_splits_mapped_kernel<<<(unsigned)((threads + 255) / 256), 256, 0, s>>>(partials, splits, qpad, q, na, qg,
                                                                                ngroups, perm, sums, peer, wide);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_combine_ranks(const double* gathered, int world, int64_t q, int na, double* sums,
                                 cudaStream_t s) {
  const int64_t e = q * na;
  combine_ranks_kernel<<<(unsigned)((e + 255) / 256), 256, 0, s>>>(gathered, world, q, na, sums);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_finalize(const double* sums, int64_t q, int d, int na, const DevConsts* c, double n_global,
                            double* est, double* dpdh, cudaStream_t s) {
  finalize_kernel<<<(unsigned)((q + 255) / 256), 256, 0, s>>>(sums, q, d, na, c, n_global, est, dpdh);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_loss_epilogue(const double* est, const double* dpdh, const double* true_sel, int64_t q, int d,
                                 int kind, double lambda, int log_bw, const DevConsts* c, double* loss_out,
                                 double* grad_out, cudaStream_t s) {
  loss_epilogue_kernel<<<1, 512, 0, s>>>(est, dpdh, true_sel, q, d, kind, lambda, log_bw, c, loss_out, grad_out);
  KDE_LAUNCH_CHECK();
}
int karma_launches() {  // kernels per karma pass: 1 (cooperative) or 2 (KDE_KARMA_TWO_PASS, A/B timing)
  static const int k = getenv("KDE_KARMA_TWO_PASS") != nullptr ? 2 : 1;
  return k;
}

static int coop_grid_limit() {
  // co-resident CTAs of the cooperative karma kernel, per device
  static int cached[64] = {0};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 0;
  int& v = cached[dev & 63];
  if (v == 0) {
    int sms = 0, per = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, karma_coop_kernel, kCoopThreads, 0);
    v = sms * (per > 0 ? per : 1);
  }
  return v;
}

cudaError_t launch_karma(const float* cvals, double* karma, int64_t n, double n_global, const double* phat, const double* p,
                         const KarmaParamsDev& kp, const float* lo, const float* hi, int d, const DevConsts* c,
                         uint32_t* bitmap, int32_t* block_counts, int64_t* block_offsets, unsigned* done,
                         int64_t row_offset, int64_t* idx_out, int64_t cap, int64_t* total_out, const StreamTail& tail,
                         cudaStream_t s) {
  const int nb = karma_blocks(n);
  if (nb == 0) return cudaSuccess;
  if (karma_launches() == 1) {
    KarmaCoopArgs a{cvals, karma, n, n_global, phat, p, kp, lo, hi, d, c, bitmap, block_counts, row_offset,
                    idx_out, cap, total_out, tail};
    int grid = coop_grid_limit();
    const int64_t passes = (n + kCoopPass - 1) / kCoopPass;
    if (grid > passes) grid = (int)passes;
    if (grid < 1) grid = 1;
    void* args[] = {&a};
    return cudaLaunchCooperativeKernel((const void*)karma_coop_kernel, grid, kCoopThreads, args, 0, s);
  }
  karma_kernel<<<nb, kKarmaThreads, 0, s>>>(cvals, karma, n, n_global, phat, p, kp, lo, hi, d, c, bitmap,
                                            block_counts, block_offsets, done + 1, nb);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  compact_fused_kernel<<<nb, kKarmaThreads, 0, s>>>(bitmap, n, block_offsets, nb, row_offset, idx_out, cap, total_out,
                                                    done, tail);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_online_update(const double* ret, const double* p, const OnlineParamsDev& op, int d, OnlineState* st,
                                 DevConsts* c, cudaStream_t s) {
  online_update_kernel<<<1, 32, 0, s>>>(ret, p, op, d, st, c);
  KDE_LAUNCH_CHECK();
}
cudaError_t launch_count_in_box(const float* rows, int64_t n, int d, const float* lo, const float* hi, int64_t q,
                                unsigned long long* counts, int num_sms, cudaStream_t s) {
  if (q == 0 || n == 0) return cudaSuccess;
  const int64_t qb = (q + 255) / 256;
  int64_t rb = (num_sms * 8 + qb - 1) / qb;
  const int64_t maxrb = (n + 255) / 256;
  if (rb > maxrb) rb = maxrb;
  if (rb < 1) rb = 1;
  int64_t rows_per_block = (n + rb - 1) / rb;
  rows_per_block = (rows_per_block + 255) / 256 * 256;
  rb = (n + rows_per_block - 1) / rows_per_block;
  count_in_box_kernel<<<dim3((unsigned)qb, (unsigned)rb), 256, 0, s>>>(rows, n, d, lo, hi, q, rows_per_block, counts);
  KDE_LAUNCH_CHECK();
}

}  // namespace kde
