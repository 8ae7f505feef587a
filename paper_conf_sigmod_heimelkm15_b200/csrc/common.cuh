// common.cuh -- internal types shared by the KDE kernels and the C-ABI runtime.
// Citations "P:L<n>" refer to lines of the paper text.
#pragma once
#include <cstdint>
#include <cstring>
#include <cuda_runtime.h>

#ifndef KDE_MAX_DIM
#define KDE_MAX_DIM 16
#endif

namespace kde {

constexpr int kMaxDim = KDE_MAX_DIM;
constexpr int kColAlign = 2048;  // columns padded to a multiple of this many points (>= the single-scan TMA tile)

// Per-dimension constants derived from the fp64 bandwidth h (device resident
// so that an on-device bandwidth update needs no host round trip).
//   ap[j]     = sqrt(log2 e) / (sqrt(2) h_j)      y' = (b - t) * ap[j] = z_j sqrt(log2 e),
//                                                  z = (b - t)/(sqrt2 h) is the erf argument of eq. (13)
//   gconst[j] = 1 / (sqrt(pi) sqrt(log2 e) h_j)   so that d p^(i)/d h_j = gconst[j] * w_j * prod_{k!=j} D_k,
//                                                  w_j = y'_l E_l - y'_u E_u (eq. 17 rewritten in z)
// Epanechnikov product kernel (reading R14): ap[j] = 1/h_j (v = (b - t)/h),
//   gconst[j] = -3 / (4 h_j), w_j = Delta (1 - S) (see phi.cuh).
//   tmin/tmax = per-column range of the (local) sample: query bounds are
//   clamped to [tmin - 14/ap, tmax + 14/ap] at box setup, which leaves every
//   fp32 result unchanged (|y'| >= 14 gives E = 0, erf = +-1 exactly) and
//   keeps y' finite, so the gradient term y' E never meets inf * 0.
enum KernelType : int { kGaussian = 0, kEpanechnikov = 1 };

struct DevConsts {
  int kernel;  // KernelType: selects the per-dimension constants below
  double h[kMaxDim];
  double gconst[kMaxDim];
  float ap[kMaxDim];
  unsigned renc[2 * kMaxDim];  // (min, max) per column, order-preserving uint encoding (atomicMin/Max)
};

// order-preserving float <-> uint encoding used for the column ranges
__host__ __device__ __forceinline__ unsigned fenc_range(float f) {
  unsigned u;
  memcpy(&u, &f, sizeof(u));
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__host__ __device__ __forceinline__ float fdec_range(unsigned e) {
  const unsigned u = (e & 0x80000000u) ? (e & 0x7fffffffu) : ~e;
  float f;
  memcpy(&f, &u, sizeof(f));
  return f;
}

// L2 residency of the streaming step's working set (karma K: 8 B/point, retained p^(i): 4 B/point;
// 48 MB at N = 2^22): the single-box scan streams the sample through L2 with an evict-first policy
// and writes p^(i) evict-last, the karma pass reads p^(i) and updates K evict-last, so both stay in
// the 126 MB L2 from one query to the next instead of round-tripping HBM (KDE_TUNE_L2KEEP=0: the
// previous streaming hints, for A/B).
#ifndef KDE_TUNE_L2KEEP
#define KDE_TUNE_L2KEEP 1
#endif
#ifdef __CUDACC__
__device__ __forceinline__ uint64_t l2_policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ float4 ld_keep_f4(const float* p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ double2 ld_keep_d2(const double* p, uint64_t pol) {
  double2 v;
  asm volatile("ld.global.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;" : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void st_keep_d2(double* p, double2 v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %3;" ::"l"(p), "d"(v.x), "d"(v.y), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_keep_f2(float* p, float2 v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v2.f32 [%0], {%1, %2}, %3;" ::"l"(p), "f"(v.x), "f"(v.y), "l"(pol) : "memory");
}
__device__ __forceinline__ void st_keep_f1(float* p, float v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(p), "f"(v), "l"(pol) : "memory");
}
#endif

// Listing 1 state (reconstruction, R6), device resident.
struct OnlineState {
  double acc[kMaxDim];
  double ms[kMaxDim];
  double lr[kMaxDim];
  double gprev[kMaxDim];
  int32_t count;
  int32_t updated;  // 1 when the last kde_online_update changed h
};

struct OnlineParamsDev {
  int32_t minibatch, log_bw, loss;
  double lambda, alpha, lr_min, lr_max, lr_inc, lr_dec;
};

struct KarmaParamsDev {
  int32_t loss, empty_region;
  double lambda, k_max, threshold;
};

// Peer-memory exchange of a sharded model (peer.cu): every rank's exchange window mapped into
// this process, the device-side epoch / arrival counters / error flag.  A window is
//   [kPeerFlagBytes) flags: uint64 epoch per source rank (128 B apart) | [2][world][slot] data slots
constexpr int kMaxWorld = 32;
constexpr size_t kPeerFlagBytes = (size_t)kMaxWorld * 128;
struct PeerArgs {
  char* base[kMaxWorld];  // every rank's exchange window (base[rank] = own)
  int rank = 0, world = 1;
  size_t slot = 0;            // bytes per (parity, source rank) slot, multiple of 256
  uint64_t* epoch = nullptr;  // device: last completed exchange
  unsigned* count = nullptr;  // device: 4 self-resetting block-arrival counters
  int* err = nullptr;         // device: set to 1 when a wait times out
  uint64_t timeout_ns = 0;
};

// scan over the sample for ONE box (q == 1): HBM-streaming reduction.
struct ScanSingleArgs {
  const float* cols;      // [d][ld] fp32 SoA sample
  int64_t ld;             // padded column length (multiple of kColAlign)
  int64_t n;              // valid points in this shard
  const float* lo;        // device, d floats
  const float* hi;        // device, d floats
  const DevConsts* consts;
  float* c_out;           // nullable: retained p^(i) (fp32) per point
  double* block_partials; // [gridDim.x][1+d]
  unsigned* counter;      // zero on entry; the last block resets it to zero
  double* sums_out;       // [1+d] raw sums S_0 = sum_i p^(i), S_j = sum_i w_j prod_{k!=j} D_k
  double* fin_out;        // nullable: [1+d] finalised (p_hat, dp_hat/dh_j) for world == 1 (retained copy)
  double* est_out;        // nullable: p_hat (caller's buffer), world == 1
  double* dpdh_out;       // nullable: d x dp_hat/dh_j (caller's buffer), world == 1, GRAD only
  double n_global;        // s (results are divided by s, so s ones give exactly 1)
  int cull;               // 1: skip points whose contribution is provably < 2^-64 (scan_single_tma.cuh)
  const PeerArgs* peer;   // nullable (device): the last block pushes sums_out into every rank's window
  // nullable: the spatially ordered copy (cells.cu, reading R17) -- with cull on and no c_out the
  // scan visits cells and skips those whose bounding box is >= 8 bandwidths outside the box
  const float* ccols;     // [d][ld]
  const float* cbb;       // [ncells][d][2]
  int64_t ncells;
  unsigned long long* stats;  // nullable (profiling, cells path): += cells read, full cells, points evaluated, classified
};

// scan for many boxes: sample tiles staged in shared memory by TMA bulk
// copies, each thread keeps QT boxes in registers.
struct ScanBatchedArgs {
  const float* cols;
  int64_t ld, n;
  const float* lo;        // device [q][d]
  const float* hi;        // device [q][d]
  int64_t q;
  const DevConsts* consts;
  int64_t split_len;      // points per split (multiple of the tile size)
  int qb;                 // boxes per CTA (power of two <= 256; 256/qb threads share a box)
  double* partials;       // [splits][1+d][q]
  int cull;               // 1: per (box, point) tail culling (scan.cuh batched_tile_cull), qb == 256 only
  const int* perm;        // nullable: CTA slot order -> box index (boxes sorted by their probed kept fraction)
};

// culled batched scan over the spatially ordered copy of the sample (scan_cells.cuh, reading R17):
// cells of kCellPts consecutive points in Morton order, each with its bounding box; a CTA owns a
// group of boxes (dealt from the probe order so groups and warps get similar cost) and the cells
// split, split + nsplit, ... (strided over the whole curve, so every CTA sees every region).
constexpr int kCellPts = 256;  // points per cell (= the batched scan's tile)
struct ScanCellsArgs {
  const float* ccols;     // [d][ld] ordered copy of the sample (cells.cu)
  int64_t ld;             // padded column length
  int64_t n;              // valid points
  int64_t ncells;         // ceil(n / kCellPts)
  const float* cbb;       // [ncells][d][2] per-cell (min, max) of the raw coordinates
  const float* lo;        // device [q][d]
  const float* hi;        // device [q][d]
  int64_t q;
  const DevConsts* consts;
  const int* perm;        // nullable: sorted position -> box index (probe order, cull_order.cu)
  double* partials;       // [nsplit][1+d][qpad], row entry r = g * QG + slot (coalesced per CTA)
  int64_t qpad;           // ngroups * QG (cells_layout)
  unsigned long long* stats;  // nullable (profiling): += items, full items, points evaluated, points classified
};

// spatial index of the sample (cells.cu): Morton keys over the column range, stable radix sort,
// gathered ordered copy (padding points 0) and per-cell bounding boxes
size_t cells_scratch_bytes(int64_t n);
cudaError_t launch_cells_build(const float* cols, int64_t ld, int64_t n, int d, const DevConsts* c, void* scratch,
                               size_t scratch_bytes, float* ccols, float* cbb, cudaStream_t s);

// host-side launchers (scan_inst_*.cu)
cudaError_t launch_scan_cells(int d, bool grad, const ScanCellsArgs& a, int num_sms, int* splits_out, cudaStream_t s,
                              bool dry_run);
// boxes per CTA group of the cells scan for dimension d (the partials' row layout, reduce_splits_mapped)
int cells_group_boxes(int d);
cudaError_t launch_scan_single(int d, bool grad, const ScanSingleArgs& a, int grid, cudaStream_t s);
cudaError_t launch_scan_batched(int d, bool grad, const ScanBatchedArgs& a, int num_sms, int* splits_out,
                                cudaStream_t s, bool dry_run);
int scan_single_grid(int d, bool grad, int64_t n, int num_sms, bool cull);
bool batched_culls(int64_t q);

}  // namespace kde
