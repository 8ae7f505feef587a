// kde_api.cu -- the C ABI (include/kde.h) and the kde_model runtime:
// device buffers, stream, argument validation, dispatch between the
// single-box streaming scan and the tiled batched scan, NCCL combine of
// per-shard partial sums, retained state for feedback, error handling.
//
// Every numeric step runs in the kernels of scan.cuh / kernels.cu; this file
// only moves arguments, validates them and orders launches on one stream.
#include <algorithm>
#include <climits>
#include <cstddef>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <vector>

#include <cuda_runtime.h>
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>

#include "../../include/kde.h"
#include "common.cuh"
#include "kernels.cuh"

using namespace kde;

// ------------------------------------------------------------------ errors
static thread_local char g_err[512] = "";

static kde_status fail(kde_status st, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
  return st;
}

struct kde_model {
  int device = 0;
  int num_sms = 148;
  cudaStream_t stream = nullptr;
  int32_t d = 0;
  int64_t n = 0;         // local points
  int64_t n_global = 0;  // s
  int64_t row_offset = 0;
  int64_t ld = 0;        // padded column length
  int rank = 0, world = 1;
  int comm_kind = KDE_COMM_NONE;   // how world > 1 ranks exchange (kde_comm)
  ncclComm_t comm = nullptr;       // KDE_COMM_NCCL
  bool attached = true;            // KDE_COMM_PEER: false until kde_peer_attach
  bool h_pending = false;          // KDE_COMM_PEER without h: Scott's rule runs in kde_peer_attach
  char* xwin = nullptr;            // KDE_COMM_PEER: this rank's exchange window (peer.cu)
  size_t xwin_bytes = 0;
  PeerArgs pa;                     // mapped windows of every rank + device epoch / counters / error flag
  PeerArgs* pa_dev = nullptr;      // device copy of pa (read by the producers' fused push)
  bool poisoned = false;

  float* cols = nullptr;       // [d][ld]
  double* karma = nullptr;     // [n]
  float* cret = nullptr;       // [ld] retained contributions
  DevConsts* consts = nullptr;
  OnlineState* online = nullptr;

  // scratch
  double* block_partials = nullptr;  // single-scan block partials
  unsigned* counter = nullptr;
  double* ret = nullptr;             // [1 + d] retained (p_hat, dp/dh)
  double* single_sums = nullptr;     // [1 + d]
  float* qbuf = nullptr;             // device bounds staging [2][qcap][d]
  int64_t qcap = 0;
  double* obuf = nullptr;            // device outputs: est [qcap], dpdh [qcap*d], sums [qcap*(1+d)], true [qcap], loss, grad
  int64_t ocap = 0;
  double* partials = nullptr;
  size_t partials_cap = 0;           // bytes
  void* order = nullptr;             // culled batched scan: box-order scratch (cull_order.cu)
  size_t order_cap = 0;              // bytes
  // spatial index for the culled batched scan (cells.cu, reading R17): ordered copy + cell boxes,
  // rebuilt lazily when the sample changed since it was built (sgen != cells_gen)
  bool cells_on = true;              // KDE_CELLS=0: the unordered culled batched scan instead
  float* ccols = nullptr;            // [d][ld]
  float* cbb = nullptr;              // [ncells][d][2]
  void* cscratch = nullptr;          // build scratch (keys, indices, radix-sort temp)
  size_t cscratch_cap = 0;
  uint64_t sgen = 1;                 // bumped whenever the sample's rows change
  uint64_t cells_gen = 0;            // sgen the index was built at (0: none)
  int64_t cells_builds = 0;          // index builds so far (kde_get_cells)
  unsigned long long* cstats = nullptr;  // device [4] cells-scan counters while profiling (kde_get_cells)
  double* gather = nullptr;          // [world][q][1+d]
  size_t gather_cap = 0;
  uint32_t* bitmap = nullptr;
  int32_t* block_counts = nullptr;
  int64_t* block_offsets = nullptr;  // [nkb + 1] exclusive offsets of the karma flags + total
  int64_t* offsets = nullptr;        // [0] = total flagged (karma compaction)
  unsigned* done = nullptr;          // compaction last-block counter (self-resetting)
  int64_t* idx_dev = nullptr;
  int64_t idx_cap = 0;
  int32_t* bad = nullptr;            // device flag
  unsigned* range_enc = nullptr;     // = consts->renc: [d][2] encoded column min/max (kernels.cu)
  double* scal = nullptr;            // [8] device scalars (true selectivity staging)
  void* pinned = nullptr;            // pinned host staging
  size_t pinned_cap = 0;
  void* apin[2] = {nullptr, nullptr};  // kde_insert_rows_async: double-buffered pinned staging
  size_t apin_cap[2] = {0, 0};
  cudaEvent_t apin_ev[2] = {nullptr, nullptr};  // recorded after the H2D copy out of apin[b]
  int apin_next = 0;
  void* rbuf = nullptr;              // replacement staging (idx + rows), grow-only
  size_t rbuf_cap = 0;
  cudaEvent_t dev_done = nullptr;    // recorded on the caller's stream at the end of every _dev call
  bool dev_pending = false;          // some _dev call enqueued work on a stream other than m->stream
  void* kbuf = nullptr;              // sharded karma gather: counts + index lists, grow-only
  size_t kbuf_cap = 0;

  // retained single-box state
  bool retain = false;
  bool cull = true;  // kde_set_cull: skip points whose contribution is provably < 2^-64 (single-box scan)
  bool ret_valid = false, ret_has_c = false, ret_has_grad = false;
  float ret_lo[kMaxDim], ret_hi[kMaxDim];
  uint64_t gen = 1;      // bumped whenever h or the sample changes (sgen: the sample only)
  uint64_t ret_gen = 0;
  bool online_init = false;
  int32_t kernel = 0;  // KDE_KERNEL_GAUSSIAN

  // profiling (kde_set_profiling): CUDA events around every scan launch on its
  // own stream, and a count of every kernel this model launched
  bool prof = false;
  std::vector<cudaEvent_t> ev;  // pairs (start, end)
  size_t ev_used = 0;
  int64_t scan_launches = 0;
  int64_t launches = 0;
};

#define CU(call)                                                                                     \
  do {                                                                                               \
    cudaError_t e_ = (call);                                                                         \
    if (e_ != cudaSuccess) {                                                                         \
      if (m) m->poisoned = true;                                                                     \
      return fail(KDE_ECUDA, "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
    }                                                                                                \
  } while (0)

// KDE_DEBUG_SYNC=1: synchronise the stream after every launch so a faulting kernel is reported by
// the call that launched it (debugging aid; off by default)
static bool debug_sync() {
  static const bool on = getenv("KDE_DEBUG_SYNC") && atoi(getenv("KDE_DEBUG_SYNC")) != 0;
  return on;
}
#define CUL(call)                                         \
  do {                                                    \
    ++m->launches;                                        \
    CU(call);                                             \
    if (debug_sync()) CU(cudaDeviceSynchronize());        \
  } while (0)

// NVTX range per ABI call (visible in Nsight Systems / ncu --nvtx; no cost without a tool attached)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
#define KDE_RANGE() NvtxRange nvtx_range_(__func__)

#define NC(call)                                                                                     \
  do {                                                                                               \
    ncclResult_t r_ = (call);                                                                        \
    if (r_ != ncclSuccess) {                                                                         \
      if (m) m->poisoned = true;                                                                     \
      return fail(KDE_ENCCL, "%s failed: %s", #call, ncclGetErrorString(r_));                       \
    }                                                                                                \
  } while (0)

#define CHECK_MODEL(m)                                                                     \
  do {                                                                                     \
    if (!(m)) return fail(KDE_EINVAL, "model is NULL");                                   \
    if ((m)->poisoned) return fail(KDE_ESTATE, "model poisoned by an earlier CUDA/NCCL error"); \
    if (!(m)->attached) return fail(KDE_ESTATE, "sharded model not attached (kde_peer_attach)"); \
  } while (0)

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
    else prev = -1;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

// Ordering between the two call styles.  _dev calls enqueue on the caller's stream; host-pointer
// calls run on the model's stream and are synchronous.  Every _dev call records dev_done on its
// stream (an external event node when the stream is being captured into a CUDA graph); every call
// that works on the model's stream first waits for it, so e.g. kde_insert_rows after a replayed
// streaming step never overlaps that step's scan / karma / replacement.
static kde_status mark_dev(kde_model* m, cudaStream_t s) {
  if (s == m->stream) return KDE_OK;
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  CU(cudaStreamIsCapturing(s, &cs));
  if (cs == cudaStreamCaptureStatusActive)
    CU(cudaEventRecordWithFlags(m->dev_done, s, cudaEventRecordExternal));
  else
    CU(cudaEventRecord(m->dev_done, s));
  m->dev_pending = true;
  return KDE_OK;
}
static kde_status wait_dev(kde_model* m) {
  if (m->dev_pending) CU(cudaStreamWaitEvent(m->stream, m->dev_done, 0));
  return KDE_OK;
}
#define WAIT_DEV(m)                        \
  do {                                     \
    kde_status wst_ = wait_dev(m);         \
    if (wst_ != KDE_OK) return wst_;       \
  } while (0)

static bool h_ok(double h) { return std::isfinite(h) && h >= 1e-30 && h <= 1e30; }

static kde_status validate_bounds(const float* lo, const float* hi, int64_t q, int d) {
  if (q < 0) return fail(KDE_EINVAL, "q < 0");
  if (q > 0 && (!lo || !hi)) return fail(KDE_EINVAL, "lo/hi is NULL");
  for (int64_t i = 0; i < q * d; ++i) {
    if (std::isnan(lo[i]) || std::isnan(hi[i])) return fail(KDE_EINVAL, "NaN in query bounds (element %lld)", (long long)i);
    if (lo[i] > hi[i]) return fail(KDE_EINVAL, "lo > hi in query bounds (element %lld)", (long long)i);
  }
  return KDE_OK;
}

static kde_status validate_loss(int32_t loss, double lambda) {
  if (loss < 0 || loss > 4) return fail(KDE_EINVAL, "unknown loss kind %d", loss);
  if (!std::isfinite(lambda) || lambda < 0.0) return fail(KDE_EINVAL, "lambda must be finite and >= 0");
  if (loss >= 2 && !(lambda > 0.0)) return fail(KDE_EINVAL, "lambda must be > 0 for relative / Q losses");
  return KDE_OK;
}

// ------------------------------------------------------------------ buffers
static kde_status ensure_pinned(kde_model* m, size_t bytes) {
  if (m->pinned_cap >= bytes) return KDE_OK;
  if (m->pinned) cudaFreeHost(m->pinned);
  for (int b = 0; b < 2; ++b) {
    if (m->apin[b]) cudaFreeHost(m->apin[b]);
    if (m->apin_ev[b]) cudaEventDestroy(m->apin_ev[b]);
  }
  m->pinned = nullptr;
  m->pinned_cap = 0;
  size_t cap = std::max<size_t>(bytes, 1 << 16);
  if (cudaMallocHost(&m->pinned, cap) != cudaSuccess) return fail(KDE_ENOMEM, "pinned host allocation of %zu bytes failed", cap);
  m->pinned_cap = cap;
  return KDE_OK;
}

static kde_status ensure_q(kde_model* m, int64_t q) {
  const int d = m->d;
  if (m->qcap < q) {
    if (m->qbuf) cudaFree(m->qbuf);
    m->qbuf = nullptr;
    int64_t cap = std::max<int64_t>(q, 64);
    if (cudaMalloc(&m->qbuf, sizeof(float) * 2 * cap * d) != cudaSuccess) return fail(KDE_ENOMEM, "bounds buffer");
    m->qcap = cap;
  }
  if (m->ocap < q) {
    if (m->obuf) cudaFree(m->obuf);
    m->obuf = nullptr;
    int64_t cap = std::max<int64_t>(q, 64);
    // est[cap] dpdh[cap*d] sums[cap*(1+d)] true[cap] loss[1] grad[d]
    size_t elems = cap + cap * d + cap * (1 + d) + cap + 1 + d;
    if (cudaMalloc(&m->obuf, sizeof(double) * elems) != cudaSuccess) return fail(KDE_ENOMEM, "output buffer");
    m->ocap = cap;
  }
  return KDE_OK;
}
static double* o_est(kde_model* m) { return m->obuf; }
static double* o_dpdh(kde_model* m) { return m->obuf + m->ocap; }
static double* o_sums(kde_model* m) { return m->obuf + m->ocap * (1 + m->d); }
static double* o_true(kde_model* m) { return m->obuf + m->ocap * (2 + 2 * m->d); }
static double* o_loss(kde_model* m) { return m->obuf + m->ocap * (3 + 2 * m->d); }
static double* o_grad(kde_model* m) { return o_loss(m) + 1; }

static kde_status ensure_bytes(void** p, size_t* cap, size_t bytes) {
  if (*cap >= bytes) return KDE_OK;
  if (*p) cudaFree(*p);
  *p = nullptr;
  *cap = 0;
  if (cudaMalloc(p, bytes) != cudaSuccess) {
    *p = nullptr;
    cudaGetLastError();  // not sticky: later launch checks must not see this error
    return fail(KDE_ENOMEM, "device allocation of %zu bytes failed", bytes);
  }
  *cap = bytes;
  return KDE_OK;
}

// ------------------------------------------------------------------ profiling
static kde_status prof_begin(kde_model* m, cudaStream_t s, cudaEvent_t* e1, cudaEvent_t* e2) {
  ++m->scan_launches;
  if (!m->prof) return KDE_OK;
  while (m->ev.size() < m->ev_used + 2) {
    cudaEvent_t e;
    CU(cudaEventCreate(&e));
    m->ev.push_back(e);
  }
  *e1 = m->ev[m->ev_used];
  *e2 = m->ev[m->ev_used + 1];
  m->ev_used += 2;
  CU(cudaEventRecord(*e1, s));
  return KDE_OK;
}

// ------------------------------------------------------------------ exchange (world > 1)
// recv[r * bytes ...] <- rank r's send[0, bytes) for every rank (an all-gather), over NCCL or
// over peer device memory (peer.cu, chunked by the window slot).  Stream-ordered.
static kde_status allgather(kde_model* m, const void* send, void* recv, size_t bytes, cudaStream_t s) {
  if (m->comm_kind == KDE_COMM_NCCL) {
    NC(ncclAllGather(send, recv, bytes, ncclChar, m->comm, s));
    return KDE_OK;
  }
  for (size_t o = 0; o < bytes; o += m->pa.slot) {
    const size_t len = std::min(m->pa.slot, bytes - o);
    CUL(launch_peer_allgather((const char*)send + o, (char*)recv + o, len, bytes, m->pa, m->num_sms, s));
  }
  return KDE_OK;
}

// after a synchronizing host call: a timed-out peer wait poisons the model
static kde_status check_peer(kde_model* m) {
  if (m->comm_kind != KDE_COMM_PEER) return KDE_OK;
  int err = 0;
  CU(cudaMemcpy(&err, m->pa.err, sizeof(int), cudaMemcpyDeviceToHost));
  if (err) {
    m->poisoned = true;
    return fail(KDE_ECUDA, "peer exchange timed out (a rank did not join a collective call)");
  }
  return KDE_OK;
}

// ------------------------------------------------------------------ scans
// The spatial index of the local shard (cells.cu), rebuilt when the sample changed since the last
// build.  Stream-ordered: the build reads m->cols on s, after every write enqueued before it.
static kde_status ensure_cells(kde_model* m, cudaStream_t s) {
  if (m->cells_gen == m->sgen && m->ccols) return KDE_OK;
  const int64_t ncells = (m->n + kCellPts - 1) / kCellPts;
  if (!m->ccols || !m->cbb) {  // both or neither (a failed allocation leaves neither behind)
    float* cc = nullptr;
    float* bb = nullptr;
    cudaError_t e = cudaMalloc(&cc, sizeof(float) * (size_t)m->d * m->ld);
    if (e == cudaSuccess) e = cudaMalloc(&bb, sizeof(float) * 2 * (size_t)m->d * (size_t)(ncells > 0 ? ncells : 1));
    if (e != cudaSuccess) {
      cudaFree(cc);
      cudaGetLastError();  // clear the allocation error: the model stays usable without the copy
      return fail(KDE_ENOMEM, "ordered copy of the sample: %s (kde_set_cells(m, 0) scans the sample itself)",
                  cudaGetErrorString(e));
    }
    cudaFree(m->ccols);
    cudaFree(m->cbb);
    m->ccols = cc;
    m->cbb = bb;
  }
  kde_status st = ensure_bytes(&m->cscratch, &m->cscratch_cap, cells_scratch_bytes(m->n));
  if (st != KDE_OK) return st;
  m->launches += 3;  // keys, gather, boxes (+ the radix sort's own kernels, library code)
  CU(launch_cells_build(m->cols, m->ld, m->n, m->d, m->consts, m->cscratch, m->cscratch_cap, m->ccols, m->cbb, s));
  if (debug_sync()) CU(cudaDeviceSynchronize());
  m->cells_gen = m->sgen;
  ++m->cells_builds;
  return KDE_OK;
}

// Raw sums for q boxes (device bounds) -> sums[q][na] combined over ranks.
// For q == 1 also retains c (if c_out) and writes the finalised values to fin.
static kde_status scan_sums(kde_model* m, const float* d_lo, const float* d_hi, int64_t q, bool grad, float* c_out,
                            double* d_sums, cudaStream_t s, double* d_est = nullptr, double* d_dpdh = nullptr) {
  const int d = m->d;
  const int na = grad ? d + 1 : 1;
  // fused exchange (peer transport): the producer's tail pushes the final sums into every rank's
  // window; one combine kernel follows (KDE_PEER_FUSED=0: the separate all-gather, for A/B tests)
  const char* fenv = getenv("KDE_PEER_FUSED");
  const PeerArgs* fused = (m->comm_kind == KDE_COMM_PEER && sizeof(double) * (size_t)q * na <= m->pa.slot &&
                           !(fenv && atoi(fenv) == 0))
                              ? m->pa_dev
                              : nullptr;
  if (q == 1) {
    ScanSingleArgs a{};
    a.peer = fused;
    a.cols = m->cols;
    a.ld = m->ld;
    a.n = m->n;
    a.lo = d_lo;
    a.hi = d_hi;
    a.consts = m->consts;
    a.c_out = c_out;
    a.block_partials = m->block_partials;
    a.counter = m->counter;
    a.sums_out = d_sums;
    // world == 1: the last block finalises straight into the retained copy and the caller's buffers
    a.fin_out = m->world == 1 ? m->ret : nullptr;
    a.est_out = m->world == 1 ? d_est : nullptr;
    a.dpdh_out = m->world == 1 ? d_dpdh : nullptr;
    a.n_global = (double)m->n_global;
    a.cull = m->cull ? 1 : 0;
    a.ccols = nullptr;
    a.cbb = nullptr;
    a.ncells = 0;
    a.stats = nullptr;
    int grid = scan_single_grid(d, grad, m->n, m->num_sms, m->cull);
    // the ordered copy, when current (built by a culled batched call since the last sample change):
    // cells far from the box are not read at all (scan_cells.cuh); not for retained contributions,
    // which are per point in the sample's own order
    static const bool env_cells1 = !(getenv("KDE_CELLS") && atoi(getenv("KDE_CELLS")) == 0);
    if (m->cull && m->cells_on && env_cells1 && !c_out && m->ccols && m->cells_gen == m->sgen) {
      a.ccols = m->ccols;
      a.cbb = m->cbb;
      a.ncells = (m->n + kCellPts - 1) / kCellPts;
      if (m->prof) {
        if (!m->cstats) {
          CU(cudaMalloc(&m->cstats, 4 * sizeof(unsigned long long)));
          CU(cudaMemsetAsync(m->cstats, 0, 4 * sizeof(unsigned long long), s));
        }
        a.stats = m->cstats;
      }
      const int64_t want = (a.ncells + 7) / 8;  // at least one cell per warp
      // CTAs per SM (waves of the 2 resident ones; KDE_CELLS1_CTAS tunes, <= 8 for block_partials)
      static const int per_sm = getenv("KDE_CELLS1_CTAS") ? std::max(1, std::min(8, atoi(getenv("KDE_CELLS1_CTAS")))) : 2;
      grid = (int)std::min<int64_t>((int64_t)m->num_sms * per_sm, std::max<int64_t>(want, 1));
    }
    cudaEvent_t e1 = nullptr, e2 = nullptr;
    kde_status pst = prof_begin(m, s, &e1, &e2);
    if (pst != KDE_OK) return pst;
    CUL(launch_scan_single(d, grad, a, grid, s));
    if (e2) CU(cudaEventRecord(e2, s));
  } else {
    ScanBatchedArgs a;
    a.cols = m->cols;
    a.ld = m->ld;
    a.n = m->n;
    a.lo = d_lo;
    a.hi = d_hi;
    a.q = q;
    a.consts = m->consts;
    static const bool env_cells = !(getenv("KDE_CELLS") && atoi(getenv("KDE_CELLS")) == 0);  // A/B switch
    bool cells = m->cull && m->cells_on && env_cells;
    if (cells) {  // build (or reuse) the ordered copy first; without the memory for it, scan the sample itself
      const kde_status cst = ensure_cells(m, s);
      if (cst == KDE_ENOMEM) {
        m->cells_on = false;  // do not retry every call (kde_set_cells(m, 1) re-enables)
        cells = false;
      } else if (cst != KDE_OK) {
        return cst;
      }
    }
    // unordered sample: culling for full 256-box CTAs only (measured: phased culling gains nothing)
    a.cull = (m->cull && (cells || batched_culls(q))) ? 1 : 0;
    a.split_len = 0;
    a.partials = nullptr;
    a.perm = nullptr;
    if (a.cull) {  // order boxes by probed cost
      const size_t ob = cull_order_bytes(q);
      kde_status st = ensure_bytes(&m->order, &m->order_cap, ob);
      if (st != KDE_OK) return st;
      int* perm = nullptr;
      CUL(launch_cull_order(m->cols, m->ld, m->n, d, d_lo, d_hi, q, m->consts, m->order, m->order_cap, &perm, s));
      a.perm = perm;
    }
    if (cells) {  // the ordered copy: cell-level skipping (scan_cells.cuh), any batch size
      kde_status st = KDE_OK;
      ScanCellsArgs c;
      c.ccols = m->ccols;
      c.ld = m->ld;
      c.n = m->n;
      c.ncells = (m->n + kCellPts - 1) / kCellPts;
      c.cbb = m->cbb;
      c.lo = d_lo;
      c.hi = d_hi;
      c.q = q;
      c.consts = m->consts;
      c.perm = a.perm;
      c.partials = nullptr;
      c.stats = nullptr;
      if (m->prof) {  // evaluated-pair counters for the bench's roofline (kde_get_cells)
        if (!m->cstats) {
          CU(cudaMalloc(&m->cstats, 4 * sizeof(unsigned long long)));
          CU(cudaMemsetAsync(m->cstats, 0, 4 * sizeof(unsigned long long), s));
        }
        c.stats = m->cstats;
      }
      int splits = 1;
      CU(launch_scan_cells(d, grad, c, m->num_sms, &splits, s, true));
      const int qg = cells_group_boxes(d);
      const int64_t ngroups = (q + qg - 1) / qg;
      c.qpad = ngroups * qg;
      st = ensure_bytes((void**)&m->partials, &m->partials_cap, sizeof(double) * (size_t)splits * na * c.qpad);
      if (st != KDE_OK) return st;
      c.partials = m->partials;
      cudaEvent_t e1 = nullptr, e2 = nullptr;
      st = prof_begin(m, s, &e1, &e2);
      if (st != KDE_OK) return st;
      CUL(launch_scan_cells(d, grad, c, m->num_sms, &splits, s, false));
      if (e2) CU(cudaEventRecord(e2, s));
      CUL(launch_reduce_splits_mapped(m->partials, splits, c.qpad, q, na, qg, (int)ngroups, c.perm, d_sums, fused, s));
      goto exchange;
    }
    int splits = 1;
    CU(launch_scan_batched(d, grad, a, m->num_sms, &splits, s, true));
    kde_status st = ensure_bytes((void**)&m->partials, &m->partials_cap, sizeof(double) * (size_t)splits * na * q);
    if (st != KDE_OK) return st;
    a.partials = m->partials;
    cudaEvent_t e1 = nullptr, e2 = nullptr;
    st = prof_begin(m, s, &e1, &e2);
    if (st != KDE_OK) return st;
    CUL(launch_scan_batched(d, grad, a, m->num_sms, &splits, s, false));
    if (e2) CU(cudaEventRecord(e2, s));
    CUL(launch_reduce_splits(m->partials, splits, q, na, d_sums, fused, s));
  }
exchange:
  if (fused) {
    CUL(launch_peer_combine(d_sums, q * na, m->pa, m->num_sms, s));
  } else if (m->world > 1) {
    const size_t bytes = sizeof(double) * (size_t)m->world * q * na;
    kde_status st = ensure_bytes((void**)&m->gather, &m->gather_cap, bytes);
    if (st != KDE_OK) return st;
    st = allgather(m, d_sums, m->gather, sizeof(double) * (size_t)q * na, s);
    if (st != KDE_OK) return st;
    CUL(launch_combine_ranks(m->gather, m->world, q, na, d_sums, s));
  }
  return KDE_OK;
}

// est/dpdh (device) for q boxes with device bounds.  A single box also leaves
// (p_hat, dp_hat/dh) in m->ret for the feedback calls (karma / online update).
static kde_status estimate_dev(kde_model* m, const float* d_lo, const float* d_hi, int64_t q, double* d_est,
                               double* d_dpdh, cudaStream_t s, bool retain_c) {
  const bool grad = d_dpdh != nullptr;
  const int na = grad ? m->d + 1 : 1;
  kde_status st = ensure_q(m, q);
  if (st != KDE_OK) return st;
  double* sums = o_sums(m);
  st = scan_sums(m, d_lo, d_hi, q, grad, (q == 1 && retain_c) ? m->cret : nullptr, sums, s, d_est, d_dpdh);
  if (st != KDE_OK) return st;
  if (q == 1 && m->world == 1) return KDE_OK;  // finalised by the scan's last block
  if (q == 1) {
    CUL(launch_finalize(sums, 1, m->d, na, m->consts, (double)m->n_global, m->ret, grad ? m->ret + 1 : nullptr, s));
    if (d_est != m->ret) CU(cudaMemcpyAsync(d_est, m->ret, sizeof(double), cudaMemcpyDeviceToDevice, s));
    if (grad && d_dpdh != m->ret + 1)
      CU(cudaMemcpyAsync(d_dpdh, m->ret + 1, sizeof(double) * m->d, cudaMemcpyDeviceToDevice, s));
    return KDE_OK;
  }
  CUL(launch_finalize(sums, q, m->d, na, m->consts, (double)m->n_global, d_est, d_dpdh, s));
  return KDE_OK;
}

// ------------------------------------------------------------------ ABI: misc
extern "C" int32_t kde_abi_version(void) { return KDE_ABI_VERSION; }
extern "C" const char* kde_last_error(void) { return g_err; }
extern "C" const char* kde_status_string(kde_status s) {
  switch (s) {
    case KDE_OK: return "KDE_OK";
    case KDE_EINVAL: return "KDE_EINVAL";
    case KDE_ENOMEM: return "KDE_ENOMEM";
    case KDE_ECUDA: return "KDE_ECUDA";
    case KDE_ENCCL: return "KDE_ENCCL";
    case KDE_ESTATE: return "KDE_ESTATE";
    case KDE_ETRUNC: return "KDE_ETRUNC";
  }
  return "KDE_UNKNOWN";
}

extern "C" kde_status kde_get_unique_id(void* id_out) {
  kde_model* m = nullptr;
  if (!id_out) return fail(KDE_EINVAL, "id_out is NULL");
  ncclUniqueId id;
  NC(ncclGetUniqueId(&id));
  memcpy(id_out, &id, sizeof(id));
  return KDE_OK;
}

static void free_model(kde_model* m) {
  if (!m) return;
  DeviceGuard g(m->device);
  if (m->stream) cudaStreamSynchronize(m->stream);
  cudaFree(m->cols);
  cudaFree(m->ccols);
  cudaFree(m->cbb);
  cudaFree(m->cscratch);
  cudaFree(m->cstats);
  cudaFree(m->karma);
  cudaFree(m->cret);
  cudaFree(m->consts);
  cudaFree(m->online);
  cudaFree(m->block_partials);
  cudaFree(m->counter);
  cudaFree(m->ret);
  cudaFree(m->single_sums);
  cudaFree(m->qbuf);
  cudaFree(m->obuf);
  cudaFree(m->partials);
  cudaFree(m->order);
  cudaFree(m->gather);
  cudaFree(m->bitmap);
  cudaFree(m->block_counts);
  cudaFree(m->block_offsets);
  cudaFree(m->offsets);
  cudaFree(m->done);
  cudaFree(m->idx_dev);
  cudaFree(m->bad);
  cudaFree(m->scal);
  cudaFree(m->rbuf);
  if (m->pinned) cudaFreeHost(m->pinned);
  for (cudaEvent_t e : m->ev) cudaEventDestroy(e);
  if (m->comm) ncclCommDestroy(m->comm);
  if (m->comm_kind == KDE_COMM_PEER) {
    for (int r = 0; r < m->world; ++r)
      if (r != m->rank && m->pa.base[r]) cudaIpcCloseMemHandle(m->pa.base[r]);
    cudaFree(m->xwin);
    cudaFree(m->pa.epoch);  // epoch, counters and error flag share one allocation
    cudaFree(m->pa_dev);
  }
  cudaFree(m->kbuf);
  if (m->dev_done) cudaEventDestroy(m->dev_done);
  if (m->stream) cudaStreamDestroy(m->stream);
  delete m;
}

extern "C" void kde_destroy(kde_model* m) { free_model(m); }

// ------------------------------------------------------------------ ABI: create
// Scott's rule (eq. 3) over the GLOBAL sample: per-shard moments, all-gathered and Chan-merged in
// rank order (world > 1), then h_j = n^(-1/(d+4)) sigma_j on the device.
static kde_status scott_bandwidth(kde_model* m) {
  const int d = m->d;
  cudaStream_t s = m->stream;
  const int nb = moments_blocks(m->n);
  double* part = nullptr;
  CU(cudaMalloc(&part, sizeof(double) * ((size_t)nb * d * 3 + (size_t)d * 3 * (m->world + 1))));
  double* mom = part + (size_t)nb * d * 3;
  double* gath = mom + (size_t)d * 3;
  kde_status st = KDE_OK;
  cudaError_t e = launch_moments(m->cols, m->ld, m->n, d, part, mom, s);
  ++m->launches;
  if (e == cudaSuccess && m->world > 1) {
    st = allgather(m, mom, gath, sizeof(double) * (size_t)d * 3, s);
    if (st == KDE_OK) e = launch_moments_merge_ranks(gath, m->world, d, mom, s);
  }
  if (e == cudaSuccess && st == KDE_OK) e = launch_scott(mom, d, m->consts, m->bad, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  cudaFree(part);
  if (st != KDE_OK) return st;
  if (e != cudaSuccess) {
    m->poisoned = true;
    return fail(KDE_ECUDA, "Scott bandwidth: %s", cudaGetErrorString(e));
  }
  st = check_peer(m);
  if (st != KDE_OK) return st;
  int32_t bad = 0;
  CU(cudaMemcpy(&bad, m->bad, sizeof(int32_t), cudaMemcpyDeviceToHost));
  if (bad) return fail(KDE_EINVAL, "Scott's rule gives h outside [1e-30, 1e30] (constant column?)");
  return KDE_OK;
}

static size_t peer_slot_bytes() {
  size_t mb = 4;
  if (const char* v = getenv("KDE_PEER_SLOT_MB")) mb = (size_t)std::max(1, atoi(v));
  return mb << 20;
}

static kde_status create_impl(const float* rows, int64_t n_local, int64_t row_offset, int64_t n_global, int32_t d,
                              const double* h, const void* nccl_id, int32_t rank, int32_t world, int comm_kind,
                              kde_model** out) {
  KDE_RANGE();
  if (!out) return fail(KDE_EINVAL, "out is NULL");
  if (d < 1 || d > KDE_MAX_DIM) return fail(KDE_EINVAL, "d = %d outside [1, %d]", d, KDE_MAX_DIM);
  if (world < 1 || rank < 0 || rank >= world) return fail(KDE_EINVAL, "bad rank/world %d/%d", rank, world);
  if (n_global < 2) return fail(KDE_EINVAL, "n = %lld < 2 (eq. 6 divides by n - 1)", (long long)n_global);
  if (n_local < 1 || row_offset < 0 || row_offset + n_local > n_global)
    return fail(KDE_EINVAL, "shard [%lld, %lld) outside [0, %lld) or empty", (long long)row_offset,
                (long long)(row_offset + n_local), (long long)n_global);
  if (!rows) return fail(KDE_EINVAL, "sample is NULL");
  if (world > 1 && comm_kind == KDE_COMM_NCCL && !nccl_id) return fail(KDE_EINVAL, "nccl_id is NULL for world > 1");
  if (world > kMaxWorld) return fail(KDE_EINVAL, "world %d > %d", world, kMaxWorld);
  if (h)
    for (int j = 0; j < d; ++j)
      if (!h_ok(h[j])) return fail(KDE_EINVAL, "h[%d] = %g not finite in [1e-30, 1e30]", j, h[j]);

  kde_model* m = new (std::nothrow) kde_model();
  if (!m) return fail(KDE_ENOMEM, "host allocation failed");
  kde_status st = KDE_OK;
  auto bail = [&](kde_status s2) {
    free_model(m);
    return s2;
  };
  if (cudaGetDevice(&m->device) != cudaSuccess) return bail(fail(KDE_ECUDA, "no CUDA device"));
  cudaDeviceGetAttribute(&m->num_sms, cudaDevAttrMultiProcessorCount, m->device);
  m->d = d;
  m->n = n_local;
  m->n_global = n_global;
  m->row_offset = row_offset;
  m->rank = rank;
  m->world = world;
  m->comm_kind = world > 1 ? comm_kind : KDE_COMM_NONE;
  m->ld = (n_local + kColAlign - 1) / kColAlign * kColAlign;
#define CUB(call)                                                                                   \
  do {                                                                                              \
    cudaError_t e_ = (call);                                                                        \
    if (e_ != cudaSuccess)                                                                          \
      return bail(fail(e_ == cudaErrorMemoryAllocation ? KDE_ENOMEM : KDE_ECUDA, "%s: %s", #call,   \
                       cudaGetErrorString(e_)));                                                    \
  } while (0)
  CUB(cudaStreamCreateWithFlags(&m->stream, cudaStreamNonBlocking));
  CUB(cudaEventCreateWithFlags(&m->dev_done, cudaEventDisableTiming));
  CUB(cudaMalloc(&m->cols, sizeof(float) * (size_t)d * m->ld));
  CUB(cudaMalloc(&m->karma, sizeof(double) * (size_t)m->ld));  // padded: 128-bit karma loads
  CUB(cudaMalloc(&m->cret, sizeof(float) * (size_t)m->ld));
  CUB(cudaMalloc(&m->consts, sizeof(DevConsts)));
  CUB(cudaMalloc(&m->online, sizeof(OnlineState)));
  // single-scan grids are at most 8 CTAs per SM (scan_single_grid)
  CUB(cudaMalloc(&m->block_partials, sizeof(double) * (size_t)m->num_sms * 8 * (kMaxDim + 1)));
  CUB(cudaMalloc(&m->counter, sizeof(unsigned)));
  CUB(cudaMalloc(&m->ret, sizeof(double) * (kMaxDim + 1)));
  CUB(cudaMalloc(&m->single_sums, sizeof(double) * (kMaxDim + 1)));
  CUB(cudaMalloc(&m->bad, sizeof(int32_t)));
  CUB(cudaMalloc(&m->scal, sizeof(double) * 8));
  const int nkb = karma_blocks(n_local);
  CUB(cudaMalloc(&m->bitmap, sizeof(uint32_t) * (size_t)nkb * (kKarmaPts / 32)));
  CUB(cudaMalloc(&m->block_counts, sizeof(int32_t) * (size_t)nkb * 4));  // also the cooperative karma CTA counts (<= passes)
  CUB(cudaMalloc(&m->block_offsets, sizeof(int64_t) * ((size_t)nkb + 1)));
  CUB(cudaMalloc(&m->offsets, sizeof(int64_t) * 2));
  CUB(cudaMalloc(&m->done, 2 * sizeof(unsigned)));
  cudaStream_t s = m->stream;
  CUB(cudaMemsetAsync(m->cols, 0, sizeof(float) * (size_t)d * m->ld, s));
  CUB(cudaMemsetAsync(m->karma, 0, sizeof(double) * (size_t)m->ld, s));
  CUB(cudaMemsetAsync(m->cret, 0, sizeof(float) * (size_t)m->ld, s));
  CUB(cudaMemsetAsync(m->consts, 0, sizeof(DevConsts), s));
  CUB(cudaMemsetAsync(m->online, 0, sizeof(OnlineState), s));
  CUB(cudaMemsetAsync(m->counter, 0, sizeof(unsigned), s));
  CUB(cudaMemsetAsync(m->done, 0, 2 * sizeof(unsigned), s));
  CUB(cudaMemsetAsync(m->bad, 0, sizeof(int32_t), s));

  if (m->comm_kind == KDE_COMM_NCCL) {
    ncclUniqueId id;
    memcpy(&id, nccl_id, sizeof(id));
    ncclResult_t r = ncclCommInitRank(&m->comm, world, id, rank);
    if (r != ncclSuccess) return bail(fail(KDE_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r)));
  } else if (m->comm_kind == KDE_COMM_PEER) {
    // exchange window (flags + 2 parities x world slots), zeroed before its handle is exported
    m->pa.slot = peer_slot_bytes();
    m->xwin_bytes = kPeerFlagBytes + 2 * (size_t)world * m->pa.slot;
    CUB(cudaMalloc(&m->xwin, m->xwin_bytes));
    CUB(cudaMemsetAsync(m->xwin, 0, kPeerFlagBytes, s));
    char* ctl = nullptr;  // epoch (8 B) | 2 arrival counters | error flag
    CUB(cudaMalloc(&ctl, 64));
    CUB(cudaMemsetAsync(ctl, 0, 64, s));
    m->pa.epoch = reinterpret_cast<uint64_t*>(ctl);
    m->pa.count = reinterpret_cast<unsigned*>(ctl + 8);  // 4 counters
    m->pa.err = reinterpret_cast<int*>(ctl + 32);
    m->pa.rank = rank;
    m->pa.world = world;
    double tmo = 60.0;
    if (const char* v = getenv("KDE_PEER_TIMEOUT_S")) tmo = atof(v);
    m->pa.timeout_ns = (uint64_t)(tmo * 1e9);
    for (int r = 0; r < kMaxWorld; ++r) m->pa.base[r] = nullptr;
    m->pa.base[rank] = m->xwin;
    m->attached = false;
  }

  // sample: host row-major -> device (chunked through a pinned buffer) -> SoA columns
  {
    const int64_t chunk_rows = std::max<int64_t>(1, (64ll << 20) / (4ll * d));
    float* d_rows = nullptr;
    const int64_t cr = std::min<int64_t>(chunk_rows, n_local);
    CUB(cudaMalloc(&d_rows, sizeof(float) * (size_t)cr * d));
    st = ensure_pinned(m, sizeof(float) * (size_t)cr * d);
    if (st != KDE_OK) {
      cudaFree(d_rows);
      return bail(st);
    }
    for (int64_t r0 = 0; r0 < n_local; r0 += cr) {
      const int64_t k = std::min<int64_t>(cr, n_local - r0);
      memcpy(m->pinned, rows + r0 * d, sizeof(float) * (size_t)k * d);
      cudaError_t e = cudaMemcpyAsync(d_rows, m->pinned, sizeof(float) * (size_t)k * d, cudaMemcpyHostToDevice, s);
      if (e == cudaSuccess) e = launch_rows_to_cols(d_rows, k, d, m->cols + r0, m->ld, m->bad, s);
      if (e == cudaSuccess) e = cudaStreamSynchronize(s);  // pinned buffer reuse
      if (e != cudaSuccess) {
        cudaFree(d_rows);
        return bail(fail(KDE_ECUDA, "sample upload: %s", cudaGetErrorString(e)));
      }
    }
    cudaFree(d_rows);
    int32_t bad = 0;
    CUB(cudaMemcpy(&bad, m->bad, sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (bad) return bail(fail(KDE_EINVAL, "non-finite value in sample"));
  }

  // column ranges (bound clamping, see DevConsts)
  {
    std::vector<unsigned> init(2 * kMaxDim);
    for (int j = 0; j < kMaxDim; ++j) {
      init[2 * j] = 0xFFFFFFFFu;
      init[2 * j + 1] = 0u;
    }
    m->range_enc = reinterpret_cast<unsigned*>(reinterpret_cast<char*>(m->consts) + offsetof(DevConsts, renc));
    CUB(cudaMemcpyAsync(m->range_enc, init.data(), sizeof(unsigned) * 2 * kMaxDim, cudaMemcpyHostToDevice, s));
    CUB(cudaStreamSynchronize(s));
    ++m->launches;
    CUB(launch_col_range(m->cols, m->ld, n_local, d, m->range_enc, m->consts, s));
  }

  // bandwidth: caller's h, or Scott's rule (eq. 3) over the global sample (peer transport: after attach)
  if (h) {
    CUB(launch_set_consts(h, d, m->consts, s));
  } else if (m->comm_kind == KDE_COMM_PEER) {
    m->h_pending = true;
  } else {
    st = scott_bandwidth(m);
    if (st != KDE_OK) return bail(st);
  }
  CUB(cudaStreamSynchronize(s));
#undef CUB
  *out = m;
  return KDE_OK;
}

extern "C" kde_status kde_create(const float* sample, int64_t n, int32_t d, const double* h, kde_model** out) {
  return create_impl(sample, n, 0, n, d, h, nullptr, 0, 1, KDE_COMM_NONE, out);
}

extern "C" kde_status kde_create_sharded(const float* local_rows, int64_t n_local, int64_t row_offset,
                                         int64_t n_global, int32_t d, const double* h, const void* nccl_id,
                                         int32_t rank, int32_t world, kde_model** out) {
  return create_impl(local_rows, n_local, row_offset, n_global, d, h, nccl_id, rank, world, KDE_COMM_NCCL, out);
}

extern "C" kde_status kde_create_sharded_peer(const float* local_rows, int64_t n_local, int64_t row_offset,
                                              int64_t n_global, int32_t d, const double* h, int32_t rank,
                                              int32_t world, kde_model** out) {
  return create_impl(local_rows, n_local, row_offset, n_global, d, h, nullptr, rank, world,
                     world > 1 ? KDE_COMM_PEER : KDE_COMM_NONE, out);
}

extern "C" kde_status kde_peer_handle(kde_model* m, void* handle_out) {
  if (!m || !handle_out) return fail(KDE_EINVAL, "NULL argument");
  if (m->comm_kind != KDE_COMM_PEER) return fail(KDE_EINVAL, "model does not use the peer transport");
  DeviceGuard g(m->device);
  cudaIpcMemHandle_t hnd;
  CU(cudaIpcGetMemHandle(&hnd, m->xwin));
  static_assert(sizeof(hnd) == KDE_PEER_HANDLE_BYTES, "IPC handle size");
  memcpy(handle_out, &hnd, sizeof(hnd));
  return KDE_OK;
}

extern "C" kde_status kde_peer_attach(kde_model* m, const void* handles) {
  KDE_RANGE();
  if (!m || !handles) return fail(KDE_EINVAL, "NULL argument");
  if (m->comm_kind != KDE_COMM_PEER) return fail(KDE_EINVAL, "model does not use the peer transport");
  if (m->attached) return fail(KDE_ESTATE, "already attached");
  if (m->poisoned) return fail(KDE_ESTATE, "model poisoned by an earlier CUDA/NCCL error");
  DeviceGuard g(m->device);
  for (int r = 0; r < m->world; ++r) {
    if (r == m->rank) continue;
    cudaIpcMemHandle_t hnd;
    memcpy(&hnd, (const char*)handles + (size_t)r * KDE_PEER_HANDLE_BYTES, sizeof(hnd));
    void* p = nullptr;
    CU(cudaIpcOpenMemHandle(&p, hnd, cudaIpcMemLazyEnablePeerAccess));
    m->pa.base[r] = (char*)p;
  }
  CU(cudaMalloc(&m->pa_dev, sizeof(PeerArgs)));
  CU(cudaMemcpy(m->pa_dev, &m->pa, sizeof(PeerArgs), cudaMemcpyHostToDevice));
  m->attached = true;
  if (m->h_pending) {  // Scott's rule needs the all-gather of the shard moments
    m->h_pending = false;
    kde_status st = scott_bandwidth(m);
    if (st != KDE_OK) {
      m->poisoned = true;
      return st;
    }
  }
  return KDE_OK;
}

extern "C" kde_status kde_get_info(const kde_model* m, int64_t* n_local, int64_t* n_global, int32_t* d,
                                   int32_t* rank, int32_t* world) {
  if (!m) return fail(KDE_EINVAL, "model is NULL");
  if (n_local) *n_local = m->n;
  if (n_global) *n_global = m->n_global;
  if (d) *d = m->d;
  if (rank) *rank = m->rank;
  if (world) *world = m->world;
  return KDE_OK;
}

extern "C" kde_status kde_get_bandwidth(kde_model* m, double* h) {
  CHECK_MODEL(m);
  if (!h) return fail(KDE_EINVAL, "h is NULL");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  DevConsts c;
  CU(cudaMemcpyAsync(&c, m->consts, sizeof(DevConsts), cudaMemcpyDeviceToHost, m->stream));
  CU(cudaStreamSynchronize(m->stream));
  for (int j = 0; j < m->d; ++j) h[j] = c.h[j];
  return KDE_OK;
}

extern "C" kde_status kde_set_bandwidth(kde_model* m, const double* h) {
  CHECK_MODEL(m);
  if (!h) return fail(KDE_EINVAL, "h is NULL");
  for (int j = 0; j < m->d; ++j)
    if (!h_ok(h[j])) return fail(KDE_EINVAL, "h[%d] = %g not finite in [1e-30, 1e30]", j, h[j]);
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  CUL(launch_set_consts(h, m->d, m->consts, m->stream));
  CU(cudaStreamSynchronize(m->stream));
  ++m->gen;
  return KDE_OK;
}

extern "C" kde_status kde_set_kernel(kde_model* m, int32_t kernel) {
  CHECK_MODEL(m);
  if (kernel != KDE_KERNEL_GAUSSIAN && kernel != KDE_KERNEL_EPANECHNIKOV)
    return fail(KDE_EINVAL, "unknown kernel %d", kernel);
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  CUL(launch_set_kernel_type(kernel, m->d, m->consts, m->stream));
  CU(cudaStreamSynchronize(m->stream));
  m->kernel = kernel;
  ++m->gen;
  return KDE_OK;
}

extern "C" kde_status kde_get_kernel(const kde_model* m, int32_t* kernel) {
  if (!m || !kernel) return fail(KDE_EINVAL, "NULL argument");
  *kernel = m->kernel;
  return KDE_OK;
}

extern "C" kde_status kde_set_retain(kde_model* m, int32_t on) {
  CHECK_MODEL(m);
  m->retain = on != 0;
  return KDE_OK;
}

extern "C" kde_status kde_set_cull(kde_model* m, int32_t on) {
  CHECK_MODEL(m);
  m->cull = on != 0;
  return KDE_OK;
}

extern "C" kde_status kde_get_cull(const kde_model* m, int32_t* on) {
  if (!m || !on) return fail(KDE_EINVAL, "NULL argument");
  *on = m->cull ? 1 : 0;
  return KDE_OK;
}

extern "C" kde_status kde_set_cells(kde_model* m, int32_t on) {
  CHECK_MODEL(m);
  m->cells_on = on != 0;
  return KDE_OK;
}

extern "C" kde_status kde_get_cells(kde_model* m, int32_t* on, int64_t* builds, int64_t* stats) {
  if (!m || !on) return fail(KDE_EINVAL, "NULL argument");
  *on = m->cells_on ? 1 : 0;
  if (builds) *builds = m->cells_builds;
  if (stats) {
    unsigned long long h[4] = {0, 0, 0, 0};
    if (m->cstats) {
      DeviceGuard g(m->device);
      WAIT_DEV(m);
      CU(cudaStreamSynchronize(m->stream));
      CU(cudaMemcpy(h, m->cstats, sizeof(h), cudaMemcpyDeviceToHost));
      CU(cudaMemset(m->cstats, 0, sizeof(h)));  // counters run from one read to the next
    }
    for (int i = 0; i < 4; ++i) stats[i] = (int64_t)h[i];
  }
  return KDE_OK;
}

extern "C" kde_status kde_synchronize(kde_model* m) {
  CHECK_MODEL(m);
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  CU(cudaStreamSynchronize(m->stream));
  return KDE_OK;
}

// ------------------------------------------------------------------ ABI: estimates
// Stage host bounds into m->qbuf (lo at [0, q*d), hi at [q*d, 2*q*d)).
static kde_status stage_bounds(kde_model* m, const float* lo, const float* hi, int64_t q) {
  const size_t bytes = sizeof(float) * (size_t)q * m->d;
  kde_status st = ensure_q(m, q);
  if (st != KDE_OK) return st;
  st = ensure_pinned(m, 2 * bytes);
  if (st != KDE_OK) return st;
  memcpy(m->pinned, lo, bytes);
  memcpy((char*)m->pinned + bytes, hi, bytes);
  CU(cudaMemcpyAsync(m->qbuf, m->pinned, 2 * bytes, cudaMemcpyHostToDevice, m->stream));
  return KDE_OK;
}

static void note_retained(kde_model* m, const float* lo, const float* hi, bool has_c, bool has_grad) {
  m->ret_valid = true;
  m->ret_has_c = has_c;
  m->ret_has_grad = has_grad;
  m->ret_gen = m->gen;
  memcpy(m->ret_lo, lo, sizeof(float) * m->d);
  memcpy(m->ret_hi, hi, sizeof(float) * m->d);
}

extern "C" kde_status kde_estimate_batch(kde_model* m, const float* lo, const float* hi, int64_t q, double* est,
                                         double* dest_dh) {
  KDE_RANGE();
  CHECK_MODEL(m);
  kde_status st = validate_bounds(lo, hi, q, m->d);
  if (st != KDE_OK) return st;
  if (q > 0 && !est) return fail(KDE_EINVAL, "est is NULL");
  if (q == 0) return KDE_OK;
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  st = stage_bounds(m, lo, hi, q);
  if (st != KDE_OK) return st;
  const float* d_lo = m->qbuf;
  const float* d_hi = m->qbuf + q * m->d;
  const bool grad = dest_dh != nullptr;
  const bool retain_c = m->retain && q == 1;
  double* d_est = q == 1 ? m->ret : o_est(m);
  double* d_dpdh = grad ? (q == 1 ? m->ret + 1 : o_dpdh(m)) : nullptr;
  st = estimate_dev(m, d_lo, d_hi, q, d_est, d_dpdh, m->stream, retain_c);
  if (st != KDE_OK) return st;
  if (q == 1) {
    CU(cudaMemcpyAsync(est, m->ret, sizeof(double), cudaMemcpyDeviceToHost, m->stream));
    if (grad) CU(cudaMemcpyAsync(dest_dh, m->ret + 1, sizeof(double) * m->d, cudaMemcpyDeviceToHost, m->stream));
  } else {
    CU(cudaMemcpyAsync(est, d_est, sizeof(double) * q, cudaMemcpyDeviceToHost, m->stream));
    if (grad) CU(cudaMemcpyAsync(dest_dh, d_dpdh, sizeof(double) * q * m->d, cudaMemcpyDeviceToHost, m->stream));
  }
  CU(cudaStreamSynchronize(m->stream));
  st = check_peer(m);
  if (st != KDE_OK) return st;
  if (q == 1) note_retained(m, lo, hi, retain_c, grad);
  return KDE_OK;
}

extern "C" kde_status kde_estimate_batch_dev(kde_model* m, const float* d_lo, const float* d_hi, int64_t q,
                                             double* d_est, double* d_dest_dh, void* stream) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (q < 0) return fail(KDE_EINVAL, "q < 0");
  if (q == 0) return KDE_OK;
  if (!d_lo || !d_hi || !d_est) return fail(KDE_EINVAL, "NULL device pointer");
  DeviceGuard g(m->device);
  cudaStream_t s = stream ? (cudaStream_t)stream : m->stream;
  m->ret_valid = false;  // bounds are device-side; no retained-state bookkeeping
  kde_status rst = estimate_dev(m, d_lo, d_hi, q, d_est, d_dest_dh, s, m->retain && q == 1);
  if (rst != KDE_OK) return rst;
  return mark_dev(m, s);
}

static kde_status loss_grad_dev_impl(kde_model* m, const float* d_lo, const float* d_hi, const double* d_true,
                                     int64_t q, int32_t loss, double lambda, int32_t log_bw, double* d_loss,
                                     double* d_grad, double* d_est_out, cudaStream_t s) {
  kde_status st = ensure_q(m, q);
  if (st != KDE_OK) return st;
  // the scan below overwrites the retained (p_hat, dp_hat/dh) of a q == 1 batch: whatever box was
  // retained before is no longer what m->ret holds (stale ret_valid after loss_and_grad)
  m->ret_valid = false;
  double* d_est = d_est_out ? d_est_out : o_est(m);
  double* d_dpdh = o_dpdh(m);
  st = estimate_dev(m, d_lo, d_hi, q, d_est, d_dpdh, s, false);
  if (st != KDE_OK) return st;
  CUL(launch_loss_epilogue(d_est, d_dpdh, d_true, q, m->d, loss, lambda, log_bw, m->consts, d_loss, d_grad, s));
  return KDE_OK;
}

extern "C" kde_status kde_loss_and_grad(kde_model* m, const float* lo, const float* hi, const double* true_sel,
                                        int64_t q, int32_t loss, double lambda, int32_t log_bandwidth,
                                        double* loss_out, double* grad_out, double* est_out) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (q < 1) return fail(KDE_EINVAL, "q must be >= 1");
  kde_status st = validate_bounds(lo, hi, q, m->d);
  if (st != KDE_OK) return st;
  st = validate_loss(loss, lambda);
  if (st != KDE_OK) return st;
  if (!true_sel || !loss_out || !grad_out) return fail(KDE_EINVAL, "NULL output/true_sel pointer");
  for (int64_t k = 0; k < q; ++k)
    if (!(true_sel[k] >= 0.0 && true_sel[k] <= 1.0)) return fail(KDE_EINVAL, "true_sel[%lld] outside [0, 1]", (long long)k);
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  st = stage_bounds(m, lo, hi, q);
  if (st != KDE_OK) return st;
  CU(cudaMemcpyAsync(o_true(m), true_sel, sizeof(double) * q, cudaMemcpyHostToDevice, m->stream));
  st = loss_grad_dev_impl(m, m->qbuf, m->qbuf + q * m->d, o_true(m), q, loss, lambda, log_bandwidth, o_loss(m),
                          o_grad(m), o_est(m), m->stream);
  if (st != KDE_OK) return st;
  CU(cudaMemcpyAsync(loss_out, o_loss(m), sizeof(double), cudaMemcpyDeviceToHost, m->stream));
  CU(cudaMemcpyAsync(grad_out, o_grad(m), sizeof(double) * m->d, cudaMemcpyDeviceToHost, m->stream));
  if (est_out) CU(cudaMemcpyAsync(est_out, o_est(m), sizeof(double) * q, cudaMemcpyDeviceToHost, m->stream));
  CU(cudaStreamSynchronize(m->stream));
  return check_peer(m);
}

extern "C" kde_status kde_loss_and_grad_dev(kde_model* m, const float* d_lo, const float* d_hi,
                                            const double* d_true_sel, int64_t q, int32_t loss, double lambda,
                                            int32_t log_bandwidth, double* d_loss, double* d_grad, double* d_est,
                                            void* stream) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (q < 1) return fail(KDE_EINVAL, "q must be >= 1");
  kde_status st = validate_loss(loss, lambda);
  if (st != KDE_OK) return st;
  if (!d_lo || !d_hi || !d_true_sel || !d_loss || !d_grad) return fail(KDE_EINVAL, "NULL device pointer");
  DeviceGuard g(m->device);
  cudaStream_t s = stream ? (cudaStream_t)stream : m->stream;
  m->ret_valid = false;
  kde_status rst = loss_grad_dev_impl(m, d_lo, d_hi, d_true_sel, q, loss, lambda, log_bandwidth, d_loss, d_grad, d_est, s);
  if (rst != KDE_OK) return rst;
  return mark_dev(m, s);
}

// ------------------------------------------------------------------ feedback parameter checks
static kde_status karma_params_dev(const kde_karma_params* kp, KarmaParamsDev* kd) {
  if (!kp) return fail(KDE_EINVAL, "NULL karma params");
  kde_status st = validate_loss(kp->loss, kp->lambda);
  if (st != KDE_OK) return st;
  if (std::isnan(kp->k_max) || std::isnan(kp->threshold)) return fail(KDE_EINVAL, "NaN k_max / threshold");
  kd->loss = kp->loss;
  kd->empty_region = kp->empty_region;
  kd->lambda = kp->lambda;
  kd->k_max = kp->k_max;
  kd->threshold = kp->threshold;
  return KDE_OK;
}

static kde_status online_params_dev(kde_model* m, const kde_online_params* op, OnlineParamsDev* od, cudaStream_t s) {
  if (!op) return fail(KDE_EINVAL, "NULL online params");
  kde_status st = validate_loss(op->loss, op->lambda);
  if (st != KDE_OK) return st;
  if (op->minibatch < 1 || !(op->alpha >= 0.0 && op->alpha < 1.0) || !(op->lr_min > 0.0) ||
      !(op->lr_max >= op->lr_min) || !(op->lr_inc >= 1.0) || !(op->lr_dec > 0.0 && op->lr_dec <= 1.0) ||
      !(op->lr0 > 0.0))
    return fail(KDE_EINVAL, "bad online parameters");
  if (!m->online_init) {
    OnlineState s0;
    memset(&s0, 0, sizeof(s0));
    for (int j = 0; j < kMaxDim; ++j) s0.lr[j] = op->lr0;
    CU(cudaMemcpyAsync(m->online, &s0, sizeof(s0), cudaMemcpyHostToDevice, s));
    CU(cudaStreamSynchronize(s));
    m->online_init = true;
  }
  od->minibatch = op->minibatch;
  od->log_bw = op->log_bandwidth;
  od->loss = op->loss;
  od->lambda = op->lambda;
  od->alpha = op->alpha;
  od->lr_min = op->lr_min;
  od->lr_max = op->lr_max;
  od->lr_inc = op->lr_inc;
  od->lr_dec = op->lr_dec;
  return KDE_OK;
}

// ------------------------------------------------------------------ ABI: feedback
static bool retained_matches(kde_model* m, const float* lo, const float* hi, bool need_c, bool need_grad) {
  if (!m->ret_valid || m->ret_gen != m->gen) return false;
  if (need_c && !m->ret_has_c) return false;
  if (need_grad && !m->ret_has_grad) return false;
  return memcmp(m->ret_lo, lo, sizeof(float) * m->d) == 0 && memcmp(m->ret_hi, hi, sizeof(float) * m->d) == 0;
}

// Make sure m->ret (p_hat, dp/dh) and (need_c) m->cret hold this box's values.
static kde_status ensure_retained(kde_model* m, const float* lo, const float* hi, bool need_c, bool need_grad) {
  if (retained_matches(m, lo, hi, need_c, need_grad)) {
    // bounds of the retained query are still needed on the device (karma eq. 20)
    kde_status st = stage_bounds(m, lo, hi, 1);
    return st;
  }
  kde_status st = stage_bounds(m, lo, hi, 1);
  if (st != KDE_OK) return st;
  const bool grad = need_grad;
  st = estimate_dev(m, m->qbuf, m->qbuf + m->d, 1, m->ret, grad ? m->ret + 1 : nullptr, m->stream, true);
  if (st != KDE_OK) return st;
  note_retained(m, lo, hi, true, grad);
  return KDE_OK;
}

extern "C" kde_status kde_karma_update(kde_model* m, const float* lo, const float* hi, double true_sel,
                                       const kde_karma_params* kp, int64_t* idx_out, int64_t idx_cap,
                                       int64_t* n_flagged) {
  KDE_RANGE();
  CHECK_MODEL(m);
  kde_status st = validate_bounds(lo, hi, 1, m->d);
  if (st != KDE_OK) return st;
  if (!kp || !n_flagged) return fail(KDE_EINVAL, "NULL karma params / n_flagged");
  if (idx_cap < 0 || (idx_cap > 0 && !idx_out)) return fail(KDE_EINVAL, "bad idx_out / idx_cap");
  if (!(true_sel >= 0.0 && true_sel <= 1.0)) return fail(KDE_EINVAL, "true_sel outside [0, 1]");
  st = validate_loss(kp->loss, kp->lambda);
  if (st != KDE_OK) return st;
  if (std::isnan(kp->k_max) || std::isnan(kp->threshold)) return fail(KDE_EINVAL, "NaN k_max / threshold");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  st = ensure_retained(m, lo, hi, true, false);
  if (st != KDE_OK) return st;
  // index output buffer: local flags at most n
  const int64_t local_cap = m->n;
  if (m->idx_cap < local_cap) {
    cudaFree(m->idx_dev);
    m->idx_dev = nullptr;
    if (cudaMalloc(&m->idx_dev, sizeof(int64_t) * (size_t)local_cap) != cudaSuccess) return fail(KDE_ENOMEM, "idx buffer");
    m->idx_cap = local_cap;
  }
  KarmaParamsDev kd;
  kd.loss = kp->loss;
  kd.empty_region = kp->empty_region;
  kd.lambda = kp->lambda;
  kd.k_max = kp->k_max;
  kd.threshold = kp->threshold;
  CU(cudaMemcpyAsync(m->scal, &true_sel, sizeof(double), cudaMemcpyHostToDevice, m->stream));
  m->launches += karma_launches() - 1;  // CUL counts one
  CUL(launch_karma(m->cret, m->karma, m->n, (double)m->n_global, m->ret, m->scal, kd, m->qbuf, m->qbuf + m->d, m->d,
                  m->consts, m->bitmap, m->block_counts, m->block_offsets, m->done, m->row_offset, m->idx_dev, local_cap, m->offsets,
                  StreamTail{}, m->stream));
  int64_t local_total = 0;
  CU(cudaMemcpyAsync(&local_total, m->offsets, sizeof(int64_t), cudaMemcpyDeviceToHost, m->stream));
  CU(cudaStreamSynchronize(m->stream));
  if (m->world == 1) {
    const int64_t ncopy = std::min(local_total, idx_cap);
    if (ncopy > 0) CU(cudaMemcpy(idx_out, m->idx_dev, sizeof(int64_t) * ncopy, cudaMemcpyDeviceToHost));
    *n_flagged = local_total;
    return local_total > idx_cap ? fail(KDE_ETRUNC, "%lld flagged > idx_cap %lld", (long long)local_total, (long long)idx_cap)
                                 : KDE_OK;
  }
  // world > 1: all-gather the counts, then the (ascending) index lists; concatenated in rank
  // order they are the ascending GLOBAL list (contiguous row shards)
  const size_t cnt_bytes = sizeof(int64_t) * (size_t)(m->world + 1);
  st = ensure_bytes(&m->kbuf, &m->kbuf_cap, cnt_bytes);
  if (st != KDE_OK) return st;
  int64_t* d_cnt = (int64_t*)m->kbuf;  // [world] gathered + [1] own
  CU(cudaMemcpyAsync(d_cnt + m->world, m->offsets, sizeof(int64_t), cudaMemcpyDeviceToDevice, m->stream));
  st = allgather(m, d_cnt + m->world, d_cnt, sizeof(int64_t), m->stream);
  if (st != KDE_OK) return st;
  std::vector<int64_t> counts(m->world);
  CU(cudaMemcpyAsync(counts.data(), d_cnt, sizeof(int64_t) * m->world, cudaMemcpyDeviceToHost, m->stream));
  CU(cudaStreamSynchronize(m->stream));
  st = check_peer(m);
  if (st != KDE_OK) return st;
  int64_t maxc = 0, total = 0;
  for (int64_t c : counts) {
    maxc = std::max(maxc, c);
    total += c;
  }
  *n_flagged = total;
  if (maxc > 0) {
    // only the first idx_cap indices are returned: no rank sends more than that
    const int64_t send = std::min(maxc, std::max<int64_t>(idx_cap, 1));
    st = ensure_bytes(&m->kbuf, &m->kbuf_cap, cnt_bytes + sizeof(int64_t) * (size_t)send * (m->world + 1));
    if (st != KDE_OK) return st;
    d_cnt = (int64_t*)m->kbuf;
    int64_t* d_all = d_cnt + m->world + 1;
    int64_t* d_send = d_all + (size_t)send * m->world;
    const int64_t mine = std::min(local_total, send);
    if (mine > 0) CU(cudaMemcpyAsync(d_send, m->idx_dev, sizeof(int64_t) * mine, cudaMemcpyDeviceToDevice, m->stream));
    st = allgather(m, d_send, d_all, sizeof(int64_t) * (size_t)send, m->stream);
    if (st != KDE_OK) return st;
    int64_t pos = 0;
    for (int rr = 0; rr < m->world && pos < idx_cap; ++rr) {
      const int64_t k = std::min(std::min(counts[rr], send), idx_cap - pos);
      if (k > 0)
        CU(cudaMemcpyAsync(idx_out + pos, d_all + (size_t)rr * send, sizeof(int64_t) * k, cudaMemcpyDeviceToHost,
                           m->stream));
      pos += k;
    }
    CU(cudaStreamSynchronize(m->stream));
    st = check_peer(m);
    if (st != KDE_OK) return st;
  }
  return total > idx_cap ? fail(KDE_ETRUNC, "%lld flagged > idx_cap %lld", (long long)total, (long long)idx_cap) : KDE_OK;
}

extern "C" kde_status kde_online_update(kde_model* m, const float* lo, const float* hi, double true_sel,
                                        const kde_online_params* op, int32_t* updated) {
  KDE_RANGE();
  CHECK_MODEL(m);
  kde_status st = validate_bounds(lo, hi, 1, m->d);
  if (st != KDE_OK) return st;
  if (!(true_sel >= 0.0 && true_sel <= 1.0)) return fail(KDE_EINVAL, "true_sel outside [0, 1]");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  OnlineParamsDev od;
  st = online_params_dev(m, op, &od, m->stream);
  if (st != KDE_OK) return st;
  st = ensure_retained(m, lo, hi, false, true);
  if (st != KDE_OK) return st;
  CU(cudaMemcpyAsync(m->scal + 1, &true_sel, sizeof(double), cudaMemcpyHostToDevice, m->stream));
  CUL(launch_online_update(m->ret, m->scal + 1, od, m->d, m->online, m->consts, m->stream));
  int32_t upd = 0;
  CU(cudaMemcpyAsync(&upd, &m->online->updated, sizeof(int32_t), cudaMemcpyDeviceToHost, m->stream));
  CU(cudaStreamSynchronize(m->stream));
  if (upd) ++m->gen;
  if (updated) *updated = upd;
  return KDE_OK;
}

// Rows owned by this shard -> device staging (grow-only buffer, no per-call allocation) -> scatter.
// idx are validated GLOBAL indices, unique; rows host row-major k x d.
static kde_status replace_impl(kde_model* m, const int64_t* idx, const float* rows, int64_t k, double k_init,
                               cudaStream_t as = nullptr) {
  std::vector<int64_t> li;
  std::vector<float> lr;
  for (int64_t r = 0; r < k; ++r) {
    const int64_t i = idx[r] - m->row_offset;
    if (i >= 0 && i < m->n) {
      li.push_back(i);
      lr.insert(lr.end(), rows + r * m->d, rows + (r + 1) * m->d);
    }
  }
  const int64_t kl = (int64_t)li.size();
  if (kl > 0) {
    const size_t ib = sizeof(int64_t) * kl, rb = sizeof(float) * kl * m->d;
    cudaStream_t s = as ? as : m->stream;
    void* pin = nullptr;
    int b = 0;
    if (as) {  // async: the staging buffer of two calls ago is free once its copy completed
      b = m->apin_next;
      m->apin_next ^= 1;
      if (!m->apin_ev[b]) CU(cudaEventCreateWithFlags(&m->apin_ev[b], cudaEventDisableTiming));
      CU(cudaEventSynchronize(m->apin_ev[b]));
      if (m->apin_cap[b] < ib + rb) {
        if (m->apin[b]) cudaFreeHost(m->apin[b]);
        m->apin[b] = nullptr;
        m->apin_cap[b] = 0;
        const size_t cap = std::max<size_t>(ib + rb, (size_t)1 << 20);
        if (cudaMallocHost(&m->apin[b], cap) != cudaSuccess) return fail(KDE_ENOMEM, "pinned staging of %zu bytes", cap);
        m->apin_cap[b] = cap;
      }
      pin = m->apin[b];
    } else {
      kde_status st = ensure_pinned(m, ib + rb);
      if (st != KDE_OK) return st;
      pin = m->pinned;
    }
    kde_status st = ensure_bytes(&m->rbuf, &m->rbuf_cap, ib + rb);  // (a reallocation synchronises the device)
    if (st != KDE_OK) return st;
    memcpy(pin, li.data(), ib);
    memcpy((char*)pin + ib, lr.data(), rb);
    CU(cudaMemcpyAsync(m->rbuf, pin, ib + rb, cudaMemcpyHostToDevice, s));
    if (as) CU(cudaEventRecord(m->apin_ev[b], s));
    CUL(launch_row_range((const float*)((char*)m->rbuf + ib), kl, m->d, m->range_enc, m->consts, s));
    CUL(launch_scatter_rows((const int64_t*)m->rbuf, (const float*)((char*)m->rbuf + ib), kl, m->d, m->cols, m->ld,
                           m->karma, k_init, s));
    ++m->sgen;
    if (!as) CU(cudaStreamSynchronize(m->stream));  // the pinned staging buffer is reused by the next call
  }
  ++m->gen;
  return KDE_OK;
}

extern "C" kde_status kde_replace_points(kde_model* m, const int64_t* idx, const float* rows, int64_t k,
                                         double k_init) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (k < 0) return fail(KDE_EINVAL, "k < 0");
  if (k == 0) return KDE_OK;
  if (!idx || !rows) return fail(KDE_EINVAL, "NULL idx / rows");
  if (!std::isfinite(k_init)) return fail(KDE_EINVAL, "k_init not finite");
  std::vector<int64_t> sorted(idx, idx + k);
  std::sort(sorted.begin(), sorted.end());
  for (int64_t r = 0; r < k; ++r) {
    if (sorted[r] < 0 || sorted[r] >= m->n_global) return fail(KDE_EINVAL, "index %lld out of range", (long long)sorted[r]);
    if (r > 0 && sorted[r] == sorted[r - 1]) return fail(KDE_EINVAL, "duplicate index %lld", (long long)sorted[r]);
  }
  for (int64_t e = 0; e < k * m->d; ++e)
    if (!std::isfinite(rows[e])) return fail(KDE_EINVAL, "non-finite value in replacement rows");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  return replace_impl(m, idx, rows, k, k_init);
}

// ------------------------------------------------------------------ ABI: reservoir inserts
extern "C" kde_status kde_reservoir_select(uint64_t seed, int64_t n_sample, int64_t n_seen, int64_t k,
                                           int64_t* slot_out) {
  if (n_sample < 1) return fail(KDE_EINVAL, "n_sample < 1");
  if (n_seen < 0 || k < 0 || n_seen > INT64_MAX - k) return fail(KDE_EINVAL, "bad n_seen / k");
  if (k > 0 && !slot_out) return fail(KDE_EINVAL, "slot_out is NULL");
  reservoir_slots(seed, n_sample, n_seen, k, slot_out);
  return KDE_OK;
}

static kde_status insert_impl(kde_model* m, const float* rows, int64_t k, uint64_t seed, int64_t* n_seen,
                              double k_init, int64_t* n_written, cudaStream_t as);

extern "C" kde_status kde_insert_rows(kde_model* m, const float* rows, int64_t k, uint64_t seed, int64_t* n_seen,
                                      double k_init, int64_t* n_written) {
  KDE_RANGE();
  CHECK_MODEL(m);
  return insert_impl(m, rows, k, seed, n_seen, k_init, n_written, nullptr);
}

extern "C" kde_status kde_insert_rows_async(kde_model* m, const float* rows, int64_t k, uint64_t seed,
                                            int64_t* n_seen, double k_init, int64_t* n_written, void* stream) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (m->world != 1) return fail(KDE_EINVAL, "kde_insert_rows_async is single-GPU (world == 1)");
  cudaStream_t s = stream ? (cudaStream_t)stream : m->stream;
  kde_status st = insert_impl(m, rows, k, seed, n_seen, k_init, n_written, s);
  if (st != KDE_OK) return st;
  return mark_dev(m, s);
}

static kde_status insert_impl(kde_model* m, const float* rows, int64_t k, uint64_t seed, int64_t* n_seen,
                              double k_init, int64_t* n_written, cudaStream_t as) {
  if (k < 0 || !n_seen || *n_seen < 0 || *n_seen > INT64_MAX - k) return fail(KDE_EINVAL, "bad k / n_seen");
  if (k > 0 && !rows) return fail(KDE_EINVAL, "rows is NULL");
  if (!std::isfinite(k_init)) return fail(KDE_EINVAL, "k_init not finite");
  {  // every arriving value finite (branch-free exponent test, vectorisable)
    const uint32_t* bits = reinterpret_cast<const uint32_t*>(rows);
    uint32_t bad = 0;
    for (int64_t e = 0; e < k * m->d; ++e) bad |= (uint32_t)((bits[e] & 0x7f800000u) == 0x7f800000u);
    if (bad) return fail(KDE_EINVAL, "non-finite value in inserted rows");
  }
  std::vector<int64_t> slot((size_t)k);
  reservoir_slots(seed, m->n_global, *n_seen, k, slot.data());
  // several arrivals of one chunk may take the same slot: the last one wins (sequential semantics);
  // only this shard's winners are transferred.  O(k): the accepted arrivals of this shard
  // (a small fraction of k once the stream is long) are walked newest first through an
  // open-addressing set of their slots sized to that count, so the host touches a few cache-resident
  // kilobytes instead of an n-entry table.
  std::vector<int32_t> acc;  // accepted arrivals of this shard, in arrival order
  for (int64_t r = 0; r < k; ++r) {
    const int64_t i = slot[r] - m->row_offset;
    if (slot[r] >= 0 && i >= 0 && i < m->n) acc.push_back((int32_t)r);
  }
  size_t cap = 16;
  while (cap < 2 * acc.size()) cap <<= 1;
  std::vector<int64_t> set(cap, -1);
  std::vector<char> win(acc.size(), 0);
  for (size_t a = acc.size(); a-- > 0;) {
    const int64_t sl = slot[(size_t)acc[a]];
    size_t hsh = (size_t)((uint64_t)sl * 0x9E3779B97F4A7C15ull >> 20) & (cap - 1);
    while (set[hsh] >= 0 && set[hsh] != sl) hsh = (hsh + 1) & (cap - 1);
    if (set[hsh] < 0) {  // newest arrival for this slot
      set[hsh] = sl;
      win[a] = 1;
    }
  }
  std::vector<int64_t> idx;
  std::vector<float> sel;
  idx.reserve(acc.size());
  sel.reserve(acc.size() * (size_t)m->d);
  for (size_t a = 0; a < acc.size(); ++a)
    if (win[a]) {
      const int64_t r = acc[a];
      idx.push_back(slot[(size_t)r]);
      sel.insert(sel.end(), rows + r * m->d, rows + (r + 1) * m->d);
    }
  DeviceGuard g(m->device);
  if (!as) WAIT_DEV(m);
  kde_status st = idx.empty() ? KDE_OK : replace_impl(m, idx.data(), sel.data(), (int64_t)idx.size(), k_init, as);
  if (st != KDE_OK) return st;
  ++m->gen;
  *n_seen += k;
  if (n_written) *n_written = (int64_t)idx.size();
  return KDE_OK;
}

extern "C" kde_status kde_karma_update_dev(kde_model* m, const float* d_lo, const float* d_hi,
                                           const double* d_true_sel, const kde_karma_params* kp, int64_t* d_idx_out,
                                           int64_t idx_cap, int64_t* d_n_flagged, void* stream) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (m->world != 1) return fail(KDE_EINVAL, "device-resident feedback calls are single-GPU (world == 1)");
  if (!d_lo || !d_hi || !d_true_sel || !d_n_flagged || idx_cap < 0 || (idx_cap > 0 && !d_idx_out))
    return fail(KDE_EINVAL, "NULL device pointer / bad idx_cap");
  KarmaParamsDev kd;
  kde_status st = karma_params_dev(kp, &kd);
  if (st != KDE_OK) return st;
  DeviceGuard g(m->device);
  cudaStream_t s = stream ? (cudaStream_t)stream : m->stream;
  m->launches += karma_launches() - 1;  // CUL counts one
  CUL(launch_karma(m->cret, m->karma, m->n, (double)m->n_global, m->ret, d_true_sel, kd, d_lo, d_hi, m->d,
                   m->consts, m->bitmap, m->block_counts, m->block_offsets, m->done, m->row_offset, d_idx_out, idx_cap, d_n_flagged,
                   StreamTail{}, s));
  return mark_dev(m, s);
}

extern "C" kde_status kde_online_update_dev(kde_model* m, const double* d_true_sel, const kde_online_params* op,
                                            void* stream) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (!d_true_sel) return fail(KDE_EINVAL, "NULL device pointer");
  DeviceGuard g(m->device);
  cudaStream_t s = stream ? (cudaStream_t)stream : m->stream;
  OnlineParamsDev od;
  kde_status st = online_params_dev(m, op, &od, s);
  if (st != KDE_OK) return st;
  CUL(launch_online_update(m->ret, d_true_sel, od, m->d, m->online, m->consts, s));
  ++m->gen;
  return mark_dev(m, s);
}

extern "C" kde_status kde_replace_points_dev(kde_model* m, const int64_t* d_idx, const float* d_rows,
                                             const int64_t* d_k, int64_t cap, double k_init, void* stream) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (cap < 0 || (cap > 0 && (!d_idx || !d_rows || !d_k))) return fail(KDE_EINVAL, "NULL device pointer / cap");
  if (!std::isfinite(k_init)) return fail(KDE_EINVAL, "k_init not finite");
  DeviceGuard g(m->device);
  cudaStream_t s = stream ? (cudaStream_t)stream : m->stream;
  ++m->launches;
  CUL(launch_scatter_rows_dev(d_idx, d_rows, d_k, cap, m->d, m->cols, m->ld, m->n, m->row_offset, m->karma, k_init,
                              m->range_enc, m->consts, s));
  ++m->sgen;
  ++m->gen;
  return mark_dev(m, s);
}

// One device-resident streaming step in three kernels: the
// single-box scan (estimate, gradient when op != NULL, retained p^(i)), the
// karma pass, and the fused compaction whose last block also runs the
// Listing 1 step and replaces the flagged points by d_rows.
extern "C" kde_status kde_stream_step_dev(kde_model* m, const float* d_lo, const float* d_hi,
                                          const double* d_true_sel, const kde_karma_params* kp,
                                          const kde_online_params* op, int64_t* d_idx_out, int64_t idx_cap,
                                          int64_t* d_n_flagged, const float* d_rows, double k_init, double* d_est,
                                          double* d_dpdh, void* stream) {
  KDE_RANGE();
  CHECK_MODEL(m);
  if (m->world != 1) return fail(KDE_EINVAL, "device-resident streaming step is single-GPU (world == 1)");
  if (!d_lo || !d_hi || !d_true_sel || !d_n_flagged || !d_est || idx_cap < 0 || (idx_cap > 0 && !d_idx_out))
    return fail(KDE_EINVAL, "NULL device pointer / bad idx_cap");
  if (op && !d_dpdh) return fail(KDE_EINVAL, "the online update needs d_dpdh (gradient of the estimate)");
  if (!std::isfinite(k_init)) return fail(KDE_EINVAL, "k_init not finite");
  KarmaParamsDev kd;
  kde_status st = karma_params_dev(kp, &kd);
  if (st != KDE_OK) return st;
  DeviceGuard g(m->device);
  cudaStream_t s = stream ? (cudaStream_t)stream : m->stream;
  StreamTail tail;
  if (op) {
    st = online_params_dev(m, op, &tail.op, s);
    if (st != KDE_OK) return st;
    tail.online = 1;
    tail.ret = m->ret;
    tail.p = d_true_sel;
    tail.st = m->online;
  }
  tail.c = m->consts;
  tail.d = m->d;
  if (d_rows && idx_cap > 0) {
    tail.rows = d_rows;
    tail.cols = m->cols;
    ++m->sgen;  // the tail may replace flagged rows
    tail.ld = m->ld;
    tail.karma = m->karma;
    tail.k_init = k_init;
  }
  m->ret_valid = false;
  st = estimate_dev(m, d_lo, d_hi, 1, d_est, op ? d_dpdh : nullptr, s, true);
  if (st != KDE_OK) return st;
  m->launches += karma_launches() - 1;  // CUL counts one
  CUL(launch_karma(m->cret, m->karma, m->n, (double)m->n_global, m->ret, d_true_sel, kd, d_lo, d_hi, m->d,
                   m->consts, m->bitmap, m->block_counts, m->block_offsets, m->done, m->row_offset, d_idx_out, idx_cap, d_n_flagged,
                   tail, s));
  ++m->gen;
  return mark_dev(m, s);
}

// ------------------------------------------------------------------ inspection
extern "C" kde_status kde_get_karma(kde_model* m, double* karma) {
  CHECK_MODEL(m);
  if (!karma) return fail(KDE_EINVAL, "NULL karma");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  CU(cudaStreamSynchronize(m->stream));
  CU(cudaMemcpy(karma, m->karma, sizeof(double) * m->n, cudaMemcpyDeviceToHost));
  return KDE_OK;
}

extern "C" kde_status kde_set_karma(kde_model* m, const double* karma) {
  CHECK_MODEL(m);
  if (!karma) return fail(KDE_EINVAL, "NULL karma");
  for (int64_t i = 0; i < m->n; ++i)
    if (std::isnan(karma[i])) return fail(KDE_EINVAL, "NaN karma");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  CU(cudaStreamSynchronize(m->stream));
  CU(cudaMemcpy(m->karma, karma, sizeof(double) * m->n, cudaMemcpyHostToDevice));
  return KDE_OK;
}

extern "C" kde_status kde_get_sample(kde_model* m, float* rows) {
  CHECK_MODEL(m);
  if (!rows) return fail(KDE_EINVAL, "NULL rows");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  float* d_rows = nullptr;
  CU(cudaMalloc(&d_rows, sizeof(float) * (size_t)m->n * m->d));
  CUL(launch_cols_to_rows(m->cols, m->ld, m->n, m->d, d_rows, m->stream));
  CU(cudaStreamSynchronize(m->stream));
  CU(cudaMemcpy(rows, d_rows, sizeof(float) * (size_t)m->n * m->d, cudaMemcpyDeviceToHost));
  cudaFree(d_rows);
  return KDE_OK;
}

extern "C" kde_status kde_get_contributions(kde_model* m, float* c) {
  CHECK_MODEL(m);
  if (!c) return fail(KDE_EINVAL, "NULL c");
  if (!m->ret_valid || !m->ret_has_c) return fail(KDE_ESTATE, "no retained contributions");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  CU(cudaStreamSynchronize(m->stream));
  CU(cudaMemcpy(c, m->cret, sizeof(float) * m->n, cudaMemcpyDeviceToHost));
  return KDE_OK;
}

extern "C" kde_status kde_get_online_state(kde_model* m, double* acc, double* ms, double* lr, double* gprev,
                                           int32_t* count) {
  CHECK_MODEL(m);
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  OnlineState s;
  CU(cudaStreamSynchronize(m->stream));
  CU(cudaMemcpy(&s, m->online, sizeof(s), cudaMemcpyDeviceToHost));
  const size_t b = sizeof(double) * m->d;
  if (acc) memcpy(acc, s.acc, b);
  if (ms) memcpy(ms, s.ms, b);
  if (lr) memcpy(lr, s.lr, b);
  if (gprev) memcpy(gprev, s.gprev, b);
  if (count) *count = s.count;
  return KDE_OK;
}

extern "C" kde_status kde_set_online_state(kde_model* m, const double* acc, const double* ms, const double* lr,
                                           const double* gprev, int32_t count) {
  CHECK_MODEL(m);
  if (!acc || !ms || !lr || !gprev || count < 0) return fail(KDE_EINVAL, "bad online state");
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  OnlineState s;
  memset(&s, 0, sizeof(s));
  const size_t b = sizeof(double) * m->d;
  memcpy(s.acc, acc, b);
  memcpy(s.ms, ms, b);
  memcpy(s.lr, lr, b);
  memcpy(s.gprev, gprev, b);
  s.count = count;
  CU(cudaStreamSynchronize(m->stream));
  CU(cudaMemcpy(m->online, &s, sizeof(s), cudaMemcpyHostToDevice));
  m->online_init = true;
  return KDE_OK;
}

extern "C" kde_status kde_set_profiling(kde_model* m, int32_t on) {
  CHECK_MODEL(m);
  m->prof = on != 0;
  if (m->cstats) {
    DeviceGuard g(m->device);
    WAIT_DEV(m);
    CU(cudaMemset(m->cstats, 0, 4 * sizeof(unsigned long long)));
  }
  m->ev_used = 0;
  m->scan_launches = 0;
  m->launches = 0;
  return KDE_OK;
}

extern "C" kde_status kde_get_profile(kde_model* m, double* scan_ms, int64_t* scan_launches, int64_t* launches) {
  CHECK_MODEL(m);
  DeviceGuard g(m->device);
  WAIT_DEV(m);
  CU(cudaDeviceSynchronize());
  double tot = 0.0;
  for (size_t i = 0; i + 1 < m->ev_used; i += 2) {
    float ms = 0.f;
    CU(cudaEventElapsedTime(&ms, m->ev[i], m->ev[i + 1]));
    tot += ms;
  }
  if (scan_ms) *scan_ms = tot;
  if (scan_launches) *scan_launches = m->scan_launches;
  if (launches) *launches = m->launches;
  m->ev_used = 0;
  m->scan_launches = 0;
  m->launches = 0;
  return KDE_OK;
}

// ------------------------------------------------------------------ harness
extern "C" kde_status kde_count_in_box_dev(const float* d_rows, int64_t n, int32_t d, const float* d_lo,
                                           const float* d_hi, int64_t q, int64_t* d_counts, void* stream) {
  kde_model* m = nullptr;
  if (d < 1 || d > KDE_MAX_DIM || n < 0 || q < 0) return fail(KDE_EINVAL, "bad count_in_box arguments");
  if (q == 0) return KDE_OK;
  if (!d_rows || !d_lo || !d_hi || !d_counts) return fail(KDE_EINVAL, "NULL device pointer");
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaStream_t s = (cudaStream_t)stream;
  CU(cudaMemsetAsync(d_counts, 0, sizeof(int64_t) * q, s));
  CU(launch_count_in_box(d_rows, n, d, d_lo, d_hi, q, (unsigned long long*)d_counts, sms, s));
  return KDE_OK;
}
