/*
 * kde.h -- C ABI of the B200-native KDE range-selectivity hot path.
 *
 * Method: Heimel, Kiefer, Markl, "Self-Tuning, GPU-Accelerated Kernel Density
 * Models for Multidimensional Selectivity Estimation", SIGMOD 2015.
 * Citations "P:L<n>" are line numbers of the paper text.
 *
 * A model owns a d-dimensional fp32 data sample S = {t^(1..s)} resident in
 * device memory (structure-of-arrays columns), a diagonal Gaussian bandwidth
 * H = diag(h_1..h_d), per-point cumulative karma K_i (eq. 8) and the
 * retained per-point contributions of the last single-query scan.
 *
 * Conventions for every entry point
 *  - Return value: KDE_OK or an error code; nothing throws across the ABI.
 *    kde_last_error() returns a thread-local message for the last failure.
 *  - Validation happens before any device work, so KDE_EINVAL leaves the
 *    model unchanged.  A CUDA / NCCL failure after launch poisons the model:
 *    every later call returns KDE_ESTATE (only kde_destroy is valid).
 *  - Host pointers: the library copies inputs during the call; outputs go to
 *    caller-allocated buffers; the caller keeps ownership of everything.
 *    Host-pointer calls are synchronous (they return after results landed).
 *  - "_dev" variants take DEVICE pointers (on the model's device) and a CUDA
 *    stream (cudaStream_t passed as void*, NULL = the model's own stream; the
 *    legacy default stream is passed as cudaStreamLegacy -- the Python binding
 *    maps torch's default stream, whose handle is 0, to it);
 *    they only enqueue work: results are valid once that stream reaches the
 *    end of the enqueued work.  Device buffers must stay alive until then.
 *    Every call that uses the model's own stream (all host-pointer calls,
 *    getters, setters) is ordered after the work of the _dev calls issued
 *    before it (an event recorded at the end of each _dev call, also inside
 *    CUDA-graph capture); ordering between _dev calls on DIFFERENT caller
 *    streams is the caller's job.
 *  - Box queries are hyper-rectangles Omega = (l_1,u_1) x ... x (l_d,u_d)
 *    over real-valued attributes, passed as row-major fp32 arrays
 *    lo[q][d], hi[q][d].  lo <= hi is required (lo == hi gives 0);
 *    +-infinity is allowed (half-open / unbounded boxes); NaN is rejected.
 *  - Sharded models (one process per GPU): every rank calls every function
 *    collectively with identical query arguments; point indices are GLOBAL.
 *  - A model is externally synchronised (one thread at a time).
 *
 * Environment (read by the library)
 *  - KDE_DEBUG_SYNC=1      synchronise after every kernel launch, so a fault
 *                          is reported by the call that launched it (debug).
 *  - KDE_PEER_TIMEOUT_S    bound on a peer-exchange wait (default 60 s).
 *  - KDE_PEER_SLOT_MB      peer exchange window slot size (default 4 MiB).
 *  - KDE_PEER_FUSED=0      peer transport: separate all-gather instead of the
 *                          producer-tail push (A/B testing).
 *  - KDE_KARMA_TWO_PASS=1  karma pass as two kernels instead of the
 *                          cooperative one (A/B timing).
 *  Every entry point that does device work opens an NVTX range named after it.
 */
#ifndef KDE_H
#define KDE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define KDE_ABI_VERSION 1
#define KDE_MAX_DIM 16          /* d in [1, KDE_MAX_DIM] */
#define KDE_NCCL_ID_BYTES 128   /* sizeof(ncclUniqueId) */
#define KDE_PEER_HANDLE_BYTES 64 /* sizeof(cudaIpcMemHandle_t) */

/* How the ranks of a sharded model exchange their per-box partial sums, shard
 * moments and karma index lists.  NCCL: ncclAllGather.
 * PEER: the library's own all-gather over peer device memory -- every rank
 * stores its payload straight into every peer's exchange window (NVLink /
 * NVSwitch, CUDA IPC mappings) and release-stores an epoch flag; consumers
 * acquire the flags (bounded wait) and combine in rank order. */
typedef enum {
    KDE_COMM_NONE = 0,
    KDE_COMM_NCCL = 1,
    KDE_COMM_PEER = 2
} kde_comm;

typedef struct kde_model kde_model;

typedef enum {
    KDE_OK = 0,
    KDE_EINVAL = 1,   /* invalid argument; model unchanged                    */
    KDE_ENOMEM = 2,   /* device or pinned host allocation failed              */
    KDE_ECUDA = 3,    /* CUDA runtime error (model poisoned)                  */
    KDE_ENCCL = 4,    /* NCCL error (model poisoned)                          */
    KDE_ESTATE = 5,   /* model poisoned by an earlier failure, or bad state   */
    KDE_ETRUNC = 6    /* output truncated (more results than capacity)        */
} kde_status;

/* Loss functions of Appendix C.1, argument order L(p_hat, p).
 * lambda is the smoothing constant of footnote 6; it must be > 0 for
 * RELATIVE, SQUARED_RELATIVE and SQUARED_Q.  SQUARED_RELATIVE uses the true
 * derivative of the printed loss, 2(p_hat-p)/(lambda+p)^2 (R7). */
typedef enum {
    KDE_LOSS_SQUARED = 0,
    KDE_LOSS_ABSOLUTE = 1,
    KDE_LOSS_RELATIVE = 2,
    KDE_LOSS_SQUARED_RELATIVE = 3,
    KDE_LOSS_SQUARED_Q = 4
} kde_loss;

/* Kernel function.  GAUSSIAN is the paper's kernel (eq. 9) and the
 * default.  EPANECHNIKOV ("a truncated second-degree polynomial"; the
 * paper derives nothing for it): the 1-D density 3/(4h) (1 - (x/h)^2) on
 * |x| <= h, i.e. h is the support half-width (reading R14); box
 * masses, gradients and the eq. (20) threshold are its exact counterparts.
 * Its variance is h^2/5, so h_epan = sqrt(5) h_gauss matches a Gaussian
 * bandwidth. */
typedef enum {
    KDE_KERNEL_GAUSSIAN = 0,
    KDE_KERNEL_EPANECHNIKOV = 1
} kde_kernel;

/* Karma-based sample maintenance, Section 4.2 and P:L250.
 *   loss, lambda : the loss L of eq. (7)
 *   k_max        : saturation constant of eq. (8); the paper uses 4
 *   k_init       : karma given to a (re)placed point (reading R8: 0)
 *   threshold    : a point is flagged when K_i < threshold after the update
 *                  ("a given threshold"; no value in the paper)
 *   empty_region : 1 = also flag points with p^(i) >= thr_20 when the true
 *                  selectivity is exactly 0 (eq. 20, Appendix E)   */
typedef struct {
    int32_t loss;
    int32_t empty_region;
    double lambda;
    double k_max;
    double k_init;
    double threshold;
} kde_karma_params;

/* Adaptive bandwidth (Section 4.1; Listing 1 reconstructed, see
 * DESIGN.md R6).  Defaults: minibatch 10, alpha 0.9,
 * lr_min 1e-6, lr_max 50, lr_inc 1.2, lr_dec 0.5.  lr0 is unspecified in the
 * paper (reading: 0.1).  log_bandwidth selects eq. (18) updates. */
typedef struct {
    int32_t minibatch;
    int32_t log_bandwidth;
    int32_t loss;
    int32_t _pad;
    double lambda;
    double alpha;
    double lr_min;
    double lr_max;
    double lr_inc;
    double lr_dec;
    double lr0;
} kde_online_params;

/* ---------------------------------------------------------------- misc */
int32_t     kde_abi_version(void);
const char *kde_last_error(void);                 /* thread-local, never NULL */
const char *kde_status_string(kde_status s);

/* ---------------------------------------------------------------- model */
/* kde_create -- build a model on the current CUDA device.
 *   sample : host, row-major n x d fp32 (copied).  Finite values only.
 *   n      : number of sample points s, n >= 2 (eq. 6 divides by s-1).
 *   d      : dimensionality, 1 <= d <= KDE_MAX_DIM.
 *   h      : host, d bandwidths, each finite in [1e-30, 1e30]; or NULL for
 *            Scott's rule, eq. (3) with population sigma,
 *            computed on the device in fp64.
 *   out    : receives the model handle (set only on KDE_OK).
 * Errors: KDE_EINVAL (arguments, non-finite sample), KDE_ENOMEM, KDE_ECUDA. */
kde_status kde_create(const float *sample, int64_t n, int32_t d, const double *h, kde_model **out);

/* kde_create_sharded -- collective over `world` processes, one GPU each.
 * This rank holds global rows [row_offset, row_offset + n_local) of a sample
 * of n_global rows.  nccl_id: KDE_NCCL_ID_BYTES bytes from
 * kde_get_unique_id() on rank 0, broadcast by the caller.  h == NULL runs
 * Scott's rule over the GLOBAL sample (per-rank moments merged in rank order).
 * world == 1 is valid and equivalent to kde_create.
 * Errors: as kde_create, plus KDE_ENCCL. */
kde_status kde_create_sharded(const float *local_rows, int64_t n_local, int64_t row_offset,
                              int64_t n_global, int32_t d, const double *h,
                              const void *nccl_id, int32_t rank, int32_t world, kde_model **out);

/* kde_create_sharded_peer -- as kde_create_sharded, with the peer-memory
 * exchange (KDE_COMM_PEER) instead of NCCL.  Two-phase: after this call every
 * rank exports its window with kde_peer_handle, the caller all-gathers the
 * world x KDE_PEER_HANDLE_BYTES handle bytes (any host transport) and every
 * rank calls kde_peer_attach; until then every other call returns KDE_ESTATE.
 * With h == NULL, Scott's rule over the global sample runs inside
 * kde_peer_attach.  One process per rank; ranks may share a GPU (tests).
 * Exchange waits are bounded (KDE_PEER_TIMEOUT_S, default 60 s): a rank that
 * misses a collective call makes the others fail with KDE_ECUDA, never hang.
 * Env KDE_PEER_SLOT_MB (default 4): window slot size; larger payloads are
 * exchanged in slot-sized pieces.  Errors: as kde_create. */
kde_status kde_create_sharded_peer(const float *local_rows, int64_t n_local, int64_t row_offset,
                                   int64_t n_global, int32_t d, const double *h, int32_t rank,
                                   int32_t world, kde_model **out);
/* kde_peer_handle -- this rank's exchange-window handle (KDE_PEER_HANDLE_BYTES). */
kde_status kde_peer_handle(kde_model *m, void *handle_out);
/* kde_peer_attach -- collective: map every rank's window (handles: world x
 * KDE_PEER_HANDLE_BYTES in rank order, host); runs the pending Scott's rule.
 * Errors: KDE_ECUDA (mapping failed), KDE_ESTATE (already attached). */
kde_status kde_peer_attach(kde_model *m, const void *handles);

/* kde_get_unique_id -- writes an ncclUniqueId (KDE_NCCL_ID_BYTES bytes). */
kde_status kde_get_unique_id(void *nccl_id_out);

/* kde_destroy -- frees all device and host resources; NULL is a no-op. */
void kde_destroy(kde_model *m);

/* kde_get_info -- any output pointer may be NULL. */
kde_status kde_get_info(const kde_model *m, int64_t *n_local, int64_t *n_global, int32_t *d,
                        int32_t *rank, int32_t *world);

/* kde_get_bandwidth / kde_set_bandwidth -- host fp64 h[d].  set validates
 * every h_j finite in [1e-30, 1e30]; it invalidates retained contributions. */
kde_status kde_get_bandwidth(kde_model *m, double *h);
kde_status kde_set_bandwidth(kde_model *m, const double *h);

/* kde_set_kernel / kde_get_kernel -- select the kernel function (kde_kernel);
 * h is kept, the per-dimension constants are re-derived on the device.
 * Invalidates retained contributions.  Errors: KDE_EINVAL (unknown kernel). */
kde_status kde_set_kernel(kde_model *m, int32_t kernel);
kde_status kde_get_kernel(const kde_model *m, int32_t *kernel);

/* kde_set_retain -- on != 0: single-query scans (q == 1) also store the
 * per-point contributions p^(i) (fp32, 4 B/point) for a following
 * kde_karma_update on the same box ("we do not discard the temporary
 * buffer").  Default off. */
kde_status kde_set_retain(kde_model *m, int32_t on);

/* kde_set_cull / kde_get_cull -- on != 0 (the default): the scans skip every
 * (point, box) pair whose product of eq. (13) factors is provably below 2^-64.
 * With o_j the distance of the point OUTSIDE the box in dimension j in units of
 * sqrt2 h_j / sqrt(log2 e), D_j <= 1/2 erfc(z_j) <= 2^{-o_j^2}, so sum_j o_j^2 >= 64
 * bounds its contribution to p_hat by 2^-64 and to each dp_hat/dh_j by
 * 2^-60 / (sqrt(pi) sqrt(log2 e) h_j) (R15).  Which scans cull: the
 * single-box scan (q == 1) always; the batched scan (q > 1) for batches that
 * fill 256-box CTAs (smaller batches measured no faster culled).  For the
 * Epanechnikov kernel a point outside the support in some dimension is skipped
 * (its contribution is exactly 0).  A skipped point's retained p^(i) is 0.
 * Points inside the box are never skipped.  on == 0: every pair is evaluated.
 * Errors: none (KDE_EINVAL for a NULL model). */
kde_status kde_set_cull(kde_model *m, int32_t on);
kde_status kde_get_cull(const kde_model *m, int32_t *on);

/* kde_set_cells / kde_get_cells -- on != 0 (the default): the culled batched
 * scan (q > 1, culling on, batches that fill 256-box CTAs) visits a spatially
 * ordered COPY of the local sample instead of the sample itself (R17):
 * points sorted by a 32-bit Morton key over the column range, cut into cells of
 * 256 points with their bounding boxes.  A (box, cell) pair whose bounding box
 * lies >= 8 scaled bandwidths outside the box is skipped as a whole (every point
 * in it obeys the R15 bound above); a cell inside the box's kept region is
 * evaluated without per-point classification.  The estimator is a sum over an
 * unordered set (eq. 2), so only the summation order changes; results
 * stay deterministic.  The copy (d x ld fp32, device) and its cell boxes are
 * built on the model's stream at the first such call and rebuilt after any call
 * that changes sample rows (replace / insert / streaming step); the sample, its
 * karma and retained contributions keep their original order.  When the device
 * memory for the copy (d x ld fp32 + 16 B/point of build scratch) cannot be
 * allocated, the call scans the sample itself and the setting turns off.
 * builds: number of index builds so far (may be NULL).
 * stats: NULL or 4 int64 -- while profiling is on (kde_set_profiling), the cells
 * scans' (box, cell) items, items evaluated without classification, points
 * evaluated (point x box pairs that reached eq. 13) and points classified, summed
 * since the previous read or kde_set_profiling call (reading resets them; zeros
 * when profiling is off).  Synchronises the model's stream when stats != NULL.
 * Errors: KDE_EINVAL for a NULL model / on; KDE_ECUDA. */
kde_status kde_set_cells(kde_model *m, int32_t on);
kde_status kde_get_cells(kde_model *m, int32_t *on, int64_t *builds, int64_t *stats);

/* ---------------------------------------------------------------- hot path */
/* kde_estimate_batch -- selectivity estimates for q boxes, eq. (2)+(13):
 *   est[k]        = p_hat_H(Omega_k) = (1/s) sum_i prod_j [Phi((u_kj - t_ij)/h_j) - Phi((l_kj - t_ij)/h_j)]
 *   dest_dh[k*d+j] = d p_hat(Omega_k) / d h_j, eq. (17); NULL = skip.
 * lo, hi: host row-major q x d fp32.  est: host q fp64.  dest_dh: host q*d fp64.
 * q == 0 is a no-op.  Per-point arithmetic is fp32, all sums fp64,
 * deterministic (fixed reduction order for a given device and world size). */
kde_status kde_estimate_batch(kde_model *m, const float *lo, const float *hi, int64_t q,
                              double *est, double *dest_dh);
kde_status kde_estimate_batch_dev(kde_model *m, const float *d_lo, const float *d_hi, int64_t q,
                                  double *d_est, double *d_dest_dh, void *stream);

/* kde_loss_and_grad -- batch objective of eq. (5) and its gradient (eq. 14):
 *   loss    = (1/q) sum_k L(p_hat_k, p_k)
 *   grad[j] = (1/q) sum_k L'(p_hat_k, p_k) * d p_hat_k / d h_j
 *             (times h_j when log_bandwidth != 0, eq. 18)
 * true_sel: host q fp64 in [0, 1].  loss_out: 1 fp64.  grad_out: d fp64.
 * est_out: q fp64 or NULL.  q >= 1.
 * Errors: KDE_EINVAL (bounds, true_sel, loss kind, lambda <= 0 where needed). */
kde_status kde_loss_and_grad(kde_model *m, const float *lo, const float *hi, const double *true_sel,
                             int64_t q, int32_t loss, double lambda, int32_t log_bandwidth,
                             double *loss_out, double *grad_out, double *est_out);
kde_status kde_loss_and_grad_dev(kde_model *m, const float *d_lo, const float *d_hi,
                                 const double *d_true_sel, int64_t q, int32_t loss, double lambda,
                                 int32_t log_bandwidth, double *d_loss, double *d_grad, double *d_est,
                                 void *stream);

/* kde_karma_update -- one query's feedback (true selectivity p) for sample
 * maintenance: for every point, eq. (6) leave-one-out estimate,
 * eq. (7) karma delta, eq. (8) saturating update of K_i, then flag K_i <
 * threshold, or (empty_region && p == 0 && p^(i) >= thr_20 of eq. 20).
 * Reuses the retained contributions when the previous single-query scan was
 * on the same box with unchanged h and sample; otherwise rescans (same
 * result).  idx_out receives the ascending GLOBAL indices of flagged points
 * (at most idx_cap of them); *n_flagged = total flagged.  Returns
 * KDE_ETRUNC (karma still updated) when total > idx_cap.  lo/hi: host d fp32. */
kde_status kde_karma_update(kde_model *m, const float *lo, const float *hi, double true_sel,
                            const kde_karma_params *kp, int64_t *idx_out, int64_t idx_cap,
                            int64_t *n_flagged);

/* kde_online_update -- adaptive bandwidth step (Section 4.1, Fig. 3 steps
 * 5-8): L'(p_hat, p) * d p_hat/d h (x h in log mode) is added to the
 * mini-batch; when `minibatch` gradients are collected the RMSprop/Rprop step
 * of Listing 1 (reconstructed, R6) updates h ON THE DEVICE.  Uses
 * the retained estimate+gradient of a preceding kde_estimate_batch(q == 1,
 * dest_dh != NULL) on the same box, else rescans.  *updated = 1 when h
 * changed (may be NULL).  lo/hi: host d fp32. */
kde_status kde_online_update(kde_model *m, const float *lo, const float *hi, double true_sel,
                             const kde_online_params *op, int32_t *updated);

/* kde_replace_points -- write k rows (host row-major k x d fp32) to the GLOBAL
 * indices idx[k] (unique, in [0, n_global)), reset their karma to k_init
 * (P:L248 reservoir inserts, P:L250 karma replacement).  Invalidates retained
 * contributions.  Errors: KDE_EINVAL on duplicates, range, non-finite rows. */
kde_status kde_replace_points(kde_model *m, const int64_t *idx, const float *rows, int64_t k,
                              double k_init);

/* kde_reservoir_select -- the host's reservoir sampling decision for an
 * insert-only workload (Section 4.2, P:L189 / P:L248: "reservoir sampling [43]
 * adds newly inserted data to the sample with probability |S|/|R|, replacing a
 * random point ... all decisions are made independently by the host").
 * Algorithm R: arrival a = n_seen + r + 1 (1-based; arrivals 1..n_sample fill
 * slots 0..n_sample-1) draws j uniform on [0, a) from a counter-based generator
 *   z = SplitMix64 finaliser of (seed + a * 0x9E3779B97F4A7C15), j = floor(z a / 2^64),
 * and takes slot j iff j < n_sample.  slot_out[r] = that slot or -1 (host,
 * k int64, caller-owned).  Pure host code (no device, no model).
 * Errors: KDE_EINVAL (n_sample < 1, n_seen < 0, k < 0, NULL slot_out). */
kde_status kde_reservoir_select(uint64_t seed, int64_t n_sample, int64_t n_seen, int64_t k, int64_t *slot_out);

/* kde_insert_rows -- insert-only maintenance of the sample: the k
 * arriving rows (host row-major k x d fp32, copied) go through
 * kde_reservoir_select(seed, n_global, *n_seen, k); ONLY the rows that enter
 * the sample are transferred to the device and written (kde_replace_points
 * semantics: karma reset to k_init, retained state invalidated).  When several
 * arrivals of the chunk draw the same slot, the last one wins (the sequential
 * result).  *n_seen (in/out): arrivals so far -- the sample itself counts as
 * the first n_global (or more) -- advanced by k.  *n_written (optional): slots
 * of this shard written.  Sharded models: every rank calls with the same rows
 * and seed; each writes the slots of its shard.  Host cost O(k) (a per-shard
 * last-writer table resolves repeated slots).  Errors: KDE_EINVAL (non-finite rows, bad
 * n_seen); state unchanged. */
kde_status kde_insert_rows(kde_model *m, const float *rows, int64_t k, uint64_t seed, int64_t *n_seen,
                           double k_init, int64_t *n_written);

/* kde_insert_rows_async -- kde_insert_rows whose device work (the H2D copy of the
 * accepted rows, the column-range update and the scatter) is enqueued on `stream`
 * (NULL: the model's stream) without waiting for it: the host decides the next
 * chunk while the device still runs the previous queries (the host makes
 * the reservoir decisions, only accepted rows cross PCIe).  The rows are copied
 * into one of two pinned staging buffers before the call returns (the caller may
 * reuse `rows`); a call waits only for the copy out of the buffer it reuses (two
 * calls back).  Later work on `stream` sees the new rows in stream order; other
 * calls of the library order themselves after it as after any _dev call.  Use one
 * stream for a model's async inserts.  Single-GPU (world == 1).
 * Errors: as kde_insert_rows; KDE_EINVAL for world > 1. */
kde_status kde_insert_rows_async(kde_model *m, const float *rows, int64_t k, uint64_t seed, int64_t *n_seen,
                                 double k_init, int64_t *n_written, void *stream);

/* ---------------------------------------------------------------- device-resident feedback loop
 * Single-GPU (world == 1) device-pointer variants of the feedback calls, so a
 * whole streaming step (estimate -> karma -> bandwidth -> replacement) runs
 * without a host round trip (the paper ships the bitmap to the
 * host).  They enqueue on `stream` (NULL = the model's stream) and use
 * the retained state of the preceding kde_estimate_batch_dev(q == 1) on the
 * same stream: p_hat and dp_hat/dh always, the contributions p^(i) only when
 * retain is on (kde_set_retain).  Arguments are NOT validated on the device:
 * the caller guarantees a valid box, 0 <= p <= 1, and (replace) unique
 * in-range indices -- the karma output satisfies this by construction. */
/* karma pass: d_true_sel 1 fp64; ascending GLOBAL flagged indices -> d_idx_out
 * (first idx_cap), total count -> *d_n_flagged (device int64). */
kde_status kde_karma_update_dev(kde_model *m, const float *d_lo, const float *d_hi, const double *d_true_sel,
                                const kde_karma_params *kp, int64_t *d_idx_out, int64_t idx_cap,
                                int64_t *d_n_flagged, void *stream);
/* Listing 1 step from the retained (p_hat, dp_hat/dh); requires the preceding
 * single-box estimate to have computed the gradient. */
kde_status kde_online_update_dev(kde_model *m, const double *d_true_sel, const kde_online_params *op, void *stream);
/* the first min(*d_k, cap) GLOBAL indices d_idx[] receive rows d_rows[] (device,
 * row-major, at least cap x d), karma reset to k_init; the column ranges used
 * for bound clamping are widened on the device. */
kde_status kde_replace_points_dev(kde_model *m, const int64_t *d_idx, const float *d_rows, const int64_t *d_k,
                                  int64_t cap, double k_init, void *stream);

/* One whole streaming step in three kernels (device pointers, single GPU):
 * single-box estimate (eq. 2/13) -> d_est[1]; gradient (eq. 17) -> d_dpdh[d]
 * when op != NULL; karma pass (eq. 6-8, 20) with retained contributions;
 * ordered compaction of the flagged GLOBAL indices -> d_idx_out (first
 * idx_cap), count -> *d_n_flagged; then, in the compaction's last block, the
 * Listing 1 step (op != NULL) and the replacement of the first
 * min(count, idx_cap) flagged points by d_rows (row-major, idx_cap x d;
 * NULL = no replacement), karma reset to k_init.  Equivalent to
 * kde_estimate_batch_dev + kde_karma_update_dev + kde_online_update_dev +
 * kde_replace_points_dev with the same arguments (retain is implied). */
kde_status kde_stream_step_dev(kde_model *m, const float *d_lo, const float *d_hi, const double *d_true_sel,
                               const kde_karma_params *kp, const kde_online_params *op, int64_t *d_idx_out,
                               int64_t idx_cap, int64_t *d_n_flagged, const float *d_rows, double k_init,
                               double *d_est, double *d_dpdh, void *stream);

/* ---------------------------------------------------------------- inspection */
kde_status kde_get_karma(kde_model *m, double *karma);   /* local n fp64          */
kde_status kde_set_karma(kde_model *m, const double *karma); /* local n fp64      */
kde_status kde_get_sample(kde_model *m, float *rows);    /* local n x d row-major */
/* last retained per-point contributions (local n fp32); KDE_ESTATE if none. */
kde_status kde_get_contributions(kde_model *m, float *c);
/* online (Listing 1) state, each d fp64 (any may be NULL), and batch count. */
kde_status kde_get_online_state(kde_model *m, double *acc, double *ms, double *lr, double *gprev,
                                int32_t *count);
kde_status kde_set_online_state(kde_model *m, const double *acc, const double *ms, const double *lr,
                                const double *gprev, int32_t count);
/* wait for all work enqueued on the model's stream. */
kde_status kde_synchronize(kde_model *m);

/* kde_set_profiling -- on != 0: record CUDA events around every scan kernel
 * launch (on the stream it is launched on) and count every kernel launch.
 * Resets the counters.  kde_get_profile synchronises the device and returns
 * the summed scan-kernel time (ms), the number of scan launches and of all
 * kernel launches since the last reset, then resets them. */
kde_status kde_set_profiling(kde_model *m, int32_t on);
kde_status kde_get_profile(kde_model *m, double *scan_ms, int64_t *scan_launches, int64_t *launches);

/* ---------------------------------------------------------------- harness */
/* kde_count_in_box_dev -- NOT part of the estimator: the exact feedback the
 * DBMS would return.  counts[k] = |{ r : l_kj < R_rj < u_kj  for all j }|
 * over a device row-major R[n][d] fp32.  All pointers are device pointers. */
kde_status kde_count_in_box_dev(const float *d_rows, int64_t n, int32_t d, const float *d_lo,
                                const float *d_hi, int64_t q, int64_t *d_counts, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* KDE_H */
