// kernels.cuh -- launchers for the non-scan kernels (kernels.cu).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "common.cuh"

namespace kde {

constexpr int kKarmaThreads = 256;
#ifndef KDE_TUNE_KARMA_PTS
#define KDE_TUNE_KARMA_PTS 4096
#endif
constexpr int kKarmaPts = KDE_TUNE_KARMA_PTS;  // contiguous points per karma block (4096: 16 passes, 2 load batches)
inline int karma_blocks(int64_t n) { return (int)((n + kKarmaPts - 1) / kKarmaPts); }

struct HVec {
  double v[kMaxDim];
};

// optional work done by the last block of the karma compaction (device-resident streaming step)
struct StreamTail {
  int online = 0;  // run the Listing 1 step
  const double* ret = nullptr;
  const double* p = nullptr;
  OnlineParamsDev op{};
  OnlineState* st = nullptr;
  DevConsts* c = nullptr;
  int d = 0;
  const float* rows = nullptr;  // non-null: replace the flagged points by rows[0..]
  float* cols = nullptr;
  int64_t ld = 0;
  double* karma = nullptr;
  double k_init = 0.0;
};

cudaError_t launch_rows_to_cols(const float* rows, int64_t n, int d, float* cols, int64_t ld, int* bad,
                                cudaStream_t s);
cudaError_t launch_cols_to_rows(const float* cols, int64_t ld, int64_t n, int d, float* rows, cudaStream_t s);
// per-column [min, max] of the local sample into DevConsts (enc: device [d][2] uint, init 0xFFFFFFFF / 0)
cudaError_t launch_col_range(const float* cols, int64_t ld, int64_t n, int d, unsigned* enc, DevConsts* c,
                             cudaStream_t s);
cudaError_t launch_row_range(const float* rows, int64_t k, int d, unsigned* enc, DevConsts* c, cudaStream_t s);
cudaError_t launch_scatter_rows_dev(const int64_t* idx_global, const float* rows, const int64_t* d_k, int64_t cap, int d,
                                    float* cols, int64_t ld, int64_t n, int64_t row_offset, double* karma, double k_init,
                                    unsigned* enc, DevConsts* c, cudaStream_t s);
cudaError_t launch_scatter_rows(const int64_t* idx_local, const float* rows, int64_t k, int d, float* cols,
                                int64_t ld, double* karma, double k_init, cudaStream_t s);
int moments_blocks(int64_t n);
cudaError_t launch_moments(const float* cols, int64_t ld, int64_t n, int d, double* part, double* mom,
                           cudaStream_t s);
cudaError_t launch_moments_merge_ranks(const double* g, int world, int d, double* mom, cudaStream_t s);
cudaError_t launch_scott(const double* mom, int d, DevConsts* c, int* bad, cudaStream_t s);
cudaError_t launch_set_consts(const double* h, int d, DevConsts* c, cudaStream_t s);
cudaError_t launch_set_kernel_type(int kernel, int d, DevConsts* c, cudaStream_t s);
// cull_order.cu: box order for the culled batched scan (probe counts + stable radix sort)
size_t cull_order_bytes(int64_t q);
cudaError_t launch_cull_order(const float* cols, int64_t ld, int64_t n, int d, const float* lo, const float* hi,
                              int64_t q, const DevConsts* c, void* scratch, size_t scratch_bytes, int** perm_out,
                              cudaStream_t s);
// sums (or, with peer != NULL, slot [epoch parity][rank] of EVERY rank's exchange window: the fused
// exchange) <- the fixed-order sum over splits
cudaError_t launch_reduce_splits(const double* partials, int splits, int64_t q, int na, double* sums,
                                 const PeerArgs* peer, cudaStream_t s);
// the cells scan's partials (row entry g * QG + slot, see scan_cells.cuh) -> sums[box][na], split order
cudaError_t launch_reduce_splits_mapped(const double* partials, int splits, int64_t qpad, int64_t q, int na, int qg,
                                        int ngroups, const int* perm, double* sums, const PeerArgs* peer,
                                        cudaStream_t s);
cudaError_t launch_combine_ranks(const double* gathered, int world, int64_t q, int na, double* sums,
                                 cudaStream_t s);
cudaError_t launch_finalize(const double* sums, int64_t q, int d, int na, const DevConsts* c, double n_global,
                            double* est, double* dpdh, cudaStream_t s);
cudaError_t launch_loss_epilogue(const double* est, const double* dpdh, const double* true_sel, int64_t q, int d,
                                 int kind, double lambda, int log_bw, const DevConsts* c, double* loss_out,
                                 double* grad_out, cudaStream_t s);
int karma_launches();  // kernels one launch_karma enqueues
// karma pass + ordered compaction: block_counts int32 [nb], block_offsets int64 [nb + 1],
// done: 2 self-resetting counters (compaction, karma); c and karma padded to a multiple of 4 points
cudaError_t launch_karma(const float* cvals, double* karma, int64_t n, double n_global, const double* phat, const double* p,
                         const KarmaParamsDev& kp, const float* lo, const float* hi, int d, const DevConsts* c,
                         uint32_t* bitmap, int32_t* block_counts, int64_t* block_offsets, unsigned* done,
                         int64_t row_offset, int64_t* idx_out, int64_t cap, int64_t* total_out, const StreamTail& tail,
                         cudaStream_t s);
cudaError_t launch_online_update(const double* ret, const double* p, const OnlineParamsDev& op, int d, OnlineState* st,
                                 DevConsts* c, cudaStream_t s);
cudaError_t launch_count_in_box(const float* rows, int64_t n, int d, const float* lo, const float* hi, int64_t q,
                                unsigned long long* counts, int num_sms, cudaStream_t s);

// reservoir.cu: Algorithm R decisions (host), slot or -1 per arrival n_seen+1 .. n_seen+k
void reservoir_slots(uint64_t seed, int64_t n_sample, int64_t n_seen, int64_t k, int64_t* slot_out);

// peer.cu: all-gather over peer device memory (the sharded model's exchange step without NCCL);
// PeerArgs / kPeerFlagBytes live in common.cuh (the scan tails push into peer windows directly)
// dst + r * stride <- rank r's src (bytes <= pa.slot, multiples of 8), for every rank r
cudaError_t launch_peer_allgather(const void* src, void* dst, size_t bytes, size_t stride, const PeerArgs& pa,
                                  int num_sms, cudaStream_t s);
// fused exchange, consumer side: wait for every rank's pushed slot of this epoch (count doubles,
// pushed by the scan tail / reduce_splits), sum the slots in rank order into dst, publish the epoch
cudaError_t launch_peer_combine(double* dst, int64_t count, const PeerArgs& pa, int num_sms, cudaStream_t s);

}  // namespace kde
