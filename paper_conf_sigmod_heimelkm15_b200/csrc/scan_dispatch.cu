// scan_dispatch.cu -- runtime d -> template D dispatch for the scan kernels.
#include "scan.cuh"

namespace kde {

#define KDE_DECL(D)                                                                                    \
  extern template cudaError_t launch_single_t<D>(bool, const ScanSingleArgs&, int, cudaStream_t);      \
  extern template cudaError_t launch_batched_t<D>(bool, const ScanBatchedArgs&, int, int*, cudaStream_t, bool); \
  extern template cudaError_t launch_cells_t<D>(bool, const ScanCellsArgs&, int, int*, cudaStream_t, bool);
KDE_DECL(1) KDE_DECL(2) KDE_DECL(3) KDE_DECL(4) KDE_DECL(5) KDE_DECL(6) KDE_DECL(7) KDE_DECL(8)
KDE_DECL(9) KDE_DECL(10) KDE_DECL(11) KDE_DECL(12) KDE_DECL(13) KDE_DECL(14) KDE_DECL(15) KDE_DECL(16)
#undef KDE_DECL

#define KDE_CASES(X) X(1) X(2) X(3) X(4) X(5) X(6) X(7) X(8) X(9) X(10) X(11) X(12) X(13) X(14) X(15) X(16)

cudaError_t launch_scan_single(int d, bool grad, const ScanSingleArgs& a, int grid, cudaStream_t s) {
  switch (d) {
#define X(D) case D: return launch_single_t<D>(grad, a, grid, s);
    KDE_CASES(X)
#undef X
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_scan_batched(int d, bool grad, const ScanBatchedArgs& a, int num_sms, int* splits_out,
                                cudaStream_t s, bool dry_run) {
  switch (d) {
#define X(D) case D: return launch_batched_t<D>(grad, a, num_sms, splits_out, s, dry_run);
    KDE_CASES(X)
#undef X
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_scan_cells(int d, bool grad, const ScanCellsArgs& a, int num_sms, int* splits_out, cudaStream_t s,
                              bool dry_run) {
  switch (d) {
#define X(D) case D: return launch_cells_t<D>(grad, a, num_sms, splits_out, s, dry_run);
    KDE_CASES(X)
#undef X
  }
  return cudaErrorInvalidValue;
}

int cells_group_boxes(int d) {
  switch (d) {
#define X(D) case D: return cells_qg<D>();
    KDE_CASES(X)
#undef X
  }
  return 0;
}

// the batched scan culls (and wants the probe order) when a CTA holds 256 boxes (one thread per box)
bool batched_culls(int64_t q) { return batched_qb(q) == kBatchedThreads; }

// ~3 resident CTAs of 256 threads per SM, never more CTAs than 8-point work items.
int scan_single_grid(int d, bool grad, int64_t n, int num_sms, bool cull) {
  if (cull) {  // culled TMA variant: one contiguous chunk of >= 1 tile per CTA
    int64_t grid = (int64_t)num_sms * cull_occ(d);
    const int64_t ntiles = (n + cull_tile(d) - 1) / cull_tile(d);
    if (grid > ntiles) grid = ntiles;
    return (int)(grid < 1 ? 1 : grid);
  }
  if (single_uses_tma(d)) {  // one contiguous chunk of >= 1 tile per CTA
    int64_t grid = (int64_t)num_sms * single_tma_occ(d);
    const int64_t ntiles = (n + kSingleTile - 1) / kSingleTile;
    if (grid > ntiles) grid = ntiles;
    return (int)(grid < 1 ? 1 : grid);
  }
  const int per_sm = single_occ(d, grad);
  int64_t grid = (int64_t)num_sms * per_sm;
  const int64_t items = (n + 15) / 16;
  const int64_t need = (items + kSingleThreads - 1) / kSingleThreads;
  if (grid > need) grid = need;
  if (grid < 1) grid = 1;
  return (int)grid;
}

}  // namespace kde
