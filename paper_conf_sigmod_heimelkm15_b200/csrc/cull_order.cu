// cull_order.cu -- box order for the culled batched scan (reading R15).
//
// The batched scan gives each CTA 256 boxes and each warp 32 of them; with
// culling a warp costs as much as its box with the most kept points.  Boxes
// are therefore ordered by their kept count on a probe of the sample's first
// kProbe points (the sample is an unordered set, so its prefix is a uniform
// probe), boxes with a narrow dimension (general Phi path) last, with a
// stable radix sort: CTAs and warps get boxes of similar cost.  The order is
// a schedule only -- every box's partial is still the same fixed-order sum.
#include <cub/cub.cuh>

#include "common.cuh"
#include "kernels.cuh"
#include "phi.cuh"

namespace kde {

constexpr int kProbe = 1024;

// one warp per box: the lanes split the probe points, the count is a warp sum
__global__ void cull_probe_kernel(const float* __restrict__ cols, int64_t ld, int nprobe, int d,
                                  const float* __restrict__ lo, const float* __restrict__ hi, int64_t q,
                                  const DevConsts* __restrict__ c, unsigned* __restrict__ keys, int* __restrict__ idx) {
  const int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (i >= q) return;  // warp-uniform
  float2 cb[kMaxDim];
  float ap[kMaxDim];
  bool nar = false;
  for (int j = 0; j < d; ++j) {
    ap[j] = c->ap[j];
    const float l = lo[i * d + j], u = hi[i * d + j];
    cb[j] = make_cullbox(l, u, ap[j], c->renc[2 * j], c->renc[2 * j + 1]);
    const float dy = (u - l) * ap[j];
    nar |= dy > 0.0f && dy < kNarrowY;
  }
  const bool epan = c->kernel == kEpanechnikov;  // cull_score: max_j o_j < 1 instead of sum_j o_j^2 < kCullY2
  if (epan) nar = false;
  unsigned cnt = 0;
  for (int p = lane; p < nprobe; p += 32) {
    float o2 = 0.0f;
    for (int j = 0; j < d; ++j) {
      const float y = fmaf(__ldg(cols + (int64_t)j * ld + p), ap[j], -cb[j].x);
      const float e = fabsf(y) - cb[j].y;
      o2 = epan ? fmaxf(o2, e) : fmaf(e + fabsf(e), e + fabsf(e), o2);  // as cull_score (phi.cuh)
    }
    cnt += o2 < (epan ? cull_limit<true>() : cull_limit<false>()) ? 1u : 0u;
  }
  for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
  if (lane == 0) {
    keys[i] = (nar ? (1u << 12) : 0u) + cnt;
    idx[i] = (int)i;
  }
}

// scratch layout: keys_in [q] u32, keys_out [q] u32, idx_in [q] i32, perm [q] i32, cub temp
size_t cull_order_bytes(int64_t q) {
  size_t temp = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, temp, (const unsigned*)nullptr, (unsigned*)nullptr, (const int*)nullptr,
                                  (int*)nullptr, (int)q, 0, 13);
  return 16 * (size_t)q + temp + 256;
}

cudaError_t launch_cull_order(const float* cols, int64_t ld, int64_t n, int d, const float* lo, const float* hi,
                              int64_t q, const DevConsts* c, void* scratch, size_t scratch_bytes, int** perm_out,
                              cudaStream_t s) {
  unsigned* kin = reinterpret_cast<unsigned*>(scratch);
  unsigned* kout = kin + q;
  int* iin = reinterpret_cast<int*>(kout + q);
  int* perm = iin + q;
  void* temp = reinterpret_cast<void*>(((uintptr_t)(perm + q) + 255) & ~(uintptr_t)255);
  size_t temp_bytes = scratch_bytes - ((char*)temp - (char*)scratch);
  const int nprobe = (int)(n < kProbe ? n : kProbe);
  cull_probe_kernel<<<(unsigned)((q * 32 + 255) / 256), 256, 0, s>>>(cols, ld, nprobe, d, lo, hi, q, c, kin, iin);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  e = cub::DeviceRadixSort::SortPairs(temp, temp_bytes, kin, kout, iin, perm, (int)q, 0, 13, s);
  if (e != cudaSuccess) return e;
  *perm_out = perm;
  return cudaGetLastError();
}

}  // namespace kde
