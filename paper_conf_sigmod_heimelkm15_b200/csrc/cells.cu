// cells.cu -- spatial index of the sample for the culled batched scan (reading R17).
//
// The sample is an unordered set (the estimator is a sum over its points), so the batched
// scan may visit it in any order.  For large batches it visits an ordered COPY: points sorted by a
// Morton key of their coordinates (quantised over the column range), cut into cells of kCellPts
// consecutive points, each with the bounding box of its points.  A box then skips the cells whose
// bounding box lies >= 8 bandwidths outside it (every point of such a cell satisfies the R15 bound)
// and evaluates every point of a cell that lies well inside its kept region without classifying
// them (scan_cells.cuh).  The copy is rebuilt whenever the sample changes (kde_api.cu: sgen); the
// sample itself, the retained contributions and karma keep their original order.
#include <cub/cub.cuh>

#include "common.cuh"

namespace kde {

// bits per dimension of the 32-bit Morton key (d * B <= 32; at most 24 so that the fp32
// quantisation below is exact in the integer it produces)
__host__ __device__ inline int morton_bits(int d) {
  const int b = 32 / d;
  return b > 24 ? 24 : b;
}

__global__ void cells_key_kernel(const float* __restrict__ cols, int64_t ld, int64_t n, int d,
                                 const DevConsts* __restrict__ c, unsigned* __restrict__ key,
                                 int* __restrict__ idx) {
  const int B = morton_bits(d);
  const float qmax = (float)((1u << B) - 1u);
  float lo[kMaxDim], sc[kMaxDim];
  for (int j = 0; j < d; ++j) {
    const float a = fdec_range(c->renc[2 * j]), b = fdec_range(c->renc[2 * j + 1]);
    const float w = b - a;
    lo[j] = a;
    sc[j] = (w > 0.0f && w < 3.0e38f) ? qmax / w : 0.0f;
  }
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    unsigned qv[kMaxDim];
    for (int j = 0; j < d; ++j) {
      const float v = (__ldg(cols + (int64_t)j * ld + i) - lo[j]) * sc[j];
      qv[j] = (unsigned)fminf(fmaxf(v, 0.0f), qmax);  // NaN-free: the sample is validated at creation
    }
    unsigned k = 0u;
    for (int b = B - 1; b >= 0; --b)
      for (int j = 0; j < d; ++j) k = (k << 1) | ((qv[j] >> b) & 1u);
    key[i] = k;
    idx[i] = (int)i;
  }
}

// ordered copy: ccols[j][p] = cols[j][perm[p]] for p < n, 0 for the padding of the last cell
__global__ void cells_gather_kernel(const float* __restrict__ cols, int64_t ld, int64_t n, int64_t npad, int d,
                                    const int* __restrict__ perm, float* __restrict__ ccols) {
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < npad; p += (int64_t)gridDim.x * blockDim.x) {
    const int src = p < n ? perm[p] : 0;
    for (int j = 0; j < d; ++j) ccols[(int64_t)j * ld + p] = p < n ? __ldg(cols + (int64_t)j * ld + src) : 0.0f;
  }
}

// one warp per cell: (min, max) per dimension over the cell's valid points
__global__ void cells_bbox_kernel(const float* __restrict__ ccols, int64_t ld, int64_t n, int64_t ncells, int d,
                                  float* __restrict__ cbb) {
  const int64_t cell = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (cell >= ncells) return;  // warp-uniform
  const int64_t p0 = cell * kCellPts;
  const int npts = (int)(n - p0 < kCellPts ? n - p0 : kCellPts);
  for (int j = 0; j < d; ++j) {
    float mn = INFINITY, mx = -INFINITY;
    for (int i = lane; i < npts; i += 32) {
      const float v = ccols[(int64_t)j * ld + p0 + i];
      mn = fminf(mn, v);
      mx = fmaxf(mx, v);
    }
    for (int o = 16; o > 0; o >>= 1) {
      mn = fminf(mn, __shfl_xor_sync(0xffffffffu, mn, o));
      mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    if (lane == 0) {
      cbb[(cell * d + j) * 2] = mn;
      cbb[(cell * d + j) * 2 + 1] = mx;
    }
  }
}

// scratch: keys in/out (u32), idx in/out (i32), cub temp
size_t cells_scratch_bytes(int64_t n) {
  size_t temp = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, temp, (const unsigned*)nullptr, (unsigned*)nullptr, (const int*)nullptr,
                                  (int*)nullptr, (int)n, 0, 32);
  return 16 * (size_t)n + temp + 1024;
}

cudaError_t launch_cells_build(const float* cols, int64_t ld, int64_t n, int d, const DevConsts* c, void* scratch,
                               size_t scratch_bytes, float* ccols, float* cbb, cudaStream_t s) {
  if (n <= 0) return cudaSuccess;
  if (n > (int64_t)INT32_MAX) return cudaErrorInvalidValue;
  unsigned* kin = reinterpret_cast<unsigned*>(scratch);
  unsigned* kout = kin + n;
  int* iin = reinterpret_cast<int*>(kout + n);
  int* iout = iin + n;
  void* temp = reinterpret_cast<void*>(((uintptr_t)(iout + n) + 255) & ~(uintptr_t)255);
  const size_t used = (size_t)((char*)temp - (char*)scratch);
  if (used > scratch_bytes) return cudaErrorInvalidValue;
  size_t temp_bytes = scratch_bytes - used;
  const int64_t ncells = (n + kCellPts - 1) / kCellPts;
  const int64_t npad = ncells * kCellPts;
  const unsigned g = (unsigned)((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096);
  cells_key_kernel<<<g, 256, 0, s>>>(cols, ld, n, d, c, kin, iin);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  e = cub::DeviceRadixSort::SortPairs(temp, temp_bytes, kin, kout, iin, iout, (int)n, 0, d * morton_bits(d), s);
  if (e != cudaSuccess) return e;
  const unsigned gg = (unsigned)((npad + 255) / 256 < 4096 ? (npad + 255) / 256 : 4096);
  cells_gather_kernel<<<gg, 256, 0, s>>>(cols, ld, n, npad, d, iout, ccols);
  e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  cells_bbox_kernel<<<(unsigned)((ncells * 32 + 255) / 256), 256, 0, s>>>(ccols, ld, n, ncells, d, cbb);
  return cudaGetLastError();
}

}  // namespace kde
