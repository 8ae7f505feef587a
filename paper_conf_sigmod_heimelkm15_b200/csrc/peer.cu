// peer.cu -- the sharded model's exchange step over peer device memory
// (SURVEY.md §8(e) "fused variant": no separate collective library call; the
// producer's results are stored straight into every peer's HBM over
// NVLink / NVSwitch, followed by a flag barrier).
//
// One process per GPU.  Every rank owns an exchange WINDOW (cudaMalloc'd,
// exported with cudaIpcGetMemHandle, opened by every peer with
// cudaIpcOpenMemHandle), laid out as
//   [kPeerFlagBytes)  flags: uint64 epoch per source rank (128 B apart)
//   [2][world][slot]  data slots, one per (parity, source rank)
// An all-gather of `bytes` per rank (<= slot) with epoch e = *epoch + 1:
//   peer_push_kernel     every block stores its part of `src` into slot
//                        [e & 1][rank] of EVERY rank's window (remote stores);
//                        the last block (arrival counter) fences system-wide
//                        and release-stores flags[rank] = e in every window.
//   peer_collect_kernel  waits (acquire) until flags[r] >= e for every r, copies
//                        the world slots of its own window in rank order into
//                        `dst` ([world][bytes], the layout ncclAllGather gives)
//                        and its last block publishes *epoch = e.
// Consumers (rank-order combine, Chan merge, index gather) are the same kernels
// the NCCL path feeds.  Reuse safety: a rank writes parity e & 1 again only at
// epoch e + 2, i.e. after passing the barrier of e + 1, which every peer enters
// only once its epoch-e collect has finished (stream order).  The wait is bounded
// (%globaltimer): on timeout *err is set and the kernel returns, never hangs.
#include <cstdint>
#include <cuda_runtime.h>

#include "common.cuh"
#include "kernels.cuh"
#include "peer.cuh"

namespace kde {

__device__ __forceinline__ char* slot_ptr(char* win, int parity, int src, int world, size_t slot) {
  return peer_slot(win, parity, src, world, slot);
}

__global__ void peer_push_kernel(const char* __restrict__ src, size_t bytes, PeerArgs pa) {
  __shared__ bool last_s;
  const uint64_t e = *pa.epoch + 1;
  const int parity = (int)(e & 1);
  // 16-byte loads of src (8-byte aligned payloads are read as pairs) and 16-byte stores into the
  // 256-byte aligned slots
  const size_t nvec = bytes / 16;
  const size_t total = nvec * (size_t)pa.world;
  for (size_t k = (size_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (size_t)gridDim.x * blockDim.x) {
    const int r = (int)(k / nvec);
    const size_t v = k - (size_t)r * nvec;
    const uint64_t* s8 = reinterpret_cast<const uint64_t*>(src) + 2 * v;
    const uint64_t a = s8[0], b = s8[1];
    reinterpret_cast<int4*>(slot_ptr(pa.base[r], parity, pa.rank, pa.world, pa.slot))[v] =
        make_int4((int)(uint32_t)a, (int)(uint32_t)(a >> 32), (int)(uint32_t)b, (int)(uint32_t)(b >> 32));
  }
  if (bytes % 16 && blockIdx.x == 0 && threadIdx.x < pa.world) {  // payloads are multiples of 8 bytes
    const int r = threadIdx.x;
    reinterpret_cast<uint64_t*>(slot_ptr(pa.base[r], parity, pa.rank, pa.world, pa.slot))[2 * nvec] =
        reinterpret_cast<const uint64_t*>(src)[2 * nvec];
  }
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) last_s = atomicAdd(pa.count, 1u) == gridDim.x - 1;
  __syncthreads();
  if (!last_s) return;
  if (threadIdx.x < pa.world) {
    __threadfence_system();
    st_release_sys(reinterpret_cast<uint64_t*>(pa.base[threadIdx.x] + (size_t)pa.rank * 128), e);
  }
  if (threadIdx.x == 0) *pa.count = 0u;
}

__global__ void peer_collect_kernel(char* __restrict__ dst, size_t bytes, size_t stride, PeerArgs pa) {
  __shared__ bool ok_s, last_s;
  const uint64_t e = *pa.epoch + 1;
  const int parity = (int)(e & 1);
  char* mine = pa.base[pa.rank];
  if (threadIdx.x == 0) {
    bool ok = true;
    const uint64_t t0 = globaltimer_ns();
    for (int r = 0; r < pa.world && ok; ++r) {
      const uint64_t* f = reinterpret_cast<const uint64_t*>(mine + (size_t)r * 128);
      while (ld_acquire_sys(f) < e) {
        if (globaltimer_ns() - t0 > pa.timeout_ns) {
          ok = false;
          atomicExch(pa.err, 1);
          break;
        }
        __nanosleep(256);
      }
    }
    ok_s = ok;
  }
  __syncthreads();
  if (ok_s) {
    const size_t nvec = bytes / 16;
    const size_t total = nvec * (size_t)pa.world;
    for (size_t k = (size_t)blockIdx.x * blockDim.x + threadIdx.x; k < total; k += (size_t)gridDim.x * blockDim.x) {
      const int r = (int)(k / nvec);
      const size_t v = k - (size_t)r * nvec;
      const int4 x = __ldcv(reinterpret_cast<const int4*>(slot_ptr(mine, parity, r, pa.world, pa.slot)) + v);
      uint64_t* o = reinterpret_cast<uint64_t*>(dst + (size_t)r * stride) + 2 * v;  // rows 8-byte aligned
      o[0] = (uint64_t)(uint32_t)x.x | ((uint64_t)(uint32_t)x.y << 32);
      o[1] = (uint64_t)(uint32_t)x.z | ((uint64_t)(uint32_t)x.w << 32);
    }
    if (bytes % 16 && blockIdx.x == 0 && threadIdx.x < pa.world) {
      const int r = threadIdx.x;
      reinterpret_cast<uint64_t*>(dst + (size_t)r * stride)[2 * nvec] =
          __ldcv(reinterpret_cast<const unsigned long long*>(slot_ptr(mine, parity, r, pa.world, pa.slot)) + 2 * nvec);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) last_s = atomicAdd(pa.count + 1, 1u) == gridDim.x - 1;
  __syncthreads();
  if (last_s && threadIdx.x == 0) {
    *pa.epoch = e;
    pa.count[1] = 0u;
  }
}

// fused exchange consumer: wait for every rank's epoch-e slot, rank-order sum into dst
__global__ void peer_combine_kernel(double* __restrict__ dst, int64_t count, PeerArgs pa) {
  __shared__ bool ok_s, last_s;
  const uint64_t e = *pa.epoch + 1;
  const int parity = (int)(e & 1);
  char* mine = pa.base[pa.rank];
  if (threadIdx.x == 0) {
    bool ok = true;
    const uint64_t t0 = globaltimer_ns();
    for (int r = 0; r < pa.world && ok; ++r) {
      const uint64_t* f = reinterpret_cast<const uint64_t*>(mine + (size_t)r * 128);
      while (ld_acquire_sys(f) < e) {
        if (globaltimer_ns() - t0 > pa.timeout_ns) {
          ok = false;
          atomicExch(pa.err, 1);
          break;
        }
        __nanosleep(256);
      }
    }
    ok_s = ok;
  }
  __syncthreads();
  if (ok_s)
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
      double t = 0.0;
      for (int r = 0; r < pa.world; ++r)
        t += __ldcv(reinterpret_cast<const double*>(slot_ptr(mine, parity, r, pa.world, pa.slot)) + i);
      dst[i] = t;
    }
  __syncthreads();
  if (threadIdx.x == 0) last_s = atomicAdd(pa.count + 1, 1u) == gridDim.x - 1;
  __syncthreads();
  if (last_s && threadIdx.x == 0) {
    *pa.epoch = e;
    pa.count[1] = 0u;
  }
}

cudaError_t launch_peer_combine(double* dst, int64_t count, const PeerArgs& pa, int num_sms, cudaStream_t s) {
  int64_t grid = (count + 255) / 256;
  if (grid > num_sms) grid = num_sms;
  if (grid < 1) grid = 1;
  peer_combine_kernel<<<(unsigned)grid, 256, 0, s>>>(dst, count, pa);
  return cudaGetLastError();
}

cudaError_t launch_peer_allgather(const void* src, void* dst, size_t bytes, size_t stride, const PeerArgs& pa,
                                  int num_sms, cudaStream_t s) {
  if (bytes == 0) return cudaSuccess;
  if (bytes > pa.slot || bytes % 8 || stride % 8) return cudaErrorInvalidValue;
  const size_t work = (bytes / 16) * (size_t)pa.world;
  int grid = (int)((work + 255) / 256);
  if (grid > 2 * num_sms) grid = 2 * num_sms;
  if (grid < 1) grid = 1;
  peer_push_kernel<<<grid, 256, 0, s>>>(reinterpret_cast<const char*>(src), bytes, pa);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  peer_collect_kernel<<<grid, 256, 0, s>>>(reinterpret_cast<char*>(dst), bytes, stride, pa);
  return cudaGetLastError();
}

}  // namespace kde
