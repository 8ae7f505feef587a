// peer.cuh -- device side of the peer-memory exchange (peer.cu): stores into every rank's
// window slot and the release of this rank's epoch flag, used by the producers' own tails
// (single-box scan last block, reduce_splits) so the partial sums leave the SM that computed
// them straight over NVLink / NVSwitch -- the fused variant of SURVEY.md §8(e).
#pragma once
#include <cstdint>

#include "common.cuh"

namespace kde {

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(uint64_t* p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ char* peer_slot(char* win, int parity, int src, int world, size_t slot) {
  return win + kPeerFlagBytes + ((size_t)parity * world + src) * slot;
}
// epoch of the exchange in progress (the consumer publishes it when done)
__device__ __forceinline__ uint64_t peer_next_epoch(const PeerArgs& pa) { return *(volatile uint64_t*)pa.epoch + 1; }
// element i (double) of this rank's payload -> every rank's slot
__device__ __forceinline__ void peer_store(const PeerArgs& pa, uint64_t e, int64_t i, double v) {
  const int parity = (int)(e & 1);
  for (int r = 0; r < pa.world; ++r)
    reinterpret_cast<double*>(peer_slot(pa.base[r], parity, pa.rank, pa.world, pa.slot))[i] = v;
}
// after ALL of this rank's stores of epoch e (caller guarantees, e.g. last block): flags up
__device__ __forceinline__ void peer_release(const PeerArgs& pa, uint64_t e) {
  __threadfence_system();
  for (int r = 0; r < pa.world; ++r) st_release_sys(reinterpret_cast<uint64_t*>(pa.base[r] + (size_t)pa.rank * 128), e);
}

}  // namespace kde
