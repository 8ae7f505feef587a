// reservoir.cu -- host-side sample maintenance for insert-only workloads
// (Section 4.2, P:L189 / P:L248): "we utilize the well-known reservoir sampling
// algorithm [43] ... all decisions are made independently by the host and only
// points that will end up in the sample are transferred to the graphics card".
//
// Algorithm R with a counter-based draw (so a decision is a pure function of
// (seed, arrival index), independent of how arrivals are chunked or which rank
// asks): arrival a (1-based; the first n_sample arrivals fill the sample) takes
//   z = SplitMix64 finaliser of (seed + a * 0x9E3779B97F4A7C15),
//   j = floor(z * a / 2^64)  (uniform on [0, a)),
// and replaces slot j iff j < n_sample.
#include <cstdint>
#include <cstring>

#include "../../include/kde.h"
#include "kernels.cuh"

namespace kde {

static inline uint64_t splitmix_final(uint64_t seed, uint64_t a) {
  uint64_t z = seed + a * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

void reservoir_slots(uint64_t seed, int64_t n_sample, int64_t n_seen, int64_t k, int64_t* slot_out) {
  for (int64_t r = 0; r < k; ++r) {
    const uint64_t a = (uint64_t)(n_seen + r + 1);
    if ((int64_t)a <= n_sample) {
      slot_out[r] = (int64_t)a - 1;
      continue;
    }
    const uint64_t j = (uint64_t)(((unsigned __int128)splitmix_final(seed, a) * (unsigned __int128)a) >> 64);
    slot_out[r] = j < (uint64_t)n_sample ? (int64_t)j : -1;
  }
}

}  // namespace kde

