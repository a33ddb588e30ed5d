// search_tile.cuh -- specialised PER_GPU tile kernel (c3/c4 fast path).
// Placeholder: the generic kernel serves every query until this lands.
#pragma once
#include "device_common.cuh"

namespace sched {

struct TileLaunch {
  int L;
};

inline bool tile_eligible(const DevParams &, TileLaunch *) { return false; }

inline cudaError_t launch_tile(const DevParams &, const TileLaunch &, int, cudaStream_t, cudaEvent_t,
                               cudaEvent_t, int *grid) {
  *grid = 0;
  return cudaErrorNotSupported;
}

}  // namespace sched
