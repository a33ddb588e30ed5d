// tile_sweep.cu -- PER_GPU tile kernel instantiation for weight set WS_SWEEP, L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_SWEEP)
}  // namespace sched
