// tile_10.cu -- PER_GPU tile kernel instantiation for weight set WS_10, L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_10)
}  // namespace sched
