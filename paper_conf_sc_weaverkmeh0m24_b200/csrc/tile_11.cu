// tile_11.cu -- PER_GPU tile kernel instantiation for weight set WS_11, L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_11)
}  // namespace sched
