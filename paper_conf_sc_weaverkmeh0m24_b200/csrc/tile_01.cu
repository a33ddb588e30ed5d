// tile_01.cu -- PER_GPU tile kernel instantiation for weight set WS_01, L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_01)
}  // namespace sched
