// tile_11_21.cu -- PER_GPU tile kernel instantiation for weight set WS_11_21, L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_11_21)
}  // namespace sched
