// tile_c1.cu -- PER_GPU tile kernel instantiation for weight set WS_C1, L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_C1)
}  // namespace sched
