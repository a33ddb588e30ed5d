// tile_p.cu -- PER_GPU tile kernel instantiation for weight set WS_P, L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_P)
}  // namespace sched
