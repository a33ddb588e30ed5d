// tile_rt.cu -- PER_GPU tile kernel instantiation for run-time weights (WS_RT, any W <= 8), L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_RT)
}  // namespace sched
