// tile_small_l.cu -- PER_GPU tile kernel instantiations for 2 and 3 searched
// levels (per-configuration path, search_tile.cuh small_l_configs): Pareto
// only and run-time weights.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(2, WS_P)
SCHED_TILE_INSTANTIATE(2, WS_RT)
SCHED_TILE_INSTANTIATE(3, WS_P)
SCHED_TILE_INSTANTIATE(3, WS_RT)
}  // namespace sched
