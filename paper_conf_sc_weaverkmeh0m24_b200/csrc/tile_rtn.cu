// tile_rtn.cu -- PER_GPU tile kernel instantiation for run-time weights without b = 0 weights (WS_RTN, WS_RT4N: <= 4 weights), L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_RTN)
SCHED_TILE_INSTANTIATE(4, WS_RT4N)
}  // namespace sched
