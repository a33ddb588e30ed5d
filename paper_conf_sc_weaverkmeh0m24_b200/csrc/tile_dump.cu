// tile_dump.cu -- PER_GPU tile kernel instantiation that dumps every
// configuration's fp32 score (WS_11_DUMP, sched_debug_scores32), L = 4.
#include "search_tile.cuh"

namespace sched {
SCHED_TILE_INSTANTIATE(4, WS_11_DUMP)
}  // namespace sched
