// dfs_sweep.cu -- L = 1 partition kernel instantiation for weight set WS_SWEEP.
#include "search_dfs.cuh"

namespace sched {
SCHED_DFS_INSTANTIATE(WS_SWEEP)
}  // namespace sched
