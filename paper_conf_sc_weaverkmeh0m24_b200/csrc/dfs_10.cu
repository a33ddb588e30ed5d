// dfs_10.cu -- L = 1 partition kernel instantiation for weight set WS_10.
#include "search_dfs.cuh"

namespace sched {
SCHED_DFS_INSTANTIATE(WS_10)
}  // namespace sched
