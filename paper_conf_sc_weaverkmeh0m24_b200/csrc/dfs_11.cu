// dfs_11.cu -- L = 1 partition kernel instantiation for weight set WS_11.
#include "search_dfs.cuh"

namespace sched {
SCHED_DFS_INSTANTIATE(WS_11)
}  // namespace sched
