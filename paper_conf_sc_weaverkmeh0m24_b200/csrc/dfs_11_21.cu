// dfs_11_21.cu -- L = 1 partition kernel instantiation for weight set WS_11_21.
#include "search_dfs.cuh"

namespace sched {
SCHED_DFS_INSTANTIATE(WS_11_21)
}  // namespace sched
