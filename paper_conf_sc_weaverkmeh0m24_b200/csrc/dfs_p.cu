// dfs_p.cu -- L = 1 partition kernel instantiation for weight set WS_P.
#include "search_dfs.cuh"

namespace sched {
SCHED_DFS_INSTANTIATE(WS_P)
}  // namespace sched
