// sfx_7.cu -- L = 1 suffix kernel instantiation, suffix length M = 7.
#include "search_sfx.cuh"

namespace sched {
template <>
const void *sfx_fn<7>() {
  return (const void *)k_sfx<7>;
}
}  // namespace sched
