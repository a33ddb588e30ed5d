// sfx_6.cu -- L = 1 suffix kernel instantiation, suffix length M = 6.
#include "search_sfx.cuh"

namespace sched {
template <>
const void *sfx_fn<6>() {
  return (const void *)k_sfx<6>;
}
}  // namespace sched
