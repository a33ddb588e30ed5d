// sfx_4.cu -- L = 1 suffix kernel instantiation, suffix length M = 4.
#include "search_sfx.cuh"

namespace sched {
template <>
const void *sfx_fn<4>() {
  return (const void *)k_sfx<4>;
}
}  // namespace sched
