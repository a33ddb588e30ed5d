// event_guard.hpp -- CUDA events owned by a scope: destroyed on every return
// path (early CUDA-error returns included), so a long-lived caller that sees
// failed calls does not leak events.
#pragma once
#include <cuda_runtime.h>

namespace sched {

template <int N>
struct EventGuard {
  cudaEvent_t e[N] = {};
  // creates all N events; false (and nothing leaked) on failure
  bool create() {
    for (int i = 0; i < N; i++)
      if (cudaEventCreate(&e[i]) != cudaSuccess) {
        e[i] = nullptr;
        return false;
      }
    return true;
  }
  ~EventGuard() {
    for (int i = 0; i < N; i++)
      if (e[i]) cudaEventDestroy(e[i]);
  }
  cudaEvent_t operator[](int i) const { return e[i]; }
};

}  // namespace sched
