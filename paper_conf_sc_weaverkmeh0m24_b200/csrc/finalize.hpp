// finalize.hpp -- exact Pareto front of the candidates by sort + sweep (finalize.cu).
#pragma once
#include <cuda_runtime.h>

#include "sched_internal.hpp"

namespace sched {
// workspace bytes of the finalize scratch for a candidate capacity
size_t finalize_bytes(uint32_t cap);
// m survivor slots at surv -> front (T ascending) after the best records in
// p.out, its size in ctr[kCtrFront]; adds its own kernel launches to *launches
cudaError_t finalize_front(const DevParams &p, unsigned char *fin, size_t fin_bytes, const unsigned int *surv, int m,
                           int out_cap, int nsm, cudaStream_t st, int *launches);
}  // namespace sched
