// tile_registry.hpp -- host-side selection of the PER_GPU tile kernel.
// The kernels are instantiated in tile_*.cu (one weight set per translation
// unit, compiled in parallel); search.cu only sees these declarations.
#pragma once
#include <algorithm>
#include <cuda_runtime.h>

#include "sched_internal.hpp"

namespace sched {

struct WS_P;
struct WS_11;
struct WS_10;
struct WS_01;
struct WS_11_21;
struct WS_SWEEP;
struct WS_C1;
struct WS_RT;
struct WS_RTN;
struct WS_RT4N;
struct WS_11_DUMP;

template <int L, class WS>
const void *tile_fn();

struct TileLaunch {
  const void *fn;
  size_t smem;
  int slots_per_cta = 1;  // best slots written per CTA (k_sfx: one per warp)
};

#ifndef SCHED_TILE_THREADS
#define SCHED_TILE_THREADS 512
#endif
#ifndef SCHED_TILE_MINB
#define SCHED_TILE_MINB 1
#endif
constexpr int kTileThreads = SCHED_TILE_THREADS;
constexpr int kTileMinBlocks = SCHED_TILE_MINB;  // __launch_bounds__ min blocks per SM
constexpr int kTileWarps = kTileThreads / 32;
constexpr int kTileMaxL = 4;
constexpr int kTileMaxG = 8;
size_t tile_smem_bytes(const DevParams &dp);
// the launch's DevParams -> its workspace copy (dp.gp), before the kernel
inline cudaError_t publish_params(const DevParams &dp, cudaStream_t st) {
  return cudaMemcpyAsync((void *)dp.gp, &dp, sizeof dp, cudaMemcpyHostToDevice, st);
}
bool tile_eligible(DevParams &dp, TileLaunch *tl);
bool dfs_eligible(DevParams &dp, TileLaunch *tl);
bool sfx_eligible(DevParams &dp, TileLaunch *tl);
bool ctile_eligible(DevParams &dp, TileLaunch *tl);
bool ctile2_eligible(DevParams &dp, TileLaunch *tl);
size_t ctile2_t64_bytes();
cudaError_t launch_ctile2(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                          cudaEvent_t e2, int *grid, bool fixed_units);
cudaError_t launch_ctile(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                         cudaEvent_t e2, int *grid, bool fixed_units);
cudaError_t launch_sfx(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                       cudaEvent_t e2, int *grid, bool fixed_units);
cudaError_t launch_dfs(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                       cudaEvent_t e2, int *grid, bool fixed_units);
cudaError_t launch_tile(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                        cudaEvent_t e2, int *grid, bool fixed_units);

}  // namespace sched
