// tile_host.cu -- weight-set matching and launch of the PER_GPU tile kernel.
#include <cstdlib>

#include "search_tile.cuh"

namespace sched {

template <class WS>
static bool ws_match(const DevParams &dp, int *perm) {
  if (dp.nw != WS::N) return false;
  bool used[kMaxW] = {false};
  for (int s = 0; s < WS::N; s++) {
    int found = -1;
    for (int w = 0; w < dp.nw; w++)
      if (!used[w] && dp.wa[w] == WS::A(s) && dp.wb[w] == WS::B(s)) {
        found = w;
        break;
      }
    if (found < 0) return false;
    used[found] = true;
    perm[s] = found;
  }
  return true;
}

template <int L>
static const void *tile_pick_ws(DevParams *dp) {
  if constexpr (L != 4) {  // 2 or 3 levels: per-configuration path, Pareto-only or run-time weights
    if (dp->dump) return nullptr;
    if (dp->nw == 0) return dp->want_pareto ? tile_fn<L, WS_P>() : nullptr;
    if (dp->nw > kMaxW) return nullptr;
    for (int s = 0; s < dp->nw; s++) dp->ws_perm[s] = s;
    return tile_fn<L, WS_RT>();
  }
  int perm[kMaxW];
  if (dp->dump) {  // sched_debug_scores32: the (1,1) kernel that also dumps every configuration's fp32 score
    if (dp->nw != 1 || dp->wa[0] != 1 || dp->wb[0] != 1) return nullptr;
    dp->ws_perm[0] = 0;
    return tile_fn<L, WS_11_DUMP>();
  }
  // SCHED_TILE_RT=1 (measurement): the run-time-weight variant even where a
  // compiled-in weight set matches
  const char *rt = std::getenv("SCHED_TILE_RT");
  const bool force_rt = rt && rt[0] == '1' && dp->nw >= 1;
#define TRY(WS)                                                 \
  if (!force_rt && ws_match<WS>(*dp, perm) && (WS::N > 0 || dp->want_pareto)) { \
    for (int s = 0; s < WS::N; s++) dp->ws_perm[s] = perm[s];     \
    return tile_fn<L, WS>();                                    \
  }
  TRY(WS_P)
  TRY(WS_11)
  TRY(WS_10)
  TRY(WS_01)
  TRY(WS_11_21)
  TRY(WS_C1)      // BASELINE configs[0]'s objectives: (1,0) (0,1) (1,1) (2,1)
  TRY(WS_SWEEP)   // configs[4]'s sweep: (1,0) (3,1) (2,1) (1,1) (1,2) (1,3) (0,1)
#undef TRY
  // any other 1 <= W <= 8: run-time exponents (query order); without b = 0
  // weights the plain tile loop (WS_RTN)
  if (dp->nw >= 1 && dp->nw <= kMaxW) {
    bool b0 = false;
    for (int s = 0; s < dp->nw; s++) {
      dp->ws_perm[s] = s;
      b0 |= dp->wb[s] == 0;
    }
    if (b0) return tile_fn<L, WS_RT>();
    return dp->nw <= 4 ? tile_fn<L, WS_RT4N>() : tile_fn<L, WS_RTN>();
  }
  return nullptr;
}

size_t tile_smem_bytes(const DevParams &dp) {
  return ((dp.blob_bytes + 15) & ~15u) + kStairSmem + sizeof(WarpPart) * kTileWarps +
         sizeof(BestRec) * kTileWarps * kMaxW + sizeof(float) * kTileThreads * (kMaxW + 1);
}

bool tile_eligible(DevParams &dp, TileLaunch *tl) {
  const char *b0 = std::getenv("SCHED_B0");
  dp.b0mode = b0 && *b0 ? std::atoi(b0) : 2;  // tile-level only: the partition-level pass costs more than it saves (c4 (1,0): 740 vs 779 ms)
  if (dp.scope != SCHED_PER_GPU || dp.g > kTileMaxG || dp.L < 2 || dp.L > 4 || !dp.gtab_ok) return false;
  // E = sum_g E_g with level-independent feasibility: COUNT_IDLE (global
  // energy term) and NO_INTERFERENCE (level-dependent feasibility) take the generic kernel
  if (dp.model & SCHED_MODEL_NO_INTERFERENCE) return false;  // level-dependent feasibility: generic kernel
  const void *fn = dp.L == 4 ? tile_pick_ws<4>(&dp) : (dp.L == 3 ? tile_pick_ws<3>(&dp) : tile_pick_ws<2>(&dp));
  if (!fn) return false;
  tl->fn = fn;
  tl->smem = tile_smem_bytes(dp);
  return true;
}

cudaError_t launch_tile(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                        cudaEvent_t e2, int *grid, bool fixed_units) {
  cudaError_t err = cudaFuncSetAttribute(tl.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tl.smem);
  if (err != cudaSuccess) return err;
  int occ = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, tl.fn, kTileThreads, tl.smem);
  if (err != cudaSuccess) return err;
  if (occ < 1) return cudaErrorInvalidConfiguration;
  *grid = std::min(4096, nsm * occ);
  // unit size: ~16 units per warp over the search, 2^12 .. 2^chunk_log2 configs
  if (!fixed_units) {
    const uint64_t range = dp.n_owned << dp.chunk_log2;
    const uint64_t warps = (uint64_t)(*grid) * kTileWarps;
    uint64_t upw = 16;  // SCHED_TILE_UPW (measurement): target units per warp
    if (const char *e = std::getenv("SCHED_TILE_UPW")) upw = std::max(1, std::atoi(e));
    int ul = 12;
    while (ul < dp.chunk_log2 && (range >> (ul + 1)) >= warps * upw) ul++;
    dp.unit_log2 = ul;
    dp.n_units = dp.n_owned << (dp.chunk_log2 - ul);
    dp.unit_stride = 1;
  }
  err = publish_params(dp, st);
  if (err != cudaSuccess) return err;
  void *args[] = {(void *)&dp};
  cudaEventRecord(e1, st);
  err = cudaLaunchKernel(tl.fn, *grid, kTileThreads, args, tl.smem, st);
  cudaEventRecord(e2, st);
  return err;
}

}  // namespace sched
