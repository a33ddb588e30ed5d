// ctile2.cu -- eligibility and launch of the group-table PER_CLIENT tile
// kernel (search_ctile2.cuh, kernel_path 6): PER_CLIENT scope, L = 4,
// 6 <= n <= 15, groups of <= 4 clients (C <= 4), G <= 8, canonical model or
// POWER_CAP (E = sum_g E_g, level-independent feasibility).
#include <cstdio>
#include <cstdlib>

#include "search_ctile2.cuh"

namespace sched {

static size_t ctile2_smem(const DevParams &dp) {
  return ((dp.blob_bytes + 15) & ~15u) + kStairSmem + sizeof(C2Warp) * kC2Warps + sizeof(BestRec) * kC2Warps * kMaxW;
}

size_t ctile2_t64_bytes() { return sizeof(double) * (size_t)kC2MaxGrid * kC2Warps * kC2Tab; }

bool ctile2_eligible(DevParams &dp, TileLaunch *tl) {
  if (dp.scope != SCHED_PER_CLIENT || dp.L != 4 || dp.n < 6 || dp.n > 15 || dp.g > 8) return false;
  if (dp.c > 4) return false;  // groups of <= 4 clients: tables <= 836 entries
  if (dp.model & (SCHED_MODEL_COUNT_IDLE | SCHED_MODEL_NO_INTERFERENCE | SCHED_MODEL_TIME_SLICE)) return false;
  if (ctile2_smem(dp) > 227 * 1024) return false;
  tl->fn = dp.nw <= 1 ? ctile2_fn<1>() : dp.nw <= 2 ? ctile2_fn<2>() : dp.nw <= 4 ? ctile2_fn<4>() : ctile2_fn<8>();
  tl->smem = ctile2_smem(dp);
  return true;
}

cudaError_t launch_ctile2(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                          cudaEvent_t e2, int *grid, bool fixed_units) {
  cudaError_t err = cudaFuncSetAttribute(tl.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tl.smem);
  if (err != cudaSuccess) return err;
  int occ = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, tl.fn, kC2Threads, tl.smem);
  if (err != cudaSuccess) return err;
  if (occ < 1) return cudaErrorInvalidConfiguration;
  *grid = std::min(kC2MaxGrid, nsm * occ);
  dp.c2_seed_tiles = 0;
  if (fixed_units && dp.chunk_log2 >= 12) {
    // seed pass: per_sm x nsm units of 2^ul indices spread over the shard
    // (SCHED_C2_SEED="ul,per_sm"); a unit only picks a place in its
    // partition, from which the kernel samples 32 whole steps of tiles
    // (c2_seed_tiles; SCHED_C2_SEED_TILES=0 for the index ranges themselves,
    // which cut every tile whose clients carry high index digits)
    if (const char *e = std::getenv("SCHED_C2_SEED_TILES")) dp.c2_seed_tiles = std::atoi(e);
    else dp.c2_seed_tiles = 1;
    int sl = 16, per = 64;  // c3-client slice: 161 ms (32 per SM: 162)
    if (const char *e = std::getenv("SCHED_C2_SEED")) std::sscanf(e, "%d,%d", &sl, &per);
    sl = std::max(10, std::min(sl, dp.chunk_log2));
    const uint64_t units = dp.n_owned << (dp.chunk_log2 - sl);
    dp.unit_log2 = sl;
    dp.n_units = std::min<uint64_t>(units, (uint64_t)nsm * std::max(1, per));
    dp.unit_stride = std::max<uint64_t>(1, units / std::max<uint64_t>(1, dp.n_units));
  }
  if (!fixed_units) {  // units of 2^12 .. 2^chunk_log2 configs, >= ~8 per warp
    const uint64_t range = dp.n_owned << dp.chunk_log2;
    const uint64_t warps = (uint64_t)(*grid) * kC2Warps;
    int ul = 12;
    while (ul < dp.chunk_log2 && (range >> (ul + 1)) >= warps * 8) ul++;
    dp.unit_log2 = ul;
    dp.n_units = dp.n_owned << (dp.chunk_log2 - ul);
    dp.unit_stride = 1;
  }
  err = publish_params(dp, st);
  if (err != cudaSuccess) return err;
  void *args[] = {(void *)&dp};
  cudaEventRecord(e1, st);
  err = cudaLaunchKernel(tl.fn, *grid, kC2Threads, args, tl.smem, st);
  cudaEventRecord(e2, st);
  return err;
}

}  // namespace sched
