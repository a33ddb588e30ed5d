// sfx_host.cu -- eligibility and launch of the L = 1 suffix kernel
// (search_sfx.cuh); instantiations in sfx_<M>.cu.
#include <cstdlib>

#include "search_sfx.cuh"

namespace sched {

static size_t sfx_smem(const DevParams &dp, int M) {
  const size_t warp = M == 7 ? sizeof(SfxWarp<7>) : M == 6 ? sizeof(SfxWarp<6>) : sizeof(SfxWarp<4>);
  return ((dp.blob_bytes + 15) & ~15u) + kStairSmem + warp * kSfxWarps + sizeof(BestRec) * kSfxWarps * kMaxW;
}

bool sfx_eligible(DevParams &dp, TileLaunch *tl) {
  if (dp.L != 1 || dp.g > kSfxMaxG || (dp.capped && dp.c > 15) || !dp.gtab_ok) return false;
  if (dp.model & SCHED_MODEL_COUNT_IDLE) return false;  // E = sum_g E_g only
  // suffix length: 7 for n >= 12 (2^7-entry rows, 16 warps x 8.3 KB of tables;
  // c5 392 ms vs 485 with M = 6: 14x fewer prefixes, so fewer table rebuilds,
  // unranks and partial grandparents), 6 for n >= 8, 4 for n = 6, 7
  int M;
  if (dp.n >= 12) M = 7;
  else if (dp.n >= 8) M = 6;
  else if (dp.n >= 6) M = 4;
  else return false;
  // SCHED_SFX_M=6 / 7 (measurement): force the suffix length where it applies
  if (const char *e = std::getenv("SCHED_SFX_M")) {
    const int m = std::atoi(e);
    if ((m == 6 && dp.n >= 8) || (m == 7 && dp.n >= 12)) M = m;
  }
  tl->fn = M == 7 ? sfx_fn<7>() : M == 6 ? sfx_fn<6>() : sfx_fn<4>();
  tl->smem = sfx_smem(dp, M);
  tl->slots_per_cta = kSfxWarps;
  return true;
}

cudaError_t launch_sfx(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                       cudaEvent_t e2, int *grid, bool fixed_units) {
  cudaError_t err = cudaFuncSetAttribute(tl.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tl.smem);
  if (err != cudaSuccess) return err;
  int occ = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, tl.fn, kSfxThreads, tl.smem);
  if (err != cudaSuccess) return err;
  if (occ < 1) return cudaErrorInvalidConfiguration;
  *grid = std::min(4096 / kSfxWarps, nsm * occ);  // per-warp best slots: grid * kSfxWarps <= kMaxGrid
  if (!fixed_units) {  // units of 2^12 .. 2^chunk_log2 configs, >= ~8 per warp
    const uint64_t range = dp.n_owned << dp.chunk_log2;
    const uint64_t warps = (uint64_t)(*grid) * kSfxWarps;
    int ul = 12;
    // <= 2^22: the suffix kernel loses to the last-unit tail with larger units (c5: 752 vs 770 ms at 2^24)
    while (ul < std::min(dp.chunk_log2, 22) && (range >> (ul + 1)) >= warps * 8) ul++;
    dp.unit_log2 = ul;
    dp.n_units = dp.n_owned << (dp.chunk_log2 - ul);
    dp.unit_stride = 1;
  }
  err = publish_params(dp, st);
  if (err != cudaSuccess) return err;
  void *args[] = {(void *)&dp};
  cudaEventRecord(e1, st);
  err = cudaLaunchKernel(tl.fn, *grid, kSfxThreads, args, tl.smem, st);
  cudaEventRecord(e2, st);
  return err;
}

}  // namespace sched
