// dfs_host.cu -- eligibility, weight-set matching and launch of the L = 1
// partition kernel (search_dfs.cuh).
#include "search_dfs.cuh"

namespace sched {

template <class WS>
static bool ws_match_d(const DevParams &dp, int *perm) {
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

bool dfs_eligible(DevParams &dp, TileLaunch *tl) {
  if (dp.L != 1 || dp.g > kDfsMaxG || dp.c > kDfsMaxC || dp.n < 4 || !dp.gtab_ok) return false;
  if (dp.model & SCHED_MODEL_COUNT_IDLE) return false;  // E = sum_g E_g only
  int perm[kMaxW];
  const void *fn = nullptr;
#define TRY(WS)                                                    \
  if (!fn && ws_match_d<WS>(dp, perm) && (WS::N > 0 || dp.want_pareto)) { \
    for (int s = 0; s < WS::N; s++) dp.ws_perm[s] = perm[s];       \
    fn = dfs_fn<WS>();                                             \
  }
  TRY(WS_P)
  TRY(WS_11)
  TRY(WS_10)
  TRY(WS_11_21)
  TRY(WS_SWEEP)
#undef TRY
  if (!fn) return false;
  tl->fn = fn;
  tl->smem = ((dp.blob_bytes + 15) & ~15u) + kStairSmem + sizeof(PairWarp) * (kDfsThreads / 32) +
             sizeof(BestRec) * (kDfsThreads / 32) * kMaxW + sizeof(float) * kDfsThreads * kMaxW;
  return true;
}

cudaError_t launch_dfs(DevParams &dp, const TileLaunch &tl, int nsm, cudaStream_t st, cudaEvent_t e1,
                       cudaEvent_t e2, int *grid, bool fixed_units) {
  cudaError_t err = cudaFuncSetAttribute(tl.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tl.smem);
  if (err != cudaSuccess) return err;
  int occ = 0;
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, tl.fn, kDfsThreads, tl.smem);
  if (err != cudaSuccess) return err;
  if (occ < 1) return cudaErrorInvalidConfiguration;
  *grid = std::min(4096, nsm * occ);
  if (!fixed_units) {  // units of 2^12 .. 2^20 configs, >= ~8 per warp
    const uint64_t range = dp.n_owned << dp.chunk_log2;
    const uint64_t warps = (uint64_t)(*grid) * (kDfsThreads / 32);
    int ul = 12;
    while (ul < 20 && ul < dp.chunk_log2 && (range >> (ul + 1)) >= warps * 8) ul++;
    dp.unit_log2 = ul;
    dp.n_units = dp.n_owned << (dp.chunk_log2 - ul);
    dp.unit_stride = 1;
  }
  err = publish_params(dp, st);
  if (err != cudaSuccess) return err;
  void *args[] = {(void *)&dp};
  cudaEventRecord(e1, st);
  err = cudaLaunchKernel(tl.fn, *grid, kDfsThreads, args, tl.smem, st);
  cudaEventRecord(e2, st);
  return err;
}

}  // namespace sched
