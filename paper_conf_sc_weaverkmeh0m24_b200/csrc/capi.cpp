// capi.cpp -- the extern "C" boundary declared in include/sched.h.
// Argument checking, handle/cache management, staging, result conversion.
// No exception crosses the ABI (every entry point catches).
#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: ranges for nsys / ncu --nvtx (SURVEY 5 tracing)
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <new>

#include "event_guard.hpp"
#include "sched_internal.hpp"


namespace {
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace

using namespace sched;

struct sched_handle {
  Profile P;
  // cached DP space for the last query shape
  int sp_key[5] = {-1, -1, -1, -1, -1};
  Space sp;
  // staged workspace state
  const void *staged_ws = nullptr;
  std::vector<unsigned char> staged_blob;
  void *pinned = nullptr;
  size_t pinned_bytes = 0;
};

namespace {

int get_space(sched_handle *h, const Query &q, const Space **out) {
  const int key[5] = {q.n, q.g, q.c, q.L, q.scope};
  if (std::memcmp(key, h->sp_key, sizeof key) != 0) {
    int st = build_space(q, &h->sp);
    if (st) {
      h->sp_key[0] = -1;
      return st;
    }
    std::memcpy(h->sp_key, key, sizeof key);
  }
  *out = &h->sp;
  return SCHED_OK;
}

int resolve(sched_handle *h, const sched_query *qin, Query *q, const Space **sp) {
  int st = resolve_query_shape(qin, h->P.lp, q);
  if (st) return st;
  if (q->n > h->P.n) return SCHED_E_INVALID;
  if ((q->model & SCHED_MODEL_POWER_CAP) && !(q->pcap > h->P.ps)) return SCHED_E_INVALID;  // R28
  st = get_space(h, *q, sp);
  if (st) return st;
  if (q->hi == UINT64_MAX || q->hi > (*sp)->total) q->hi = (*sp)->total;
  if (q->lo > q->hi) return SCHED_E_INVALID;
  return SCHED_OK;
}

// query for the subset-DP front: shape + profile checks, whole space, one
// shard; no DP count table (the literal per-client spaces exceed 2^63)
int resolve_dp(sched_handle *h, const sched_query *qin, Query *q, std::vector<unsigned char> *blob, DevParams *dp) {
  int st = resolve_query_shape(qin, h->P.lp, q);
  if (st) return st;
  if (q->n > h->P.n) return SCHED_E_INVALID;
  if ((q->model & SCHED_MODEL_POWER_CAP) && !(q->pcap > h->P.ps)) return SCHED_E_INVALID;
  if (q->lo != 0 || (q->hi != 0 && q->hi != UINT64_MAX) || q->count != 1) return SCHED_E_INVALID;
  q->lo = 0;
  q->hi = 0;
  Space empty;
  empty.n = q->n;
  empty.g = q->g;
  empty.c = q->c;
  empty.L = q->L;
  empty.scope = q->scope;
  return build_stage(h->P, *q, empty, blob, dp);
}

int need_device() {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n < 1) {
    cudaGetLastError();
    return SCHED_E_NODEVICE;
  }
  return SCHED_OK;
}

int do_stage(sched_handle *h, const DevParams &dp, const std::vector<unsigned char> &blob, void *ws,
             void *stream) {
  if (h->pinned_bytes < blob.size()) {
    if (h->pinned) cudaFreeHost(h->pinned);
    h->pinned = nullptr;
    h->pinned_bytes = 0;
    if (cudaHostAlloc(&h->pinned, blob.size() + 4096, cudaHostAllocDefault) != cudaSuccess) {
      cudaGetLastError();
      return SCHED_E_CUDA;
    }
    h->pinned_bytes = blob.size() + 4096;
  }
  int st = stage_tables(dp, blob, ws, h->pinned, stream);
  if (st) return st;
  h->staged_ws = ws;
  h->staged_blob = blob;
  return SCHED_OK;
}

void fill_pick(const Query &q, const DevParams &dp, int w, const BestRec &b, sched_pick *o) {
  std::memset(o, 0, sizeof *o);
  if (!b.valid) return;
  o->valid = 1;
  o->index = b.idx;
  o->makespan_s = b.t;
  o->energy_j = b.e;
  o->x64 = dp.tseq / b.t;
  o->y64 = dp.eseq / b.e;
  o->score64 = b.f;
  o->x32 = 1.f / b.t32;
  o->y32 = 1.f / b.e32;
  float s = 1.f;
  for (int i = 0; i < q.wa[w]; i++) s *= o->x32;
  for (int i = 0; i < q.wb[w]; i++) s *= o->y32;
  o->score32 = s;
}

// split search setup (R29): admissible split vectors and the unsplit baselines
int split_setup(sched_handle *h, const sched_query *qin, const int32_t *tasks, const int32_t *max_split,
                std::vector<std::vector<int>> *svs, double *tseq, double *eseq) {
  if (!h || !qin || !tasks) return SCHED_E_INVALID;
  Query q;
  int st = resolve_query_shape(qin, h->P.lp, &q);
  if (st) return st;
  if (q.n > h->P.n) return SCHED_E_INVALID;
  if ((q.model & SCHED_MODEL_POWER_CAP) && !(q.pcap > h->P.ps)) return SCHED_E_INVALID;
  if (qin->index_lo != 0 || qin->index_hi != UINT64_MAX || q.count != 1) return SCHED_E_INVALID;
  st = split_vectors(q.n, tasks, max_split, svs);
  if (st) return st;
  host_constants(h->P, q, tseq, eseq);
  return SCHED_OK;
}

}  // namespace

#define GUARD_BEGIN try {
#define GUARD_END                 \
  }                               \
  catch (const std::bad_alloc &) { \
    return SCHED_E_TOO_LARGE;     \
  }                               \
  catch (...) {                   \
    return SCHED_E_INVALID;       \
  }

extern "C" {

int sched_create(const sched_profile *profile, sched_handle **out) {
  GUARD_BEGIN
  NvtxRange nvtx_range_("sched_create");
  if (!out) return SCHED_E_INVALID;
  *out = nullptr;
  sched_handle *h = new sched_handle();
  int st = validate_profile(profile, &h->P);
  if (st) {
    delete h;
    return st;
  }
  *out = h;
  return SCHED_OK;
  GUARD_END
}

int sched_destroy(sched_handle *h) {
  GUARD_BEGIN
  if (!h) return SCHED_E_INVALID;
  if (h->pinned) cudaFreeHost(h->pinned);
  delete h;
  return SCHED_OK;
  GUARD_END
}

int sched_count(const sched_query *qin, uint64_t *count) {
  GUARD_BEGIN
  if (!count) return SCHED_E_INVALID;
  Query q;
  int st = resolve_query_shape(qin, 32, &q);
  if (st) return st;
  Space sp;
  st = build_space(q, &sp);
  if (st) return st;
  *count = sp.total;
  return SCHED_OK;
  GUARD_END
}

int sched_workspace_size(const sched_handle *hc, const sched_query *qin, size_t *bytes) {
  GUARD_BEGIN
  if (!hc || !bytes) return SCHED_E_INVALID;
  sched_handle *h = const_cast<sched_handle *>(hc);
  Query q;
  const Space *sp;
  int st = resolve(h, qin, &q, &sp);
  if (st) return st;
  std::vector<unsigned char> blob;
  DevParams dp;
  st = build_stage(h->P, q, *sp, &blob, &dp);
  if (st) return st;
  *bytes = workspace_bytes(dp, 0);
  return SCHED_OK;
  GUARD_END
}

int sched_stage(sched_handle *h, const sched_query *qin, void *ws, size_t ws_bytes, void *stream) {
  GUARD_BEGIN
  if (!h || !ws) return SCHED_E_INVALID;
  int st = need_device();
  if (st) return st;
  Query q;
  const Space *sp;
  st = resolve(h, qin, &q, &sp);
  if (st) return st;
  std::vector<unsigned char> blob;
  DevParams dp;
  st = build_stage(h->P, q, *sp, &blob, &dp);
  if (st) return st;
  if (ws_bytes < workspace_bytes(dp, 0) || ((uintptr_t)ws & 255)) return SCHED_E_WORKSPACE;
  return do_stage(h, dp, blob, ws, stream);
  GUARD_END
}

int sched_search(sched_handle *h, const sched_query *qin, void *ws, size_t ws_bytes, void *stream,
                 sched_pick *best, sched_pick *pareto, uint64_t pareto_cap, uint64_t *n_pareto,
                 sched_stats *stats) {
  GUARD_BEGIN
  NvtxRange nvtx_range_("sched_search");
  if (!h || !ws) return SCHED_E_INVALID;
  int st = need_device();
  if (st) return st;
  Query q;
  const Space *sp;
  st = resolve(h, qin, &q, &sp);
  if (st) return st;
  if (q.nw > 0 && !best) return SCHED_E_INVALID;
  if (q.want_pareto && (!n_pareto || (pareto_cap > 0 && !pareto))) return SCHED_E_INVALID;
  std::vector<unsigned char> blob;
  DevParams dp;
  st = build_stage(h->P, q, *sp, &blob, &dp);
  if (st) return st;
  if (ws_bytes < workspace_bytes(dp, 0) || ((uintptr_t)ws & 255)) return SCHED_E_WORKSPACE;
  EventGuard<2> ev;  // destroyed on every return path
  if (!ev.create()) return SCHED_E_CUDA;
  cudaEvent_t t0 = ev[0], t1 = ev[1];
  cudaEventRecord(t0, (cudaStream_t)stream);
  uint64_t h2d = 0;
  if (h->staged_ws != ws || h->staged_blob != blob) {
    st = do_stage(h, dp, blob, ws, stream);
    if (st) return st;
    h2d = blob.size();
  }
  LaunchInfo info{};
  std::vector<BestRec> bres;
  std::vector<CandRec> front;
  uint64_t ctr[kCtrN];
  st = launch_search(dp, ws, ws_bytes, stream, &info, &bres, &front, ctr);
  cudaEventRecord(t1, (cudaStream_t)stream);
  cudaEventSynchronize(t1);
  float total_ms = 0.f;
  cudaEventElapsedTime(&total_ms, t0, t1);
  if (st && st != SCHED_E_CAPACITY) return st;
  if (ctr[kCtrOverflow]) st = SCHED_E_CAPACITY;
  for (int w = 0; w < q.nw; w++) fill_pick(q, dp, w, bres[w], &best[w]);
  if (q.want_pareto) {
    *n_pareto = front.size();
    if (front.size() > pareto_cap) {
      st = SCHED_E_CAPACITY;
    } else {
      for (size_t k = 0; k < front.size(); k++) {
        sched_pick &o = pareto[k];
        std::memset(&o, 0, sizeof o);
        o.valid = 1;
        o.index = front[k].idx;
        o.makespan_s = front[k].t;
        o.energy_j = front[k].e;
        o.x64 = dp.tseq / front[k].t;
        o.y64 = dp.eseq / front[k].e;
        o.score64 = o.x64;  // Pareto picks: score = X (throughput)
        o.x32 = 1.f / front[k].t32;
        o.y32 = 1.f / front[k].e32;
        o.score32 = o.x32;
      }
    }
  } else if (n_pareto) {
    *n_pareto = 0;
  }
  if (stats) {
    std::memset(stats, 0, sizeof *stats);
    stats->n_configs = ctr[kCtrConfigs];
    stats->n_feasible = ctr[kCtrFeasible];
    stats->n_refined = ctr[kCtrRefined];
    stats->n_candidates = ctr[kCtrCand];
    stats->t_seq_s = dp.tseq;
    stats->e_seq_j = dp.eseq;
    stats->search_ms = info.search_ms;
    stats->main_ms = info.main_ms;
    stats->total_ms = total_ms;
    stats->kernel_path = info.path;
    stats->grid_ctas = info.grid;
    stats->kernel_launches = info.launches;
    stats->passes = info.passes;
    stats->h2d_bytes = h2d;
    stats->d2h_bytes = info.d2h_bytes;
  }
  if (st) return st;
  if (ctr[kCtrFeasible] == 0) return SCHED_E_INFEASIBLE;
  return SCHED_OK;
  GUARD_END
}

int sched_merge(int32_t n_ranks, int32_t n_weights, const sched_pick *rank_best,
                const sched_pick *rank_pareto, const uint64_t *rank_npareto, sched_pick *best,
                sched_pick *pareto, uint64_t pareto_cap, uint64_t *n_pareto) {
  GUARD_BEGIN
  NvtxRange nvtx_range_("sched_merge");
  return merge_picks(n_ranks, n_weights, rank_best, rank_pareto, rank_npareto, best, pareto, pareto_cap,
                     n_pareto);
  GUARD_END
}

int sched_unrank(const sched_query *qin, uint64_t index, int8_t *group_of, int8_t *level_of) {
  GUARD_BEGIN
  if (!group_of || !level_of) return SCHED_E_INVALID;
  Query q;
  int st = resolve_query_shape(qin, 32, &q);
  if (st) return st;
  Space sp;
  st = build_space(q, &sp);
  if (st) return st;
  int8_t dig[kMaxN];
  int k;
  st = host_unrank(sp, index, group_of, dig, &k);
  if (st) return st;
  for (int i = 0; i < q.n; i++) level_of[i] = q.scope == SCHED_PER_CLIENT ? dig[i] : dig[group_of[i]];
  return SCHED_OK;
  GUARD_END
}

int sched_rank(const sched_query *qin, const int8_t *group_of, const int8_t *level_of, uint64_t *index) {
  GUARD_BEGIN
  if (!group_of || !level_of || !index) return SCHED_E_INVALID;
  Query q;
  int st = resolve_query_shape(qin, 32, &q);
  if (st) return st;
  Space sp;
  st = build_space(q, &sp);
  if (st) return st;
  int8_t dig[kMaxN];
  int k = 0;
  for (int i = 0; i < q.n; i++) {  // validate before any dig[] write (group ids index dig)
    if (group_of[i] < 0 || group_of[i] >= q.g || group_of[i] >= kMaxG) return SCHED_E_INVALID;
    if (level_of[i] < 0 || level_of[i] >= q.L) return SCHED_E_INVALID;
    k = group_of[i] + 1 > k ? group_of[i] + 1 : k;
  }
  if (q.scope == SCHED_PER_CLIENT) {
    for (int i = 0; i < q.n; i++) dig[i] = level_of[i];
  } else {
    for (int g = 0; g < k; g++) dig[g] = -1;
    for (int i = 0; i < q.n; i++) {
      const int g = group_of[i];
      if (g < 0 || g >= kMaxG) return SCHED_E_INVALID;
      if (dig[g] >= 0 && dig[g] != level_of[i]) return SCHED_E_INVALID;
      dig[g] = level_of[i];
    }
  }
  return host_rank(sp, group_of, dig, index);
  GUARD_END
}

int sched_unrank_device(sched_handle *h, const sched_query *qin, const uint64_t *d_index, uint64_t n,
                        uint64_t advance, int8_t *d_group_of, int8_t *d_level_of, void *ws, size_t ws_bytes,
                        void *stream) {
  GUARD_BEGIN
  NvtxRange nvtx_range_("sched_unrank_device");
  if (!h || !ws || (n > 0 && (!d_index || !d_group_of || !d_level_of))) return SCHED_E_INVALID;
  int st = need_device();
  if (st) return st;
  Query q;
  const Space *sp;
  st = resolve(h, qin, &q, &sp);
  if (st) return st;
  std::vector<unsigned char> blob;
  DevParams dp;
  st = build_stage(h->P, q, *sp, &blob, &dp);
  if (st) return st;
  if (ws_bytes < workspace_bytes(dp, 0) || ((uintptr_t)ws & 255)) return SCHED_E_WORKSPACE;
  if (h->staged_ws != ws || h->staged_blob != blob) {
    st = do_stage(h, dp, blob, ws, stream);
    if (st) return st;
  }
  return launch_unrank(dp, ws, ws_bytes, stream, d_index, n, advance, d_group_of, d_level_of);
  GUARD_END
}

int sched_debug_scores32(sched_handle *h, const sched_query *qin, void *ws, size_t ws_bytes, void *stream,
                         float *d_scores) {
  GUARD_BEGIN
  if (!h || !qin || !ws || !d_scores) return SCHED_E_INVALID;
  int st = need_device();
  if (st) return st;
  sched_query qq = *qin;
  const int32_t w11[2] = {1, 1};
  qq.weights = w11;
  qq.n_weights = 1;
  qq.want_pareto = 0;
  Query q;
  const Space *sp;
  st = resolve(h, &qq, &q, &sp);
  if (st) return st;
  if (q.hi - q.lo > ((uint64_t)1 << 26)) return SCHED_E_INVALID;
  std::vector<unsigned char> blob;
  DevParams dp;
  st = build_stage(h->P, q, *sp, &blob, &dp);
  if (st) return st;
  if (ws_bytes < workspace_bytes(dp, 0) || ((uintptr_t)ws & 255)) return SCHED_E_WORKSPACE;
  if (h->staged_ws != ws || h->staged_blob != blob) {
    st = do_stage(h, dp, blob, ws, stream);
    if (st) return st;
  }
  dp.dump = (unsigned char *)d_scores;
  dp.dump_lo = q.lo;
  dp.dump_n = q.hi - q.lo;
  LaunchInfo info{};
  std::vector<BestRec> bres;
  std::vector<CandRec> front;
  uint64_t ctr[kCtrN];
  st = launch_search(dp, ws, ws_bytes, stream, &info, &bres, &front, ctr);
  if (st) return st;
  if (info.path != 1) return SCHED_E_INVALID;
  return SCHED_OK;
  GUARD_END
}

int sched_score(const sched_handle *hc, const sched_query *qin, uint64_t index, int32_t w, sched_pick *out) {
  GUARD_BEGIN
  if (!hc || !out) return SCHED_E_INVALID;
  sched_handle *h = const_cast<sched_handle *>(hc);
  Query q;
  const Space *sp;
  int st = resolve(h, qin, &q, &sp);
  if (st) return st;
  if (w < 0 || (q.nw > 0 && w >= q.nw) || (q.nw == 0 && w != 0)) return SCHED_E_INVALID;
  int8_t a[kMaxN], dig[kMaxN];
  int k;
  st = host_unrank(*sp, index, a, dig, &k);
  if (st) return st;
  std::memset(out, 0, sizeof *out);
  out->index = index;
  double T, E, ts, es;
  host_constants(h->P, q, &ts, &es);
  if (!host_score(h->P, q, a, k, dig, &T, &E)) return SCHED_OK;  // valid = 0: infeasible
  out->valid = 1;
  out->makespan_s = T;
  out->energy_j = E;
  out->x64 = ts / T;
  out->y64 = es / E;
  const int ea = q.nw ? q.wa[w] : 1, eb = q.nw ? q.wb[w] : 0;
  out->score64 = host_objective(ts, es, T, E, ea, eb);
  return SCHED_OK;
  GUARD_END
}

int sched_dp_workspace_size(const sched_handle *hc, const sched_query *qin, size_t *bytes) {
  GUARD_BEGIN
  if (!hc || !bytes) return SCHED_E_INVALID;
  sched_handle *h = const_cast<sched_handle *>(hc);
  Query q;
  std::vector<unsigned char> blob;
  DevParams dp;
  int st = resolve_dp(h, qin, &q, &blob, &dp);
  if (st) return st;
  return dp_front_workspace(h->P, q, dp, bytes);
  GUARD_END
}

int sched_front_dp(sched_handle *h, const sched_query *qin, void *ws, size_t ws_bytes, void *stream,
                   sched_dp_point *best, sched_dp_point *front, uint64_t front_cap, uint64_t *n_front,
                   sched_stats *stats) {
  GUARD_BEGIN
  NvtxRange nvtx_range_("sched_front_dp");
  if (!h || !ws || !n_front || (front_cap > 0 && !front)) return SCHED_E_INVALID;
  int st = need_device();
  if (st) return st;
  Query q;
  std::vector<unsigned char> blob;
  DevParams dp;
  st = resolve_dp(h, qin, &q, &blob, &dp);
  if (st) return st;
  if (q.nw > 0 && !best) return SCHED_E_INVALID;
  std::vector<DpPoint> pts;
  int bpos[kMaxW];
  float ms = 0.f;
  int launches = 0;
  st = dp_front_run(h->P, q, dp, blob, ws, ws_bytes, stream, &pts, bpos, &ms, &launches);
  if (st) return st;
  double ts, es;
  host_constants(h->P, q, &ts, &es);
  auto fill = [&](const DpPoint &d, double score, sched_dp_point *o) {
    std::memset(o, 0, sizeof *o);
    o->valid = 1;
    o->makespan_s = d.t;
    o->energy_j = d.e;
    o->x64 = ts / d.t;
    o->y64 = es / d.e;
    o->score64 = score;
    o->n_groups = d.k;
    for (int i = 0; i < q.n; i++) {
      o->group_of[i] = d.group_of[i];
      o->level_of[i] = d.level_of[i];
    }
  };
  for (int w = 0; w < q.nw; w++) {
    if (pts.empty() || bpos[w] < 0) {
      std::memset(&best[w], 0, sizeof best[w]);
      continue;
    }
    const DpPoint &d = pts[bpos[w]];
    fill(d, host_objective(ts, es, d.t, d.e, q.wa[w], q.wb[w]), &best[w]);
  }
  *n_front = pts.size();
  if (pts.size() <= front_cap)
    for (size_t i = 0; i < pts.size(); i++) fill(pts[i], ts / pts[i].t, &front[i]);
  if (stats) {
    std::memset(stats, 0, sizeof *stats);
    stats->t_seq_s = ts;
    stats->e_seq_j = es;
    stats->search_ms = ms;
    stats->main_ms = ms;
    stats->total_ms = ms;
    stats->kernel_path = 4;
    stats->kernel_launches = launches;
    stats->h2d_bytes = blob.size();
  }
  if (pts.empty()) return SCHED_E_INFEASIBLE;
  if (pts.size() > front_cap) return SCHED_E_CAPACITY;
  return SCHED_OK;
  GUARD_END
}

int sched_heuristic(const sched_handle *hc, const sched_query *qin, int32_t priority, int32_t w,
                    int8_t *group_of, int8_t *level_of, uint64_t *index, sched_pick *out) {
  GUARD_BEGIN
  if (!hc || !group_of || !level_of || !index || !out || (priority != 0 && priority != 1))
    return SCHED_E_INVALID;
  sched_handle *h = const_cast<sched_handle *>(hc);
  Query q;
  const Space *sp;
  int st = resolve(h, qin, &q, &sp);
  if (st) return st;
  if (w < 0 || (q.nw > 0 && w >= q.nw) || (q.nw == 0 && w != 0)) return SCHED_E_INVALID;
  const Profile &P = h->P;
  const int n = q.n, top = q.L - 1, lvl = q.lev[top];
  // (1) ascending solo SM utilisation at 100 %, queue order on ties
  int order[kMaxN];
  for (int i = 0; i < n; i++) order[i] = i;
  std::stable_sort(order, order + n, [&](int x, int y) {
    return P.u[(size_t)x * P.lp + P.l100] < P.u[(size_t)y * P.lp + P.l100];
  });
  const int cap_clients = priority == 0 ? std::min(2, q.c) : q.c;
  int gpu_of[kMaxN], ng = 0, cnt[kMaxG] = {0};
  double util[kMaxG] = {0}, mem[kMaxG] = {0};
  for (int r = 0; r < n; r++) {
    const int i = order[r];
    const double ui = P.u[(size_t)i * P.lp + lvl], mi = P.mem[i];
    int pick = -1;
    for (int g = 0; g < ng && pick < 0; g++)  // (2) (3) (4)
      if (cnt[g] < cap_clients && util[g] + ui <= 1.0 && mem[g] + mi <= P.mem_cap) pick = g;
    if (pick < 0 && ng < q.g) pick = ng++;
    if (pick < 0) {  // no GPU keeps compute <= 100 %: least utilised one that fits (3) (4)
      for (int g = 0; g < ng; g++)
        if (cnt[g] < cap_clients && mem[g] + mi <= P.mem_cap && (pick < 0 || util[g] < util[pick])) pick = g;
    }
    if (pick < 0) return SCHED_E_INFEASIBLE;
    gpu_of[i] = pick;
    cnt[pick]++;
    util[pick] += ui;
    mem[pick] += mi;
  }
  // canonical RGS relabelling (groups by first member)
  int relabel[kMaxG];
  for (int g = 0; g < kMaxG; g++) relabel[g] = -1;
  int k = 0;
  int8_t a[kMaxN], dig[kMaxN];
  for (int i = 0; i < n; i++) {
    if (relabel[gpu_of[i]] < 0) relabel[gpu_of[i]] = k++;
    a[i] = (int8_t)relabel[gpu_of[i]];
  }
  const int nd = q.scope == SCHED_PER_CLIENT ? n : k;
  for (int d = 0; d < nd; d++) dig[d] = (int8_t)top;
  st = host_rank(*sp, a, dig, index);
  if (st) return st;
  for (int i = 0; i < n; i++) {
    group_of[i] = a[i];
    level_of[i] = (int8_t)top;
  }
  std::memset(out, 0, sizeof *out);
  out->index = *index;
  double T, E, ts, es;
  host_constants(P, q, &ts, &es);
  if (!host_score(P, q, a, k, dig, &T, &E)) return SCHED_OK;
  out->valid = 1;
  out->makespan_s = T;
  out->energy_j = E;
  out->x64 = ts / T;
  out->y64 = es / E;
  const int ea = q.nw ? q.wa[w] : 1, eb = q.nw ? q.wb[w] : 0;
  out->score64 = host_objective(ts, es, T, E, ea, eb);
  return SCHED_OK;
  GUARD_END
}

int sched_split_workspace_size(const sched_handle *hc, const sched_query *qin, const int32_t *tasks,
                               const int32_t *max_split, size_t *bytes, uint32_t *n_splits) {
  GUARD_BEGIN
  if (!bytes) return SCHED_E_INVALID;
  sched_handle *h = const_cast<sched_handle *>(hc);
  std::vector<std::vector<int>> svs;
  double tseq, eseq;
  int st = split_setup(h, qin, tasks, max_split, &svs, &tseq, &eseq);
  if (st) return st;
  size_t mx = 0;
  sched_handle tmp;
  for (const auto &sv : svs) {
    st = expand_split(h->P, qin->n, tasks, sv, &tmp.P);
    if (st) return st;
    tmp.sp_key[0] = -1;
    sched_query q2 = *qin;
    q2.n = tmp.P.n;
    size_t b = 0;
    st = sched_workspace_size(&tmp, &q2, &b);
    if (st) return st;
    mx = std::max(mx, b);
  }
  *bytes = mx;
  if (n_splits) *n_splits = (uint32_t)svs.size();
  return SCHED_OK;
  GUARD_END
}

int sched_search_splits(sched_handle *h, const sched_query *qin, const int32_t *tasks, const int32_t *max_split,
                        void *ws, size_t ws_bytes, void *stream, sched_split_pick *best,
                        sched_split_pick *pareto, uint64_t pareto_cap, uint64_t *n_pareto,
                        sched_stats *stats) {
  GUARD_BEGIN
  NvtxRange nvtx_range_("sched_search_splits");
  if (!ws) return SCHED_E_INVALID;
  int st = need_device();
  if (st) return st;
  std::vector<std::vector<int>> svs;
  double tseq, eseq;
  st = split_setup(h, qin, tasks, max_split, &svs, &tseq, &eseq);
  if (st) return st;
  const int nw = qin->n_weights, n = qin->n;
  const bool want_par = qin->want_pareto != 0;
  if (nw > 0 && !best) return SCHED_E_INVALID;
  if (want_par && (!n_pareto || (pareto_cap > 0 && !pareto))) return SCHED_E_INVALID;
  auto fill_split = [&](sched_split_pick *o, const sched_pick &pk, uint32_t r) {
    std::memset(o, 0, sizeof *o);
    o->pick = pk;
    o->split_rank = r;
    for (int i = 0; i < n; i++) o->n_clients += (o->split[i] = svs[r][i]);
  };
  std::vector<sched_split_pick> bst(std::max(nw, 1));
  for (auto &b : bst) std::memset(&b, 0, sizeof b);
  struct PP {
    double t, e;
    uint32_t r;
    uint64_t idx;
    sched_pick pk;
  };
  std::vector<PP> pts;
  sched_stats agg;
  std::memset(&agg, 0, sizeof agg);
  sched_handle tmp;
  std::vector<sched_pick> pb(std::max(nw, 1)), pp(4096);
  int rc = SCHED_OK;
  for (uint32_t r = 0; r < svs.size() && rc == SCHED_OK; r++) {
    st = expand_split(h->P, n, tasks, svs[r], &tmp.P);
    if (st) { rc = st; break; }
    tmp.P.tseq_base = tseq;
    tmp.P.eseq_base = eseq;
    tmp.sp_key[0] = -1;
    tmp.staged_ws = nullptr;
    sched_query q2 = *qin;
    q2.n = tmp.P.n;
    uint64_t np = 0;
    sched_stats s1;
    for (;;) {
      st = sched_search(&tmp, &q2, ws, ws_bytes, stream, pb.data(), pp.data(), pp.size(), &np, &s1);
      if (st == SCHED_E_CAPACITY && want_par && np > pp.size()) {
        pp.resize(np);
        continue;
      }
      break;
    }
    if (st && st != SCHED_E_INFEASIBLE) { rc = st; break; }
    agg.n_configs += s1.n_configs;
    agg.n_feasible += s1.n_feasible;
    agg.n_refined += s1.n_refined;
    agg.n_candidates += s1.n_candidates;
    agg.search_ms += s1.search_ms;
    agg.main_ms += s1.main_ms;
    agg.total_ms += s1.total_ms;
    agg.kernel_launches += s1.kernel_launches;
    agg.passes += s1.passes;
    agg.h2d_bytes += s1.h2d_bytes;
    agg.d2h_bytes += s1.d2h_bytes;
    agg.grid_ctas = std::max(agg.grid_ctas, s1.grid_ctas);
    agg.kernel_path = s1.kernel_path;
    if (st == SCHED_E_INFEASIBLE) continue;
    for (int w = 0; w < nw; w++) {
      const sched_pick &c = pb[w];
      if (!c.valid) continue;
      // ranks ascend: a later split replaces only on a strictly greater score
      if (!bst[w].pick.valid || c.score64 > bst[w].pick.score64) fill_split(&bst[w], c, r);
    }
    if (want_par)
      for (uint64_t k = 0; k < np; k++) pts.push_back({pp[k].makespan_s, pp[k].energy_j, r, pp[k].index, pp[k]});
  }
  if (tmp.pinned) cudaFreeHost(tmp.pinned);
  tmp.pinned = nullptr;
  if (rc) return rc;
  for (int w = 0; w < nw; w++) best[w] = bst[w];
  uint64_t nf = 0;
  if (want_par) {
    std::sort(pts.begin(), pts.end(), [](const PP &a, const PP &b) {
      if (a.t != b.t) return a.t < b.t;
      if (a.e != b.e) return a.e < b.e;
      if (a.r != b.r) return a.r < b.r;
      return a.idx < b.idx;
    });
    bool have = false;
    double bestE = 0.0;
    for (const PP &x : pts) {
      if (have && !(x.e < bestE)) continue;
      have = true;
      bestE = x.e;
      if (nf < pareto_cap) fill_split(&pareto[nf], x.pk, x.r);
      nf++;
    }
    *n_pareto = nf;
  } else if (n_pareto) {
    *n_pareto = 0;
  }
  if (stats) {
    *stats = agg;
    stats->t_seq_s = tseq;
    stats->e_seq_j = eseq;
  }
  if (want_par && nf > pareto_cap) return SCHED_E_CAPACITY;
  if (agg.n_feasible == 0) return SCHED_E_INFEASIBLE;
  return SCHED_OK;
  GUARD_END
}

const char *sched_strerror(int s) {
  switch (s) {
    case SCHED_OK: return "ok";
    case SCHED_E_INVALID: return "invalid argument";
    case SCHED_E_TOO_LARGE: return "space or tables too large";
    case SCHED_E_CUDA: return "CUDA runtime error";
    case SCHED_E_CAPACITY: return "capacity too small";
    case SCHED_E_INFEASIBLE: return "no feasible configuration";
    case SCHED_E_WORKSPACE: return "workspace too small or misaligned";
    case SCHED_E_NODEVICE: return "no CUDA device (no CPU fallback)";
    default: return "unknown status";
  }
}

const char *sched_version(void) { return "sched-b200 0.1 sm_100a"; }

}  // extern "C"
