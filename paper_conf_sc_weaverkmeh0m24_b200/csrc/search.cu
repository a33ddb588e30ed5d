// search.cu -- the exhaustive configuration search on sm_100a.
//
//   k_generic   any scope / L / G / C / weights: per-lane unrank + successor
//               walk, incremental fp32 group scoring, fp32 screens, fp64
//               canonical refine of near-best / possibly-Pareto configurations.
//   k_best_final, k_pareto_* : per-GPU finalize (exact best, exact Pareto).
//
// The method (PAPER.md L87 interference
// predicate + memory clause, L91, L96 metrics, L116 product metric) is
// evaluated in fp32 for every configuration; any configuration that could be
// the best for some weight (within the proven fp32 error margin delta_w of
// the running best) or could be on the Pareto front (not surely dominated by
// a verified point) is re-scored in fp64 in the canonical order, so the
// chosen indices and the Pareto set are bitwise those of the fp64 oracle.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>

#include "device_common.cuh"
#include "event_guard.hpp"
#include "finalize.hpp"
#include "tile_registry.hpp"

namespace sched {

__device__ __forceinline__ void decode_levels(const DevParams &p, const LaneCfg &c, int *lam) {
  const int nd = p.scope == SCHED_PER_CLIENT ? p.n : c.k;
  int dig[kMaxN];
  u64 x = c.v;
  if ((p.L & (p.L - 1)) == 0) {  // L = 1, 2, 4, 8: shifts (a u64 division is ~100 instructions)
    const int sh = __ffs(p.L) - 1;
    for (int d = nd - 1; d >= 0; d--) {
      dig[d] = (int)(x & (u64)(p.L - 1));
      x >>= sh;
    }
  } else if (x <= 0xffffffffull) {  // 32-bit division
    uint32_t y = (uint32_t)x;
    for (int d = nd - 1; d >= 0; d--) {
      dig[d] = (int)(y % (uint32_t)p.L);
      y /= (uint32_t)p.L;
    }
  } else {
    for (int d = nd - 1; d >= 0; d--) {
      dig[d] = (int)(x % (u64)p.L);
      x /= (u64)p.L;
    }
  }
  for (int i = 0; i < p.n; i++) lam[i] = p.scope == SCHED_PER_CLIENT ? dig[i] : dig[c.a[i]];
}

// fp32 score, normalised (hot-loop precision): T/T_seq and E/E_seq of the
// lane's configuration, per group U, B, D (members ascending), c_g, sigma_i,
// T_g = max_i t_i sigma_i c_g; T = max_g T_g, E = sum_g (P_s T_g + D_g) in
// group order.  Incremental over the successor walk: the per-group terms
// (T_g, P_s T_g + D_g, D_g) of the lane's current partition are cached and
// only the groups holding a client whose level changed (or every group after
// a partition change) are re-scored -- the same per-group operations and the
// same group-order combination as a from-scratch evaluation, hence the same
// fp32 values.
struct GroupCache {
  float t[kMaxG], e[kMaxG], d[kMaxG];
  int lam[kMaxN];
  bool valid;
};

__device__ __forceinline__ void score32_inc(const Tables &tb, const DevParams &p, const LaneCfg &c,
                                            const int *lam, GroupCache &gc, float &T, float &E) {
  uint32_t dirty = 0;
  if (!gc.valid) {
    dirty = c.k >= 32 ? 0xffffffffu : (1u << c.k) - 1;
  } else {
    for (int i = 0; i < p.n; i++)
      if (lam[i] != gc.lam[i]) dirty |= 1u << c.a[i];
  }
  for (uint32_t dd = dirty; dd; dd &= dd - 1) {
    const int g = __ffs(dd) - 1;
    const uint32_t m = c.mask[g];
    float U = 0.f, B = 0.f, D = 0.f;
    for (uint32_t mm = m; mm; mm &= mm - 1) {
      const int i = __ffs(mm) - 1, r = i * p.L + lam[i];
      U += tb.u[r];
      B += tb.bw[r];
      D += tb.dh[r];
    }
    const float cg = fmaxf(fmaxf(1.f, U), B);
    float Tg = 0.f;
    if (p.model & SCHED_MODEL_TIME_SLICE) {  // R30: sum of the solo slices (per-slice cap)
      for (uint32_t mm = m; mm; mm &= mm - 1) {
        const int r = (__ffs(mm) - 1) * p.L + lam[__ffs(mm) - 1];
        Tg += (p.model & SCHED_MODEL_POWER_CAP) ? fmaxf(tb.th[r], tb.dh[r] * p.kcap) : tb.th[r];
      }
    } else {
      for (uint32_t mm = m; mm; mm &= mm - 1) {
        const int i = __ffs(mm) - 1, ri = i * p.L + lam[i];
        float s = 1.f;
        for (uint32_t m2 = m & ~(1u << i); m2; m2 &= m2 - 1) s += tb.d[ri * p.ds + (__ffs(m2) - 1) * p.L + lam[__ffs(m2) - 1]];
        Tg = fmaxf(Tg, tb.th[ri] * s * cg);
      }
      if (p.model & SCHED_MODEL_POWER_CAP) Tg = fmaxf(Tg, D * p.kcap);  // R28
    }
    gc.t[g] = Tg;
    gc.e[g] = p.phat * Tg + D;
    gc.d[g] = D;
  }
  for (int i = 0; i < p.n; i++) gc.lam[i] = lam[i];
  gc.valid = true;
  T = 0.f;
  E = 0.f;
  float Dall = 0.f;
  for (int g = 0; g < c.k; g++) {
    T = fmaxf(T, gc.t[g]);
    E += gc.e[g];
    Dall += gc.d[g];
  }
  if (p.model & SCHED_MODEL_COUNT_IDLE) E = p.kidle * T + Dall;  // R26
}

__device__ __forceinline__ float proxy(float T, float E, int a, int b) {
  float q = 1.f;
  for (int i = 0; i < a; i++) q *= T;
  for (int i = 0; i < b; i++) q *= E;
  return q;
}

// ------------------------------------------------------------ generic kernel
constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;

__global__ void __launch_bounds__(kThreads) k_generic(const DevParams p) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned char *after = sm + ((p.blob_bytes + 15) & ~15u);
  Stair stair = stair_at(after);
  BestRec *red = (BestRec *)(after + kStairSmem);
  stair_init(stair);
  __syncthreads();
  u64 stair_ver = 0;

  float thr[kMaxW];
  BestRec lb[kMaxW];
#pragma unroll
  for (int w = 0; w < kMaxW; w++) {
    thr[w] = __int_as_float(0x7f800000);
    best_init(lb[w]);
  }
  u64 ncfg = 0, nfeas = 0, nref = 0;
  const int ul = p.unit_log2, cl = p.chunk_log2;
  LaneCfg c;
  int lam[kMaxN];
  GroupCache gc;

  for (;;) {
    u64 unit = 0;
    if (lane == 0) unit = atomicAdd(p.ctr + kCtrUnit, 1ull);
    unit = __shfl_sync(0xffffffffu, unit, 0);
    if (unit >= p.n_units) break;
    const u64 ue = unit * p.unit_stride;
    const u64 ch = p.first_chunk + (ue >> (cl - ul)) * (u64)p.shard_count;
    u64 s = (ch << cl) + ((ue & ((1ull << (cl - ul)) - 1)) << ul);
    u64 e = s + (1ull << ul);
    s = s > p.lo ? s : p.lo;
    e = e < p.hi ? e : p.hi;
    if (s >= e) continue;
    // refresh shared thresholds and the staircase
#pragma unroll
    for (int w = 0; w < kMaxW; w++)
      if (w < p.nw) thr[w] = fminf(thr[w], __uint_as_float(__ldcg(p.thr + w)));
    if (p.want_pareto) {
      stair_sync(stair, p, stair_ver, __ldcg(p.ctr + kCtrStairVer));
    }

    // lanes interleave (idx = s + lane + 32 j) or take contiguous runs
    const u64 run = p.lane_strided ? 0 : (e - s + 31) / 32;
    u64 idx = p.lane_strided ? s + lane : s + lane * run;
    const u64 lend = p.lane_strided ? e : (idx + run < e ? idx + run : e);
    const u64 step = p.lane_strided ? 32 : 1;
    if (idx < lend && dev_unrank(tb, p, idx, c)) {
      gc.valid = false;
      for (;;) {
        ncfg++;
        bool feas = c.feasible;
        if (feas && (p.model & SCHED_MODEL_NO_INTERFERENCE)) {  // level-dependent (R27)
          decode_levels(p, c, lam);
          feas = no_interference64(tb, p, c.mask, c.k, lam);
        }
        if (feas) {
          nfeas++;
          decode_levels(p, c, lam);
          float T, E;
          score32_inc(tb, p, c, lam, gc, T, E);
          bool need = false;
          unsigned wneed = 0;
#pragma unroll
          for (int w = 0; w < kMaxW; w++) {
            if (w < p.nw) {
              const float q = proxy(T, E, p.wa[w], p.wb[w]);
              thr[w] = fminf(thr[w], q);
              if (q <= thr[w] * (1.f + p.delta[w])) {
                need = true;
                wneed |= 1u << w;
              }
            }
          }
          bool par = false;
          if (p.want_pareto) {  // certified lower bound of the exact T (sound screen)
            par = !stair_dominated(stair, p, __dmul_rd((double)T, p.tlb_scale), E);
          }
          if (need || par) {
            nref++;
            double T64, E64;
            refine64(tb, p, c.mask, c.k, lam, &T64, &E64);
#pragma unroll
            for (int w = 0; w < kMaxW; w++) {
              if (wneed >> w & 1u) {
                const double F = objective64(p, T64, E64, p.wa[w], p.wb[w]);
                if (!lb[w].valid || better(F, idx, lb[w].f, lb[w].idx)) {
                  lb[w].f = F;
                  lb[w].idx = idx;
                  lb[w].t = T64;
                  lb[w].e = E64;
                  lb[w].t32 = T;
                  lb[w].e32 = E;
                  lb[w].valid = 1;
                }
              }
            }
            if (par && !stair_dominated(stair, p, T64, __double2float_rd(__ddiv_rd(E64, p.eseq))) &&
                !stair_dominated_exact(stair, p, T64, E64))
              emit_candidate(p, stair, idx, T64, E64, T, E);
          }
        }
        idx += step;
        if (idx >= lend) break;
        if (c.v + step >= c.Pn) gc.valid = false;  // the successor walk leaves the partition
        if (!dev_advance(tb, p, c, step)) break;
      }
    }
    __syncwarp();
    // publish thresholds (warp min, one atomic per weight)
#pragma unroll
    for (int w = 0; w < kMaxW; w++) {
      if (w < p.nw) {
        float t = thr[w];
#pragma unroll
        for (int o = 16; o; o >>= 1) t = fminf(t, __shfl_xor_sync(0xffffffffu, t, o));
        thr[w] = t;
        if (lane == 0 && t < __uint_as_float(__ldcg(p.thr + w))) atomicMin(p.thr + w, __float_as_uint(t));
      }
    }
  }
  // ---- reductions: counters, per-CTA best slots ----
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    ncfg += __shfl_xor_sync(0xffffffffu, ncfg, o);
    nfeas += __shfl_xor_sync(0xffffffffu, nfeas, o);
    nref += __shfl_xor_sync(0xffffffffu, nref, o);
  }
  if (lane == 0) {
    atomicAdd(p.ctr + kCtrConfigs, ncfg);
    atomicAdd(p.ctr + kCtrFeasible, nfeas);
    atomicAdd(p.ctr + kCtrRefined, nref);
  }
#pragma unroll
  for (int w = 0; w < kMaxW; w++) {
    if (w < p.nw) {
      warp_best(lb[w]);
      if (lane == 0) red[warp * kMaxW + w] = lb[w];
    }
  }
  __syncthreads();
  if (threadIdx.x < p.nw) {
    const int w = threadIdx.x;
    BestRec b = red[w];
    for (int k = 1; k < kWarps; k++) {
      const BestRec x = red[k * kMaxW + w];
      if (x.valid && (!b.valid || better(x.f, x.idx, b.f, b.idx))) b = x;
    }
    ((BestRec *)p.slots)[(size_t)blockIdx.x * p.nw + w] = b;
  }
}

// ------------------------------------------------------------ group table
// Every (group mask, level) tuple of the query, once per search: fp32
// normalised T_g, E_g and the exact fp64 T_g (t32 = +inf: memory-infeasible
// or more than C members).  L2-resident; replaces per-partition evaluation.
__global__ void __launch_bounds__(256) k_groups(const DevParams p, GroupRec *gtab) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  const unsigned long long total = (unsigned long long)p.L << p.n;
  for (unsigned long long id = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x; id < total;
       id += (unsigned long long)gridDim.x * blockDim.x) {
    const uint32_t m = (uint32_t)(id / p.L);
    const int mu = (int)(id % p.L);
    GroupRec r, x;
    r.t32 = __int_as_float(0x7f800000);
    r.e32 = 0.f;
    r.t64 = __longlong_as_double(0x7ff0000000000000ll);
    r.e64 = 0.0;
    if (m != 0 && __popc(m) <= p.c) {
      long long M = 0;
      for (uint32_t mm = m; mm; mm &= mm - 1) M += tb.mem[__ffs(mm) - 1];
      if (M <= (long long)p.mem_cap && group_eval(tb, p, m, mu, x.t32, x.e32, x.t64, x.e64)) r = x;
    }
    gtab[id] = r;
  }
}

// ------------------------------------------------------------ init / finalize
// keep = 0: fresh search; 1: seeded re-run after overflow (keep staircase +
// thresholds, drop candidates); 2: after the seed pass (keep staircase,
// thresholds and the seed pass's in-range candidates); 3: after the seed pass
// with a new staircase bucketing (keep thresholds and candidates, reset the
// staircase, which k_rebucket then rebuilds from the candidates).
__global__ void k_init(const DevParams p, int keep) {
  const int t = threadIdx.x;
  const bool kept = keep && (t == kCtrStairVer || t == kCtrPass ||
                             (keep >= 2 && (t == kCtrCand || t == kCtrOverflow)));
  if (t < kCtrN && !kept) p.ctr[t] = 0ull;
  if (keep != 2)  // a fresh log (re-run: its slot ids are rewritten by k_reseed)
    for (int i = t; i < kLog; i += blockDim.x) ((LogEnt *)p.stlog)[i].tag = 0u;
  if ((keep == 1 || keep == 3) && t == kCtrStairVer) p.ctr[t] = (unsigned long long)kLog + 1;  // full merge
  if (keep == 1 || keep == 2) return;
  if (t < kMaxW && keep == 0) p.thr[t] = 0x7f800000u;
  for (int i = t; i < kBuckets; i += blockDim.x) {
    p.stv[i] = 0x7f800000u;
    p.stp[i] = ~0ull;
    p.ste[i] = ~0ull;
  }
}

// Span of the verified points after the seed pass: out[0] = min T, out[1] =
// the T of the lowest-energy point (the front's two ends).  One block.
__global__ void __launch_bounds__(1024) k_stair_span(const DevParams p, int ncand, double *out) {
  __shared__ double s_t[1024], s_e[1024], s_te[1024];
  double tlo = __longlong_as_double(0x7ff0000000000000ll), emin = tlo, temin = tlo;
  for (int i = threadIdx.x; i < ncand; i += blockDim.x) {
    const CandRec c = ((const CandRec *)p.cand)[i];
    tlo = fmin(tlo, c.t);
    if (c.e < emin || (c.e == emin && c.t < temin)) {
      emin = c.e;
      temin = c.t;
    }
  }
  s_t[threadIdx.x] = tlo;
  s_e[threadIdx.x] = emin;
  s_te[threadIdx.x] = temin;
  __syncthreads();
  for (int o = 512; o; o >>= 1) {
    if (threadIdx.x < o) {
      const int q = threadIdx.x + o;
      s_t[threadIdx.x] = fmin(s_t[threadIdx.x], s_t[q]);
      if (s_e[q] < s_e[threadIdx.x] || (s_e[q] == s_e[threadIdx.x] && s_te[q] < s_te[threadIdx.x])) {
        s_e[threadIdx.x] = s_e[q];
        s_te[threadIdx.x] = s_te[q];
      }
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    out[0] = s_t[0];
    out[1] = s_te[0];
  }
}

// Re-insert the seed pass's candidate records into the staircase under the
// new bucketing (same values as emit_candidate).
__global__ void k_rebucket(const DevParams p, int ncand) {
  const double g1 = 1.0 + (double)p.gamma;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < ncand; i += gridDim.x * blockDim.x) {
    const CandRec c = ((const CandRec *)p.cand)[i];
    const unsigned int vb = __float_as_uint(__double2float_ru(__dmul_ru(__ddiv_ru(c.e, p.eseq), g1)));
    const int jb = bucket_of(c.t, p);
    atomicMin(p.stv + jb, vb);
    atomicMin(p.stp + jb, ((unsigned long long)vb << 32) | (unsigned int)i);
    atomicMin(p.ste + jb, (unsigned long long)__double_as_longlong(c.e));
  }
}

// Before a seeded re-run: keep only the candidate records the same-bucket
// staircase references (compacted to slots 0..m-1, ids rewritten), so the
// re-run's candidate buffer starts with them.  One block of 1024 threads.
__global__ void __launch_bounds__(1024) k_reseed(const DevParams p, CandRec *tmp) {
  __shared__ unsigned int cnt[1024];
  constexpr int K = kBuckets / 1024;
  const int t = threadIdx.x;
  unsigned int mine = 0;
  for (int k = 0; k < K; k++) {
    const int j = t * K + k;
    const unsigned long long x = p.stp[j];
    if (x != ~0ull) {
      tmp[j] = ((const CandRec *)p.cand)[(unsigned int)x];
      mine++;
    }
  }
  cnt[t] = mine;
  __syncthreads();
  for (int o = 1; o < 1024; o <<= 1) {  // inclusive scan
    const unsigned int v = t >= o ? cnt[t - o] : 0u;
    __syncthreads();
    cnt[t] += v;
    __syncthreads();
  }
  unsigned int slot = cnt[t] - mine;
  for (int k = 0; k < K; k++) {
    const int j = t * K + k;
    const unsigned long long x = p.stp[j];
    if (x != ~0ull) {
      ((CandRec *)p.cand)[slot] = tmp[j];
      p.stp[j] = (x & 0xffffffff00000000ull) | slot;
      slot++;
    }
  }
  __threadfence();
  if (t == 1023) p.ctr[kCtrCand] = cnt[1023];
}

// best per weight over the per-CTA slots -> out[0 .. W)
__global__ void k_best_final(const DevParams p, int nslots) {
  __shared__ BestRec red[32];
  const int w = blockIdx.x, lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  BestRec b;
  best_init(b);
  for (int s = threadIdx.x; s < nslots; s += blockDim.x) {
    const BestRec x = ((const BestRec *)p.slots)[(size_t)s * p.nw + w];
    if (x.valid && (!b.valid || better(x.f, x.idx, b.f, b.idx))) b = x;
  }
  warp_best(b);
  if (lane == 0) red[warp] = b;
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int k = 1; k < (int)(blockDim.x >> 5); k++) {
      const BestRec x = red[k];
      if (x.valid && (!b.valid || better(x.f, x.idx, b.f, b.idx))) b = x;
    }
    ((BestRec *)p.out)[w] = b;
  }
}

// Pareto finalize, stage 1: drop candidates surely (strictly) dominated by a
// verified point of the final global staircase; compact survivors.
__global__ void k_pareto_prefilter(const DevParams p, int ncand, unsigned int *surv) {
  __shared__ unsigned int s_pm[kBuckets];
  __shared__ unsigned long long s_bp[kBuckets], s_pe[kBuckets];
  Stair stair{s_pm, s_bp, s_pe};
  stair_init(stair);
  __syncthreads();
  if (threadIdx.x < 32) stair_merge(stair, p);
  __syncthreads();
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < ncand; i += gridDim.x * blockDim.x) {
    const CandRec c = ((const CandRec *)p.cand)[i];
    const bool dom = stair_dominated(stair, p, c.t, __double2float_rd(__ddiv_rd(c.e, p.eseq))) ||
                     stair_dominated_exact(stair, p, c.t, c.e);
    if (!dom) {
      const unsigned int k = (unsigned int)atomicAdd(p.ctr + kCtrSurv, 1ull);
      surv[k] = (unsigned int)i;
    }
  }
}


// ------------------------------------------------------------ launcher
namespace {
// SCHED_KERNEL=generic|tile|dfs|sfx|ctile|ctile2 restricts the kernel choice (testing and
// measurement of the individual paths); unset = the fastest eligible path.
bool want_path(int path) {
  static const char *names[] = {"generic", "tile", "dfs", "sfx", "dp", "ctile", "ctile2"};
  const char *e = std::getenv("SCHED_KERNEL");
  if (!e || !*e) return true;
  return std::strcmp(e, names[path]) == 0;
}

// seed pass: nsm x 128 sampled units of 2^10 configurations (SCHED_SEED_UNITS_PER_SM,
// SCHED_SEED_UNIT_LOG2 override; tools/seed_sweep.py): vs the earlier 64 x 2^12 the
// critical path of the seed launch is shorter (c4 bench step at 8 ranks 88.2 -> 86.4 ms)
// with half the Pareto candidates
int seed_units_per_sm() {
  const char *e = std::getenv("SCHED_SEED_UNITS_PER_SM");
  const int v = e && *e ? std::atoi(e) : 128;
  return v < 1 ? 1 : (v > 1024 ? 1024 : v);
}

int seed_unit_log2() {
  const char *e = std::getenv("SCHED_SEED_UNIT_LOG2");
  const int v = e && *e ? std::atoi(e) : 10;
  return v < 8 ? 8 : (v > 12 ? 12 : v);
}

constexpr int kMaxGrid = 4096;
constexpr int kFrontCap = 1 << 16;

struct WsLayout {
  size_t ctr, thr, stv, stp, ste, stlog, blob, slots, cand, surv, fin, out, gtab, params, c2t64, total;
};

WsLayout layout(const DevParams &dp) {
  WsLayout L;
  size_t o = 0;
  auto take = [&](size_t b) {
    o = (o + 255) / 256 * 256;
    size_t r = o;
    o += b;
    return r;
  };
  L.ctr = take(8 * kCtrN);
  L.thr = take(4 * kMaxW);
  L.stv = take(4 * kBuckets);
  L.stp = take(8 * kBuckets);
  L.ste = take(8 * kBuckets);
  L.stlog = take(sizeof(LogEnt) * kLog);
  L.blob = take(dp.blob_bytes);
  L.slots = take(sizeof(BestRec) * kMaxW * (size_t)kMaxGrid);
  L.cand = take(sizeof(CandRec) * (size_t)dp.cand_cap);
  L.surv = take(4 * (size_t)dp.cand_cap);
  L.fin = take(finalize_bytes(dp.cand_cap));
  L.params = take(sizeof(DevParams));
  {  // per-warp fp64 T tables of the group-table PER_CLIENT kernel (only when it runs)
    DevParams tmp = dp;
    TileLaunch tl;
    L.c2t64 = take(ctile2_eligible(tmp, &tl) && dp.want_pareto ? ctile2_t64_bytes() : 0);
  }
  L.out = take(sizeof(BestRec) * kMaxW + sizeof(CandRec) * (size_t)kFrontCap);
  L.gtab = take(dp.gtab_ok ? sizeof(GroupRec) * ((size_t)dp.L << dp.n) : 0);
  L.total = (o + 255) / 256 * 256;
  return L;
}
}  // namespace

size_t workspace_bytes(const DevParams &dp, int) { return layout(dp).total; }

#define CK(x)                                   \
  do {                                          \
    cudaError_t e_ = (x);                       \
    if (e_ != cudaSuccess) return SCHED_E_CUDA; \
  } while (0)

int stage_tables(const DevParams &dp, const std::vector<unsigned char> &blob, void *d_ws, void *host_pinned,
                 void *stream) {
  const WsLayout L = layout(dp);
  cudaStream_t st = (cudaStream_t)stream;
  unsigned char *ws = (unsigned char *)d_ws;
  const void *src = blob.data();
  if (host_pinned) {
    std::memcpy(host_pinned, blob.data(), blob.size());
    src = host_pinned;
  }
  CK(cudaMemcpyAsync(ws + L.blob, src, blob.size(), cudaMemcpyHostToDevice, st));
  return SCHED_OK;
}

// device unrank (+ successor walk) of a batch of indices (sched_unrank_device)
__global__ void __launch_bounds__(256) k_unrank(const DevParams p, const u64 *idx, u64 n, u64 advance,
                                                int8_t *gout, int8_t *lout) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  for (u64 t = blockIdx.x * (u64)blockDim.x + threadIdx.x; t < n; t += (u64)gridDim.x * blockDim.x) {
    int8_t *g = gout + t * p.n, *l = lout + t * p.n;
    const u64 i0 = idx[t];
    LaneCfg c;
    if (i0 >= tb.W[p.root] || !dev_unrank(tb, p, i0, c) || (advance && !dev_advance(tb, p, c, advance))) {
      g[0] = -1;
      continue;
    }
    // level digits of residue v, base L, most significant = client 0 / group 0
    const int nd = p.scope == SCHED_PER_CLIENT ? p.n : c.k;
    int8_t dig[kMaxN];
    u64 v = c.v;
    for (int d = nd - 1; d >= 0; d--) {
      dig[d] = (int8_t)(v % (u64)p.L);
      v /= (u64)p.L;
    }
    for (int i = 0; i < p.n; i++) {
      g[i] = c.a[i];
      l[i] = p.scope == SCHED_PER_CLIENT ? dig[i] : dig[c.a[i]];
    }
  }
}

int launch_unrank(DevParams dp, void *d_ws, size_t ws_bytes, void *stream, const uint64_t *d_idx, uint64_t n,
                  uint64_t advance, int8_t *gout, int8_t *lout) {
  const WsLayout L = layout(dp);
  if (ws_bytes < L.total || ((uintptr_t)d_ws & 255)) return SCHED_E_WORKSPACE;
  if (n == 0) return SCHED_OK;
  unsigned char *ws = (unsigned char *)d_ws;
  cudaStream_t st = (cudaStream_t)stream;
  dp.blob = ws + L.blob;
  const size_t smem = (dp.blob_bytes + 15) & ~15u;
  CK(cudaFuncSetAttribute(k_unrank, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int dev = 0, nsm = 0;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  const int grid = (int)std::min<uint64_t>((n + 255) / 256, (uint64_t)nsm * 4);
  k_unrank<<<grid, 256, smem, st>>>(dp, (const u64 *)d_idx, n, advance, gout, lout);
  CK(cudaGetLastError());
  return SCHED_OK;
}

int launch_search(DevParams dp, void *d_ws, size_t ws_bytes, void *stream, LaunchInfo *info,
                  std::vector<BestRec> *best, std::vector<CandRec> *pareto, uint64_t *ctr_out) {
  const WsLayout L = layout(dp);
  if (ws_bytes < L.total || ((uintptr_t)d_ws & 255)) return SCHED_E_WORKSPACE;
  unsigned char *ws = (unsigned char *)d_ws;
  cudaStream_t st = (cudaStream_t)stream;
  dp.blob = ws + L.blob;
  dp.ctr = (unsigned long long *)(ws + L.ctr);
  dp.thr = (unsigned int *)(ws + L.thr);
  dp.stv = (unsigned int *)(ws + L.stv);
  dp.stp = (unsigned long long *)(ws + L.stp);
  dp.ste = (unsigned long long *)(ws + L.ste);
  dp.stlog = ws + L.stlog;
  dp.slots = ws + L.slots;
  dp.cand = ws + L.cand;
  dp.out = ws + L.out;
  dp.gtab = dp.gtab_ok ? ws + L.gtab : nullptr;
  dp.gp = (const DevParams *)(ws + L.params);
  dp.c2t64 = (double *)(ws + L.c2t64);
  int dev = 0, nsm = 0;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));

  EventGuard<3> ev;  // destroyed on every return path
  if (!ev.create()) return SCHED_E_CUDA;
  cudaEvent_t e0 = ev[0], e1 = ev[1], e2 = ev[2];
  CK(cudaEventRecord(e0, st));
  int grid = 0, path = 0, launches = 0, passes = 0;
  uint64_t d2h = 0;
  float search_ms = 0.f;
  uint64_t ctr[kCtrN];
  // pass 0 from an empty staircase; on candidate-buffer overflow, pass 1
  // re-runs seeded with pass 0's final staircase and thresholds (sound).
  // pass 0: seed pass over a sample of in-range units (2^10 configs each,
  // spread over the shard) that fills the staircase and thresholds; pass 1:
  // the full search; pass 2 only after a candidate-buffer overflow.
  if (dp.gtab_ok) {  // group-tuple table (part of the search: counted in search_ms)
    const size_t gsm = (dp.blob_bytes + 15) & ~15u;
    CK(cudaFuncSetAttribute(k_groups, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)gsm));
    const unsigned long long tot = (unsigned long long)dp.L << dp.n;
    const int gb = (int)std::min<unsigned long long>((tot + 255) / 256, (unsigned long long)nsm * 8);
    CK(cudaEventRecord(e1, st));
    k_groups<<<gb, 256, gsm, st>>>(dp, (GroupRec *)(ws + L.gtab));
    CK(cudaGetLastError());
    CK(cudaEventRecord(e2, st));
    CK(cudaStreamSynchronize(st));
    float gms = 0.f;
    CK(cudaEventElapsedTime(&gms, e1, e2));
    search_ms += gms;
    launches++;
  }
  DevParams dp_full = dp;
  const char *noseed = std::getenv("SCHED_NO_SEED");  // measurement: no seed pass
  const bool seed = !(noseed && noseed[0] == '1') && dp.want_pareto && dp.n_owned > 0 && dp.chunk_log2 >= 12 &&
                    (dp.n_owned << (dp.chunk_log2 - 12)) >= ((uint64_t)1 << 20);  // >= 2^32 configs
  // passes: 0 seed (large searches), 1 full search, 2 re-run after a
  // candidate-buffer overflow (unseeded: re-bucketed to the overflowing
  // pass's front span with a fresh staircase; seeded: reseeded staircase),
  // 3 reseeded re-run if 2 overflowed as well
  for (int pass = seed ? 0 : 1; pass < 4; pass++) {
    dp = dp_full;
    if (pass == 0) {
      const int sl = seed_unit_log2();
      const uint64_t u12 = dp.n_owned << (dp.chunk_log2 - sl);
      dp.unit_log2 = sl;
      dp.n_units = (uint64_t)nsm * seed_units_per_sm();
      dp.unit_stride = u12 / dp.n_units;
    }
    passes++;
    int keep = pass == 0 ? 0 : (pass == 1 ? (seed ? 2 : 0) : 1);
    // pass 2 (after an overflow): re-bucketed to the overflowing pass's
    // candidate span with a fresh staircase -- a dense front flooded coarse
    // buckets, or (seeded) the seed's front missed the region the flood came
    // from and its fine buckets clamped it
    const bool span_rerun = pass == 2 && dp.want_pareto;
    // passes 1 and 2 stop early once they overflow (they are re-run); the
    // seed pass and the last re-run go to the end
    dp.abort_ovf = (pass == 1 || pass == 2) ? 1 : 0;
    const int ncand0 = (pass == 1 && seed && dp.want_pareto) || span_rerun
                           ? (int)std::min<uint64_t>(ctr[kCtrCand], dp.cand_cap) : 0;
    if (ncand0 > 0) {
      // Re-bucket the staircase to the span of the seed pass's front: about
      // 1024 buckets between its lowest T and the T of its lowest-E point,
      // so that front points closer than the default 2^-7 relative bucket
      // width are screened exactly (dense local fronts of index windows).
      double span[2];
      k_stair_span<<<1, 1024, 0, st>>>(dp, ncand0, (double *)dp.out);
      CK(cudaGetLastError());
      CK(cudaMemcpyAsync(span, dp.out, sizeof span, cudaMemcpyDeviceToHost, st));
      CK(cudaStreamSynchronize(st));
      launches++;
      d2h += sizeof span;
      if (span[0] > 0.0 && span[1] >= span[0] && std::isfinite(span[1])) {
        const double binades = std::log2(span[1] / span[0]);
        int sh = (int)std::ceil(52.0 - std::log2(1024.0 / std::max(binades, 1e-9)));
        sh = std::max(kBucketShiftMin, std::min(kBucketShift, sh));
        uint64_t b;
        std::memcpy(&b, &span[0], 8);
        const int64_t base = (int64_t)(b >> sh) - 512;
        set_buckets(dp_full, sh, (uint32_t)std::max<int64_t>(0, base));
        set_buckets(dp, sh, dp_full.bucket_base);
        keep = span_rerun ? 0 : 3;   // the re-run starts a fresh staircase in the finer buckets
      }
    }
    k_init<<<1, 256, 0, st>>>(dp, keep);
    CK(cudaGetLastError());
    launches++;
    if (keep == 3) {
      k_rebucket<<<std::max(1, std::min(4 * nsm, (ncand0 + 255) / 256)), 256, 0, st>>>(dp, ncand0);
      CK(cudaGetLastError());
      launches++;
    }
    if (pass >= 2 && keep == 1 && dp.want_pareto) {
      k_reseed<<<1, 1024, 0, st>>>(dp, (CandRec *)dp.out);
      CK(cudaGetLastError());
      launches++;
    }
    TileLaunch tl;
    if (want_path(1) && tile_eligible(dp, &tl)) {
      path = 1;
      CK(launch_tile(dp, tl, nsm, st, e1, e2, &grid, pass == 0));
    } else if (want_path(6) && ctile2_eligible(dp, &tl)) {
      path = 6;
      CK(launch_ctile2(dp, tl, nsm, st, e1, e2, &grid, pass == 0));
    } else if (want_path(5) && ctile_eligible(dp, &tl)) {
      path = 5;
      CK(launch_ctile(dp, tl, nsm, st, e1, e2, &grid, pass == 0));
    } else if (want_path(3) && sfx_eligible(dp, &tl)) {
      path = 3;
      CK(launch_sfx(dp, tl, nsm, st, e1, e2, &grid, pass == 0));
    } else if (want_path(2) && dfs_eligible(dp, &tl)) {
      path = 2;
      CK(launch_dfs(dp, tl, nsm, st, e1, e2, &grid, pass == 0));
    } else {
      const size_t smem = ((dp.blob_bytes + 15) & ~15u) + kStairSmem + sizeof(BestRec) * kWarps * kMaxW;
      CK(cudaFuncSetAttribute(k_generic, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
      int occ = 0;
      CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_generic, kThreads, smem));
      if (occ < 1) return SCHED_E_TOO_LARGE;
      grid = std::min(kMaxGrid, nsm * occ);
      CK(publish_params(dp, st));
      CK(cudaEventRecord(e1, st));
      k_generic<<<grid, kThreads, smem, st>>>(dp);
      CK(cudaGetLastError());
      CK(cudaEventRecord(e2, st));
    }
    launches++;
    if (dp.nw > 0) {
      k_best_final<<<dp.nw, 256, 0, st>>>(dp, grid * (path == 3 ? tl.slots_per_cta : 1));
      CK(cudaGetLastError());
      launches++;
    }
    CK(cudaMemcpyAsync(ctr, dp.ctr, sizeof ctr, cudaMemcpyDeviceToHost, st));
    d2h += sizeof ctr;
    CK(cudaStreamSynchronize(st));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, e1, e2));
    search_ms += ms;
    info->main_ms = ms;  // the last pass run is the full pass the result comes from
    if (pass >= 1 && !ctr[kCtrOverflow]) break;
  }
  int ncand = (int)std::min<uint64_t>(ctr[kCtrCand], dp.cand_cap);
  if (dp.want_pareto && ncand > 0) {
    // exact front: staircase prefilter, then sort + sweep (finalize.cu)
    unsigned int *surv = (unsigned int *)(ws + L.surv);
    k_pareto_prefilter<<<std::max(1, std::min(4 * nsm, (ncand + 255) / 256)), 256, 0, st>>>(dp, ncand, surv);
    CK(cudaGetLastError());
    launches++;
    unsigned long long nsurv = 0;
    CK(cudaMemcpyAsync(&nsurv, dp.ctr + kCtrSurv, sizeof nsurv, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    d2h += sizeof nsurv;
    CK(finalize_front(dp, ws + L.fin, finalize_bytes(dp.cand_cap), surv, (int)nsurv, kFrontCap, nsm, st, &launches));
  }
  CK(cudaMemcpyAsync(ctr, dp.ctr, sizeof ctr, cudaMemcpyDeviceToHost, st));
  best->resize(kMaxW);
  CK(cudaMemcpyAsync(best->data(), dp.out, sizeof(BestRec) * kMaxW, cudaMemcpyDeviceToHost, st));
  d2h += sizeof ctr + sizeof(BestRec) * kMaxW;
  CK(cudaStreamSynchronize(st));
  const uint64_t nfront = dp.want_pareto && ncand > 0 ? ctr[kCtrFront] : 0;
  pareto->resize(std::min<uint64_t>(nfront, kFrontCap));
  if (!pareto->empty()) {
    CK(cudaMemcpyAsync(pareto->data(), dp.out + sizeof(BestRec) * kMaxW, sizeof(CandRec) * pareto->size(),
                       cudaMemcpyDeviceToHost, st));
    d2h += sizeof(CandRec) * pareto->size();
    CK(cudaStreamSynchronize(st));
  }
  info->search_ms = search_ms;
  info->grid = grid;
  info->path = path;
  info->launches = launches;
  info->passes = passes;
  info->d2h_bytes = d2h;
  for (int k = 0; k < kCtrN; k++) ctr_out[k] = ctr[k];
  ctr_out[kCtrFront] = nfront;
  if (nfront > kFrontCap) return SCHED_E_CAPACITY;
  return SCHED_OK;
}

}  // namespace sched
