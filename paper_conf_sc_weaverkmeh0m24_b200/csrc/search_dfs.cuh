// search_dfs.cuh -- L = 1 partition kernel (c5 fast path).
//
// With one MPS level every configuration is a set partition (RGS).  Each
// lane walks a contiguous index range.  A *parent* is the partition of
// workflows 0..n-2; its leaves are the admissible groups for workflow
// x = n-1 (existing groups with room, ascending, then a new group), which
// are consecutive indices.  The lane keeps per-group fp32 sums of the parent
// (U, B, D, memory, member slowdown partials sigma_i, T_g, E_g) in local
// memory, recomputing only the groups the lexicographic successor changed.
// A leaf costs one incremental group update (<= C members):
//   U' = U_j + u_x, B' = B_j + bw_x, c' = max(1, U', B')
//   tau_i = t_i (sigma_i + d[i][x]) c', tau_x = t_x (1 + sum_i d[x][i]) c'
//   T = max(max_{g != j} T_g, max tau), E = E_all - E_j + (P_s T'_j + D_j + dyn_x)
// (all terms >= 0 and E' >= E_j, so the subtraction keeps the relative error
// bound of DESIGN.md section 5).  Per parent the proxies and (T, E) are
// min-reduced over its leaves and screened once; a parent that is not
// cleared re-checks its leaves one by one with the fp64 refine.
#pragma once
#include "device_common.cuh"
#include "search_tile.cuh"

namespace sched {

constexpr int kDfsMaxC = 4;
constexpr int kDfsMaxG = 8;
constexpr int kDfsThreads = 256;

struct DGroup {
  float U, B, D, T, E;
  int M;
  float sig[kDfsMaxC];
  int mem[kDfsMaxC];  // member workflow ids (ascending), -1 = empty
};

struct DfsLane {
  LaneCfg cfg;        // RGS of the parent in elements 0..n-2 (element n-1 unplaced)
  DGroup g[kDfsMaxG];
};

__device__ __forceinline__ void dgroup_eval(const Tables &tb, const DevParams &p, uint32_t m, DGroup &G) {
  float U = 0.f, B = 0.f, D = 0.f;
  int M = 0, c = 0;
  for (uint32_t mm = m; mm; mm &= mm - 1) {
    const int i = __ffs(mm) - 1;
    U += tb.u[i];
    B += tb.bw[i];
    D += tb.dh[i];
    M += tb.mem[i];
    G.mem[c++] = i;
  }
  for (int q = c; q < kDfsMaxC; q++) G.mem[q] = -1;
  const float cg = fmaxf(fmaxf(1.f, U), B);
  float T = 0.f;
  for (int a = 0; a < c; a++) {
    const int i = G.mem[a];
    float s = 1.f;
    for (int b = 0; b < c; b++)
      if (b != a) s += tb.d[i * p.ds + G.mem[b]];
    G.sig[a] = s;
    T = fmaxf(T, tb.th[i] * s * cg);
  }
  G.U = U;
  G.B = B;
  G.D = D;
  G.M = M;
  G.T = T;
  G.E = p.phat * T + D;
}

// successor of the parent RGS (positions 1..n-2), keeping workflow n-1
// placeable (W > 0 in the DP table); greedy fill up to n-2.
__device__ __forceinline__ bool dfs_parent_successor(const Tables &tb, const DevParams &p, LaneCfg &c) {
  const int last = p.n - 2;
  for (int i = last; i >= 1; i--) {
    const int j0 = c.a[i];
    c.mask[j0] &= ~(1u << i);
    if (--c.sz[j0] == 0) c.k--;
    const int s = c.st[i - 1];
    for (int j = j0 + 1; j <= c.k; j++) {
      const int col = col_for(p, j, c.k, c.sz);
      if (col < 0) {
        if (j == c.k) break;
        continue;
      }
      const uint16_t s2 = tb.trans[s * p.tc + col];
      if (s2 == kNoState || tb.W[s2] == 0) continue;
      place(c, i, j);
      c.st[i] = s2;
      for (int m = i + 1; m <= last; m++) {
        const int sm = c.st[m - 1];
        for (int jj = 0; jj <= c.k; jj++) {
          const int cl = col_for(p, jj, c.k, c.sz);
          if (cl < 0) {
            if (jj == c.k) break;
            continue;
          }
          const uint16_t t2 = tb.trans[sm * p.tc + cl];
          if (t2 == kNoState || tb.W[t2] == 0) continue;
          place(c, m, jj);
          c.st[m] = t2;
          break;
        }
      }
      return true;
    }
  }
  return false;
}

// leaf of the parent: workflow x joins group j (j == k: a new group).
// Returns false if memory-infeasible.
__device__ __forceinline__ bool dfs_leaf(const Tables &tb, const DevParams &p, const DfsLane &L, int j, int x,
                                         float Tex, float Eall, float &T, float &E) {
  const int k = L.cfg.k;
  if (j == k) {
    if (tb.mem[x] > p.mem_cap) return false;
    const float tn = tb.th[x] * fmaxf(fmaxf(1.f, tb.u[x]), tb.bw[x]);
    T = fmaxf(Tex, tn);
    E = Eall + (p.phat * tn + tb.dh[x]);
    return true;
  }
  const DGroup &G = L.g[j];
  if (G.M + tb.mem[x] > p.mem_cap) return false;
  const float U = G.U + tb.u[x], B = G.B + tb.bw[x];
  const float cg = fmaxf(fmaxf(1.f, U), B);
  float sx = 1.f, tmax = 0.f;
#pragma unroll
  for (int a = 0; a < kDfsMaxC; a++) {
    const int i = G.mem[a];
    if (i >= 0) {
      sx += tb.d[x * p.ds + i];
      tmax = fmaxf(tmax, tb.th[i] * (G.sig[a] + tb.d[i * p.ds + x]));
    }
  }
  tmax = fmaxf(tmax, tb.th[x] * sx);
  const float Tj = tmax * cg;
  T = fmaxf(Tex, Tj);
  E = (Eall - G.E) + (p.phat * Tj + (G.D + tb.dh[x]));
  return true;
}

template <class WS>
__device__ __noinline__ int dfs_slow(const Tables &tb, const DevParams &p, const Stair &stair, DfsLane &L,
                                     const Thr<WS> thr, BestRec *lb, u64 base, int o0, int o1, float T1,
                                     int j1, float T2, float Eall) {
  const int x = p.n - 1, k = L.cfg.k;
  int nref = 0, ord = 0;
  for (int j = 0; j <= k && ord < o1; j++) {
    if (j < k ? L.cfg.sz[j] >= p.c : k >= p.g) continue;
    const int o = ord++;
    if (o < o0) continue;
    float T, E;
    if (!dfs_leaf(tb, p, L, j, x, j == j1 ? T2 : T1, Eall, T, E)) continue;
    unsigned need = 0;
    if constexpr (WS::N > 0) {
      float q[WS::N];
      WS::q(T, E, q);
#pragma unroll
      for (int s = 0; s < WS::N; s++)
        if (q[s] <= fminf(thr.v[s], q[s]) * (1.f + p.delta[p.ws_perm[s]])) need |= 1u << s;
    }
    const bool par = p.want_pareto && !stair_dominated_f(stair, p, __fmul_rd(T, p.tlb_scale_f), E);
    if (!need && !par) continue;
    nref++;
    // configuration: parent + x in group j
    uint32_t masks[kDfsMaxG + 1];
    for (int g = 0; g < k; g++) masks[g] = L.cfg.mask[g];
    masks[k] = 0;
    masks[j] |= 1u << x;
    int lam[kMaxN];
    for (int i = 0; i < p.n; i++) lam[i] = 0;
    double T64, E64;
    refine64(tb, p, masks, j == k ? k + 1 : k, lam, &T64, &E64);
    const u64 idx = base + o;
    if constexpr (WS::N > 0) {
#pragma unroll
      for (int s = 0; s < WS::N; s++) {
        if (need >> s & 1u) {
          const double F = objective64(p, T64, E64, WS::A(s), WS::B(s));
          BestRec &b = lb[s];
          if (!b.valid || better(F, idx, b.f, b.idx)) {
            b.f = F;
            b.idx = idx;
            b.t = T64;
            b.e = E64;
            b.t32 = T;
            b.e32 = E;
            b.valid = 1;
          }
        }
      }
    }
    if (par && !stair_dominated(stair, p, T64, __double2float_rd(__ddiv_rd(E64, p.eseq))))
      emit_candidate(p, stair, idx, T64, E64, T, E);
  }
  return nref;
}

template <class WS>
__global__ void __launch_bounds__(kDfsThreads, 2) k_dfs(const DevParams p) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned char *after = sm + ((p.blob_bytes + 15) & ~15u);
  Stair stair{(unsigned int *)(after + 8 * kBuckets), (unsigned long long *)after};
  BestRec *red = (BestRec *)(after + 12 * kBuckets);
  stair_init(stair);
  __syncthreads();

  Thr<WS> thr;
  BestRec lb[WS::N > 0 ? WS::N : 1];
#pragma unroll
  for (int s = 0; s < (WS::N > 0 ? WS::N : 1); s++) {
    thr.v[s] = __int_as_float(0x7f800000);
    best_init(lb[s]);
  }
  float mul[WS::N > 0 ? WS::N : 1];
#pragma unroll
  for (int s = 0; s < WS::N; s++) mul[s] = 1.f + p.delta[p.ws_perm[s]];
  u64 ncfg = 0, nfeas = 0, stair_ver = 0, nref = 0;
  const int ul = p.unit_log2, cl = p.chunk_log2, x = p.n - 1;
  DfsLane L;

  for (;;) {
    u64 unit = 0;
    if (lane == 0) unit = atomicAdd(p.ctr + kCtrUnit, 1ull);
    unit = __shfl_sync(0xffffffffu, unit, 0);
    if (unit >= p.n_units) break;
    const u64 ue = unit * p.unit_stride;
    const u64 ch = p.first_chunk + (ue >> (cl - ul)) * (u64)p.shard_count;
    u64 us = (ch << cl) + ((ue & ((1ull << (cl - ul)) - 1)) << ul);
    u64 uend = us + (1ull << ul);
    us = us > p.lo ? us : p.lo;
    uend = uend < p.hi ? uend : p.hi;
    if (us >= uend) continue;
#pragma unroll
    for (int w = 0; w < WS::N; w++) thr.v[w] = fminf(thr.v[w], __uint_as_float(__ldcg(p.thr + p.ws_perm[w])));
    if (p.want_pareto) {
      const u64 v = __ldcg(p.ctr + kCtrStairVer);
      if (v != stair_ver) {
        stair_ver = v;
        stair_merge(stair, p);
      }
    }
    // this lane's contiguous run
    const u64 run = (uend - us + 31) / 32;
    const u64 s = us + lane * run, e = s + run < uend ? s + run : uend;
    if (s < e && dev_unrank(tb, p, s, L.cfg)) {
      // detach workflow x: parent state + ordinal of the current leaf
      const int jx = L.cfg.a[x];
      L.cfg.mask[jx] &= ~(1u << x);
      if (--L.cfg.sz[jx] == 0) L.cfg.k--;
      int ord = 0;
      for (int j = 0; j < jx; j++)
        if (L.cfg.sz[j] < p.c) ord++;
      u64 base = s - ord;
      for (int g = 0; g < L.cfg.k; g++) dgroup_eval(tb, p, L.cfg.mask[g], L.g[g]);
      for (;;) {
        const int k = L.cfg.k;
        // parent aggregates: top-2 group makespans, total energy, feasibility
        float T1 = 0.f, T2 = 0.f, Eall = 0.f;
        int j1 = -1;
        bool pfeas = true;
        int nleaf = k < p.g ? 1 : 0;
        for (int g = 0; g < k; g++) {
          const float t = L.g[g].T;
          if (t > T1) {
            T2 = T1;
            T1 = t;
            j1 = g;
          } else {
            T2 = fmaxf(T2, t);
          }
          Eall += L.g[g].E;
          pfeas &= L.g[g].M <= p.mem_cap;
          nleaf += L.cfg.sz[g] < p.c;
        }
        const int o0 = s > base ? (int)(s - base) : 0;
        const int o1 = e - base < (u64)nleaf ? (int)(e - base) : nleaf;
        if (pfeas) {
          float mq[WS::N > 0 ? WS::N : 1], mT = __int_as_float(0x7f800000), mE = mT;
#pragma unroll
          for (int w = 0; w < WS::N; w++) mq[w] = __int_as_float(0x7f800000);
          int ord2 = 0, nf = 0;
          for (int j = 0; j <= k && ord2 < o1; j++) {
            if (j < k ? L.cfg.sz[j] >= p.c : k >= p.g) continue;
            const int o = ord2++;
            if (o < o0) continue;
            float T, E;
            if (!dfs_leaf(tb, p, L, j, x, j == j1 ? T2 : T1, Eall, T, E)) continue;
            nf++;
            mT = fminf(mT, T);
            mE = fminf(mE, E);
            if constexpr (WS::N > 0) {
              float q[WS::N];
              WS::q(T, E, q);
#pragma unroll
              for (int w = 0; w < WS::N; w++) mq[w] = fminf(mq[w], q[w]);
            }
          }
          nfeas += nf;
          bool hit = false;
#pragma unroll
          for (int w = 0; w < WS::N; w++) {
            thr.v[w] = fminf(thr.v[w], mq[w]);
            hit |= mq[w] <= thr.v[w] * mul[w];
          }
          if (nf && !hit && p.want_pareto) hit = !stair_dominated_f(stair, p, __fmul_rd(mT, p.tlb_scale_f), mE);
          if (nf && hit) nref += dfs_slow<WS>(tb, p, stair, L, thr, lb, base, o0, o1, T1, j1, T2, Eall);
        }
        ncfg += (u64)(o1 - o0);
        base += nleaf;
        if (base >= e) break;
        // next parent; recompute the groups whose membership changed
        uint32_t old[kDfsMaxG];
        for (int g = 0; g < kDfsMaxG; g++) old[g] = g < k ? L.cfg.mask[g] : 0u;
        if (!dfs_parent_successor(tb, p, L.cfg)) break;
        for (int g = 0; g < L.cfg.k; g++)
          if (L.cfg.mask[g] != old[g]) dgroup_eval(tb, p, L.cfg.mask[g], L.g[g]);
      }
    }
    __syncwarp();
#pragma unroll
    for (int w = 0; w < WS::N; w++) {
      float t = thr.v[w];
#pragma unroll
      for (int o = 16; o; o >>= 1) t = fminf(t, __shfl_xor_sync(0xffffffffu, t, o));
      thr.v[w] = t;
      if (lane == 0 && t < __uint_as_float(__ldcg(p.thr + p.ws_perm[w])))
        atomicMin(p.thr + p.ws_perm[w], __float_as_uint(t));
    }
  }
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
  for (int w = 0; w < WS::N; w++) {
    warp_best(lb[w]);
    if (lane == 0) red[warp * kMaxW + w] = lb[w];
  }
  __syncthreads();
  if (threadIdx.x < WS::N) {
    const int w = threadIdx.x;
    BestRec b = red[w];
    for (int k = 1; k < kDfsThreads / 32; k++) {
      const BestRec xx = red[k * kMaxW + w];
      if (xx.valid && (!b.valid || better(xx.f, xx.idx, b.f, b.idx))) b = xx;
    }
    ((BestRec *)p.slots)[(size_t)blockIdx.x * p.nw + p.ws_perm[w]] = b;
  }
}

template <class WS>
const void *dfs_fn();

#define SCHED_DFS_INSTANTIATE(WS)         \
  template <>                             \
  const void *dfs_fn<WS>() {              \
    return (const void *)k_dfs<WS>;       \
  }

}  // namespace sched
