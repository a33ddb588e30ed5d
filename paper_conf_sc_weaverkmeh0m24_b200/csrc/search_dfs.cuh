// search_dfs.cuh -- L = 1 partition kernel (c5 fast path), warp-cooperative.
//
// With one MPS level every configuration is a set partition (RGS).  A warp
// walks *prefixes*: partitions of workflows 0..n-3.  The completions of a
// prefix -- admissible groups (j1, j2) of the last two workflows x1 = n-2,
// x2 = n-1, in lexicographic order -- are consecutive indices.  Per prefix:
//   * lane (g, kind) loads from the group-tuple table (k_groups, L2-resident)
//     the tuple of prefix group g, of "g + x1", "g + x2" and "g + x1 + x2"
//     (fp32 T_g, E_g and the exact fp64 T_g, E_g; +inf = over C / memory);
//   * lanes test the <= 90 candidate pairs and a ballot scan builds the
//     ordered completion list;
//   * each lane scores its completions from lookups:
//       T = max(max of prefix groups not touched, new tuples),
//       E = E_all - sum(E of touched groups) + sum(new tuples' E)
//     (all terms >= 0 and touched groups only grow, so the subtraction keeps
//     the relative error bound of DESIGN.md section 5), min-reduces the
//     proxies and (T, E), and screens them once; a lane that is not cleared
//     re-checks its completions one by one; the fp64 canonical re-score is
//     T = max of the exact group T_g, E = sum of the exact E_g in block order.
#pragma once
#include "device_common.cuh"
#include "search_tile.cuh"

namespace sched {

// per-lane thresholds of the pair kernel: value and 1 + delta per weight slot
template <class WS>
struct DThr {
  float v[WS::N > 0 ? WS::N : 1];
  float m[WS::N > 0 ? WS::N : 1];
};

constexpr int kDfsMaxC = 4;
constexpr int kDfsMaxG = 8;
constexpr int kDfsThreads = 256;
constexpr int kPairCand = (kDfsMaxG + 1) * (kDfsMaxG + 2);  // 90

struct Tup {
  float t, e;      // fp32 normalised T_g, E_g; t = +inf: infeasible / over C members
  double t64, e64; // exact canonical fp64 T_g, E_g
};

__device__ __forceinline__ Tup tup_load(const GroupRec *gt, uint32_t m) {
  const GroupRec r = gt[m];
  return Tup{r.t32, r.e32, r.t64, r.e64};
}

struct PairWarp {
  LaneCfg cfg;       // prefix: workflows 0..n-3 placed
  u64 base;          // index of the prefix's first completion
  Tup g[kDfsMaxG], a1[kDfsMaxG], a2[kDfsMaxG], ab[kDfsMaxG];
  Tup n1, n2, n12;   // new groups {x1}, {x2}, {x1, x2}
  uint8_t pj[kPairCand];  // completion list: j1 * 16 + j2
  int npairs;
  float top[3];
  int topi[3];
  float Eall;
  int feas;
};

// successor of the prefix RGS (positions 1..n-3), keeping the last two
// workflows placeable (W > 0 in the DP table); greedy fill up to n-3.
__device__ __forceinline__ bool pair_prefix_successor(const Tables &tb, const DevParams &p, LaneCfg &c) {
  const int last = p.n - 3;
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

// (T, E) of completion (j1, j2) of the warp's prefix; false if infeasible
__device__ __forceinline__ bool pair_score(const PairWarp &w, int j1, int j2, float &T, float &E) {
  const int k = w.cfg.k;
  Tup ta, tb2;
  int x1g = -1, x2g = -1;  // touched prefix groups
  if (j1 == j2) {
    if (j1 < k) {
      ta = w.ab[j1];
      x1g = j1;
    } else {
      ta = w.n12;
    }
    tb2 = Tup{0.f, 0.f, 0.0, 0.0};
  } else {
    if (j1 < k) {
      ta = w.a1[j1];
      x1g = j1;
    } else {
      ta = w.n1;
    }
    if (j2 < k) {
      tb2 = w.a2[j2];
      x2g = j2;
    } else {
      tb2 = w.n2;
    }
  }
  if (!(ta.t < __int_as_float(0x7f800000)) || !(tb2.t < __int_as_float(0x7f800000))) return false;
  // max over prefix groups not touched: first of the top-3 not in {x1g, x2g}
  float ex = 0.f;
#pragma unroll
  for (int q = 2; q >= 0; q--)
    if (w.topi[q] >= 0 && w.topi[q] != x1g && w.topi[q] != x2g) ex = w.top[q];
  T = fmaxf(fmaxf(ex, ta.t), tb2.t);
  float Er = w.Eall;
  if (x1g >= 0) Er -= w.g[x1g].e;
  if (x2g >= 0) Er -= w.g[x2g].e;
  E = Er + (ta.e + tb2.e);
  return true;
}

template <class WS>
__device__ __noinline__ int pair_slow(const Tables &tb, const DevParams &p, const Stair &stair, const PairWarp &w,
                                      const float *thr, BestRec *lb, int o0, int o1, int lane) {
  const int k = w.cfg.k, x1 = p.n - 2, x2 = p.n - 1;
  int nref = 0;
  for (int o = o0 + lane; o < o1; o += 32) {
    const int j1 = w.pj[o] >> 4, j2 = w.pj[o] & 15;
    float T, E;
    if (!pair_score(w, j1, j2, T, E)) continue;
    unsigned need = 0;
    if constexpr (WS::N > 0) {
      float q[WS::N];
      WS::q(T, E, q);
#pragma unroll
      for (int s = 0; s < WS::N; s++)
        if (q[s] <= fminf(thr[s], q[s]) * p.mul[p.ws_perm[s]]) need |= 1u << s;
    }
    const bool par = p.want_pareto && !stair_dominated_f(stair, p, __fmul_rd(T, p.tlb_scale_f), E);
    if (!need && !par) continue;
    nref++;
    // fp64 canonical re-score from the exact group tuples: groups in block
    // order (prefix groups, then new groups), T = max T_g, E = sum E_g left to right
    double T64 = 0.0, E64 = 0.0;
    for (int g = 0; g < k; g++) {
      const Tup &t = g == j1 ? (j1 == j2 ? w.ab[g] : w.a1[g]) : (g == j2 ? w.a2[g] : w.g[g]);
      T64 = fmax(T64, t.t64);
      E64 = __dadd_rn(E64, t.e64);
    }
    if (j1 >= k || j2 >= k) {  // new groups: j1 == j2 == k | j1 == k < j2 | j1 < k == j2
      if (j1 == j2) {
        T64 = fmax(T64, w.n12.t64);
        E64 = __dadd_rn(E64, w.n12.e64);
      } else {
        if (j1 >= k) {
          T64 = fmax(T64, w.n1.t64);
          E64 = __dadd_rn(E64, w.n1.e64);
        }
        if (j2 >= k) {
          T64 = fmax(T64, w.n2.t64);
          E64 = __dadd_rn(E64, w.n2.e64);
        }
      }
    }
    const u64 idx = w.base + o;
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
    if (par && !stair_dominated(stair, p, T64, __double2float_rd(__ddiv_rd(E64, p.eseq))) &&
        !stair_dominated_exact(stair, p, T64, E64))
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
  Stair stair = stair_at(after);
  PairWarp *pws = (PairWarp *)(after + kStairSmem);
  PairWarp &w = pws[warp];
  BestRec *red = (BestRec *)(pws + kDfsThreads / 32);
  float *thr_sm = (float *)(red + (kDfsThreads / 32) * kMaxW) + threadIdx.x * kMaxW;
  stair_init(stair);
  const int x1 = p.n - 2, x2 = p.n - 1;
  const GroupRec *gtab = (const GroupRec *)p.gtab;
  if (lane == 0) {
    w.n1 = tup_load(gtab, 1u << x1);
    w.n2 = tup_load(gtab, 1u << x2);
    w.n12 = tup_load(gtab, (1u << x1) | (1u << x2));
  }
  __syncthreads();

  DThr<WS> thr;
  BestRec lb[WS::N > 0 ? WS::N : 1];
#pragma unroll
  for (int s = 0; s < (WS::N > 0 ? WS::N : 1); s++) {
    thr.v[s] = __int_as_float(0x7f800000);
    best_init(lb[s]);
  }
  u64 ncfg = 0, nfeas = 0, stair_ver = 0;
  int nref = 0;
  const int ul = p.unit_log2, cl = p.chunk_log2;

  for (;;) {
    u64 unit = 0;
    if (lane == 0)  // a pass that overflowed the candidate buffer stops early (it is re-run)
      unit = (p.abort_ovf && __ldcg(p.ctr + kCtrOverflow)) ? ~0ull : atomicAdd(p.ctr + kCtrUnit, 1ull);
    unit = __shfl_sync(0xffffffffu, unit, 0);
    if (unit >= p.n_units) break;
    const u64 ue = unit * p.unit_stride;
    const u64 ch = p.first_chunk + (ue >> (cl - ul)) * (u64)p.shard_count;
    u64 s = (ch << cl) + ((ue & ((1ull << (cl - ul)) - 1)) << ul);
    u64 e = s + (1ull << ul);
    s = s > p.lo ? s : p.lo;
    e = e < p.hi ? e : p.hi;
    if (s >= e) continue;
#pragma unroll
    for (int q = 0; q < WS::N; q++) thr.v[q] = fminf(thr.v[q], __uint_as_float(__ldcg(p.thr + p.ws_perm[q])));
    if (p.want_pareto) {
      stair_sync(stair, p, stair_ver, __ldcg(p.ctr + kCtrStairVer));
    }
    if (lane == 0) {  // unrank s, detach the last two workflows: prefix + completion ordinal
      dev_unrank(tb, p, s, w.cfg);
      const int j2 = w.cfg.a[x2];
      w.cfg.mask[j2] &= ~(1u << x2);
      if (--w.cfg.sz[j2] == 0) w.cfg.k--;
      const int j1 = w.cfg.a[x1];
      w.cfg.mask[j1] &= ~(1u << x1);
      if (--w.cfg.sz[j1] == 0) w.cfg.k--;
      // ordinal of (j1, j2) among the prefix's completions
      const int k = w.cfg.k;
      int ord = 0;
      for (int a = 0; a <= k && a <= j1; a++) {
        if (a < k ? w.cfg.sz[a] >= p.c : k >= p.g) continue;
        const int k2 = k + (a == k);
        for (int b = 0; b <= k2; b++) {
          if (a == j1 && b >= j2) break;
          const int szb = b < k ? w.cfg.sz[b] + (b == a) : (b == a ? 1 : 0);
          if (b < k2 ? szb >= p.c : k2 >= p.g) continue;
          ord++;
        }
      }
      w.base = s - ord;
    }
    __syncwarp();
    u64 ver_pref = p.want_pareto ? __shfl_sync(0xffffffffu, __ldcg(p.ctr + kCtrStairVer), 0) : 0;
    for (;;) {
      if (p.want_pareto) {
        stair_sync(stair, p, stair_ver, ver_pref);
        ver_pref = __shfl_sync(0xffffffffu, __ldcg(p.ctr + kCtrStairVer), 0);
      }
      const int k = w.cfg.k;
      // ---- per-prefix tables (lane-parallel) ----
      if ((lane >> 2) < k) {  // lane = (group, kind): group, + x1, + x2, + both (table lookups)
        const int gg = lane >> 2, kind = lane & 3;
        const uint32_t m = w.cfg.mask[gg] | (kind & 1 ? 1u << x1 : 0u) | (kind & 2 ? 1u << x2 : 0u);
        const Tup t = tup_load(gtab, m);  // > C members or over memory: t = +inf
        (kind == 0 ? w.g : kind == 1 ? w.a1 : kind == 2 ? w.a2 : w.ab)[gg] = t;
      }
      // completion list: candidate c = j1 * (G + 2) + j2 in lexicographic order
      int npairs = 0;
      for (int c0 = 0; c0 < kPairCand; c0 += 32) {
        const int c = c0 + lane, j1 = c / (kDfsMaxG + 2), j2 = c % (kDfsMaxG + 2);
        bool ok = c < kPairCand && j1 <= k;
        if (ok) ok = j1 < k ? w.cfg.sz[j1] < p.c : k < p.g;
        const int k2 = k + (j1 == k);
        if (ok) ok = j2 <= k2;
        if (ok) {
          const int szb = j2 < k ? w.cfg.sz[j2] + (j2 == j1) : (j2 == j1 ? 1 : 0);
          ok = j2 < k2 ? szb < p.c : k2 < p.g;
        }
        const unsigned bal = __ballot_sync(0xffffffffu, ok);
        if (ok) w.pj[npairs + __popc(bal & ((1u << lane) - 1))] = (uint8_t)(j1 * 16 + j2);
        npairs += __popc(bal);
      }
      __syncwarp();
      if (lane == 0) {
        float t0 = 0.f, t1 = 0.f, t2 = 0.f, Ea = 0.f;
        int i0 = -1, i1 = -1, i2 = -1, ok = 1;
        for (int g = 0; g < k; g++) {
          const float t = w.g[g].t;
          ok &= t < __int_as_float(0x7f800000);
          Ea += w.g[g].e;
          if (t > t0) {
            t2 = t1; i2 = i1; t1 = t0; i1 = i0; t0 = t; i0 = g;
          } else if (t > t1) {
            t2 = t1; i2 = i1; t1 = t; i1 = g;
          } else if (t > t2) {
            t2 = t; i2 = g;
          }
        }
        w.top[0] = t0; w.top[1] = t1; w.top[2] = t2;
        w.topi[0] = i0; w.topi[1] = i1; w.topi[2] = i2;
        w.Eall = Ea;
        w.feas = ok;
        w.npairs = npairs;
      }
      __syncwarp();
      const u64 base = w.base;
      const int o0 = s > base ? (int)(s - base) : 0;
      const int o1 = e - base < (u64)npairs ? (int)(e - base) : npairs;
      if (lane == 0) ncfg += (u64)(o1 - o0);
      if (w.feas) {
        float mq[WS::N > 0 ? WS::N : 1], mT = __int_as_float(0x7f800000), mE = mT;
#pragma unroll
        for (int q = 0; q < WS::N; q++) mq[q] = __int_as_float(0x7f800000);
        int nf = 0;
        for (int o = o0 + lane; o < o1; o += 32) {
          float T, E;
          if (!pair_score(w, w.pj[o] >> 4, w.pj[o] & 15, T, E)) continue;
          nf++;
          mT = fminf(mT, T);
          mE = fminf(mE, E);
          if constexpr (WS::N > 0) {
            float q[WS::N];
            WS::q(T, E, q);
#pragma unroll
            for (int qq = 0; qq < WS::N; qq++) mq[qq] = fminf(mq[qq], q[qq]);
          }
        }
        nfeas += nf;
        bool hit = false;
#pragma unroll
        for (int q = 0; q < WS::N; q++) {
          thr.v[q] = fminf(thr.v[q], mq[q]);
          hit |= mq[q] <= thr.v[q] * p.mul[p.ws_perm[q]];
        }
        if (nf && !hit && p.want_pareto) hit = !stair_dominated_f(stair, p, __fmul_rd(mT, p.tlb_scale_f), mE);
        if (nf && hit) {
#pragma unroll
          for (int q = 0; q < WS::N; q++) thr_sm[q] = thr.v[q];
          nref += pair_slow<WS>(tb, p, stair, w, thr_sm, lb, o0, o1, lane);
        }
      }
      __syncwarp();
      if (base + npairs >= e) break;
      if (lane == 0) {
        w.base = base + npairs;
        w.feas = pair_prefix_successor(tb, p, w.cfg) ? 1 : -1;
      }
      __syncwarp();
      if (w.feas < 0) break;
    }
#pragma unroll
    for (int q = 0; q < WS::N; q++) {
      float t = thr.v[q];
#pragma unroll
      for (int o = 16; o; o >>= 1) t = fminf(t, __shfl_xor_sync(0xffffffffu, t, o));
      thr.v[q] = t;
      if (lane == 0 && t < __uint_as_float(__ldcg(p.thr + p.ws_perm[q])))
        atomicMin(p.thr + p.ws_perm[q], __float_as_uint(t));
    }
  }
  u64 nref64 = (u64)nref;
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    ncfg += __shfl_xor_sync(0xffffffffu, ncfg, o);
    nfeas += __shfl_xor_sync(0xffffffffu, nfeas, o);
    nref64 += __shfl_xor_sync(0xffffffffu, nref64, o);
  }
  if (lane == 0) {
    atomicAdd(p.ctr + kCtrConfigs, ncfg);
    atomicAdd(p.ctr + kCtrFeasible, nfeas);
    atomicAdd(p.ctr + kCtrRefined, nref64);
  }
#pragma unroll
  for (int q = 0; q < WS::N; q++) {
    warp_best(lb[q]);
    if (lane == 0) red[warp * kMaxW + q] = lb[q];
  }
  __syncthreads();
  if (threadIdx.x < WS::N) {
    const int q = threadIdx.x;
    BestRec b = red[q];
    for (int kk = 1; kk < kDfsThreads / 32; kk++) {
      const BestRec xx = red[kk * kMaxW + q];
      if (xx.valid && (!b.valid || better(xx.f, xx.idx, b.f, b.idx))) b = xx;
    }
    ((BestRec *)p.slots)[(size_t)blockIdx.x * p.nw + p.ws_perm[q]] = b;
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
