// search_ctile.cuh -- PER_CLIENT tile kernel (c1/c2-style spaces, L = 4).
//
// In PER_CLIENT scope every client has its own MPS level, so a group's tuple
// (T_g, E_g) depends on its members' level sub-vector.  A warp walks the
// partitions of its index unit.  For a partition with k >= 3 groups the tile
// clients x1, x2, x3 are the highest-numbered members of the last three
// groups (blocks k-3, k-2, k-1 in RGS order); the other n-3 clients' level
// strings ("outer" strings) are split over the lanes.  Per outer string a
// lane evaluates the k-3 fixed groups once and each varying group at the 4
// levels of its tile client (12 group evaluations), then scores the 4^3 = 64
// configurations of the tile from registers exactly like the PER_GPU tile
// kernel: T = max(T_fix, A_a, B_b, C_c), E = ((E_fix + A_a) + B_b) + C_c --
// the canonical block order, since the varying groups are the last three
// blocks -- min-reduced to the tile's exact lower corner, screened once
// against the weights' thresholds and the Pareto staircase.  A tile that is
// not cleared is re-checked configuration by configuration with the exact
// fp64 group values (same canonical order as refine64, hence bitwise the
// oracle's).  A tile that straddles the unit's index range [v0, v1) is
// checked configuration by configuration inside the range; partitions with
// k < 3 take the per-configuration path (from-scratch fp32, refine64).
#pragma once
#include "search_tile.cuh"

namespace sched {

constexpr int kCtThreads = 256;
constexpr int kCtWarps = kCtThreads / 32;

struct CtWarp {
  LaneCfg cfg;
  u64 base;
};

// fp32 normalised (T_g, E-term) of group m at the levels packed in lw
// (2 bits per client: register-resident, no local-memory level array; the
// per-group operations of the generic kernel's score32_inc)
__device__ __forceinline__ void ct_group32(const Tables &tb, const DevParams &p, uint32_t m, uint32_t lw,
                                           float &Tg, float &Eg) {
  float U = 0.f, B = 0.f, D = 0.f;
  for (uint32_t mm = m; mm; mm &= mm - 1) {
    const int i = __ffs(mm) - 1, r = i * 4 + (int)((lw >> (2 * i)) & 3u);
    U += tb.u[r];
    B += tb.bw[r];
    D += tb.dh[r];
  }
  const float cg = fmaxf(fmaxf(1.f, U), B);
  float T = 0.f;
  for (uint32_t mm = m; mm; mm &= mm - 1) {
    const int i = __ffs(mm) - 1, ri = i * 4 + (int)((lw >> (2 * i)) & 3u);
    float s = 1.f;
    for (uint32_t m2 = m & ~(1u << i); m2; m2 &= m2 - 1) {
      const int j = __ffs(m2) - 1;
      s += tb.d[ri * p.ds + j * 4 + (int)((lw >> (2 * j)) & 3u)];
    }
    T = fmaxf(T, tb.th[ri] * s * cg);
  }
  if (p.model & SCHED_MODEL_POWER_CAP) T = fmaxf(T, D * p.kcap);  // R28
  Tg = T;
  Eg = p.phat * T + D;
}

// The same fp32 group values at the 4 levels of the group's HIGHEST member
// x (the tile client): x's terms come last in every ascending-member sum, so
// the sums over the other members are formed once and each level appends
// x's terms -- the same operations in the same order as ct_group32, hence
// the same values, in one pass (and one inlined copy) instead of four.
__device__ __forceinline__ void ct_group32_x4(const Tables &tb, const DevParams &p, uint32_t m, int x, uint32_t lw,
                                              float *Tg, float *Eg) {
  const uint32_t rest = m & ~(1u << x);
  float U = 0.f, B = 0.f, D = 0.f;
  for (uint32_t mm = rest; mm; mm &= mm - 1) {
    const int i = __ffs(mm) - 1, r = i * 4 + (int)((lw >> (2 * i)) & 3u);
    U += tb.u[r];
    B += tb.bw[r];
    D += tb.dh[r];
  }
  float Ux[4], Bx[4], Dx[4], Tm[4];
#pragma unroll
  for (int l = 0; l < 4; l++) {
    const int rx = x * 4 + l;
    Ux[l] = U + tb.u[rx];
    Bx[l] = B + tb.bw[rx];
    Dx[l] = D + tb.dh[rx];
    Tm[l] = 0.f;
  }
  // the other members, in ascending order: sigma over the others, then + d[i][x, l]
  for (uint32_t mm = rest; mm; mm &= mm - 1) {
    const int i = __ffs(mm) - 1, ri = i * 4 + (int)((lw >> (2 * i)) & 3u);
    float s = 1.f;
    for (uint32_t m2 = rest & ~(1u << i); m2; m2 &= m2 - 1) {
      const int j = __ffs(m2) - 1;
      s += tb.d[ri * p.ds + j * 4 + (int)((lw >> (2 * j)) & 3u)];
    }
#pragma unroll
    for (int l = 0; l < 4; l++) {
      const float cg = fmaxf(fmaxf(1.f, Ux[l]), Bx[l]);
      Tm[l] = fmaxf(Tm[l], tb.th[ri] * (s + tb.d[ri * p.ds + x * 4 + l]) * cg);
    }
  }
  // x itself (its sigma sums the others in ascending order; x is the highest member)
#pragma unroll
  for (int l = 0; l < 4; l++) {
    const int rx = x * 4 + l;
    float s = 1.f;
    for (uint32_t m2 = rest; m2; m2 &= m2 - 1) {
      const int j = __ffs(m2) - 1;
      s += tb.d[rx * p.ds + j * 4 + (int)((lw >> (2 * j)) & 3u)];
    }
    const float cg = fmaxf(fmaxf(1.f, Ux[l]), Bx[l]);
    float T = fmaxf(Tm[l], tb.th[rx] * s * cg);
    if (p.model & SCHED_MODEL_POWER_CAP) T = fmaxf(T, Dx[l] * p.kcap);  // R28
    Tg[l] = T;
    Eg[l] = p.phat * T + Dx[l];
  }
}

__device__ __forceinline__ uint32_t ct_set(uint32_t lw, int x, int l) {
  return (lw & ~(3u << (2 * x))) | ((uint32_t)l << (2 * x));
}

// exact canonical fp64 (T_g, E_g) of group m (refine64 for one group)
__device__ __forceinline__ void ct_group64(const Tables &tb, const DevParams &p, uint32_t m, uint32_t lw,
                                           double &Tg, double &Eg) {
  int lam[kMaxN];
  for (uint32_t mm = m; mm; mm &= mm - 1) {
    const int i = __ffs(mm) - 1;
    lam[i] = (int)((lw >> (2 * i)) & 3u);
  }
  refine64(tb, p, &m, 1, lam, &Tg, &Eg);
}

// One configuration with known fp32 (T, E) and a way to get its exact fp64
// (T, E): weight screens (lane thresholds), Pareto screen, fp64 record.
template <int WM, class Exact>
__device__ __forceinline__ int ct_check(const DevParams &p, const Stair &stair, float *thr, BestRec *lb, u64 idx,
                                        float T, float E, Exact exact) {
  unsigned need = 0;
#pragma unroll
  for (int w = 0; w < WM; w++) {
    if (w < p.nw) {
      float q = 1.f;
      for (int i = 0; i < p.wa[w]; i++) q *= T;
      for (int i = 0; i < p.wb[w]; i++) q *= E;
      thr[w] = fminf(thr[w], q);
      if (q <= thr[w] * p.mul[w]) need |= 1u << w;
    }
  }
  double T64 = 0.0, E64 = 0.0;
  bool have = false;
  bool par = false;
  if (p.want_pareto) {
    exact(T64, E64);
    have = true;
    par = !stair_dominated(stair, p, T64, E);
  }
  if (!need && !par) return 0;
  if (!have) exact(T64, E64);
  // weights with b = 0 (F = X^a depends on T alone): a best with makespan
  // <= T64 at a lower index cannot be replaced -- exact early reject
#pragma unroll
  for (int w = 0; w < WM; w++)
    if ((need >> w & 1u) && p.wb[w] == 0 && lb[w].valid && T64 >= lb[w].t && idx > lb[w].idx) need &= ~(1u << w);
#pragma unroll
  for (int w = 0; w < WM; w++) {
    if (need >> w & 1u) {
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
  return 1;
}

// Per-configuration path: level vectors v in [v0, v1) step `step` of the
// partition (from-scratch fp32 score, refine64 when screened in).
template <int WM>
__device__ __noinline__ int ct_edge(const Tables &tb, const DevParams &p, const Stair &stair, const CtWarp &wp,
                                    float *thr, BestRec *lb, uint32_t v0, uint32_t v1, uint32_t step) {
  const int n = p.n, k = wp.cfg.k;
  int nref = 0;
  int lam[kMaxN];
  for (uint32_t v = v0; v < v1; v += step) {
    uint32_t lw = 0;
    for (int i = 0; i < n; i++) {
      lam[i] = (int)(v >> (2 * (n - 1 - i))) & 3;
      lw |= (uint32_t)lam[i] << (2 * i);
    }
    float T = 0.f, E = 0.f;
    for (int g = 0; g < k; g++) {
      float Tg, Eg;
      ct_group32(tb, p, wp.cfg.mask[g], lw, Tg, Eg);
      T = fmaxf(T, Tg);
      E += Eg;
    }
    nref += ct_check<WM>(p, stair, thr, lb, wp.base + v, T, E, [&](double &T64, double &E64) {
      refine64(tb, p, wp.cfg.mask, k, lam, &T64, &E64);
    });
  }
  return nref;
}

// WM: weights held per lane (thresholds, best records) -- the smallest of
// 1, 2, 4, 8 that covers the query, to keep the per-thread stack small
template <int WM>
__global__ void __launch_bounds__(kCtThreads, 2) k_ctile(const DevParams p) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned char *after = sm + ((p.blob_bytes + 15) & ~15u);
  Stair stair = stair_at(after);
  CtWarp *wps = (CtWarp *)(after + kStairSmem);
  CtWarp &wp = wps[warp];
  BestRec *red = (BestRec *)(wps + kCtWarps);
  stair_init(stair);
  __syncthreads();

  float thr[WM];
  BestRec lb[WM];
#pragma unroll
  for (int w = 0; w < WM; w++) {
    thr[w] = __int_as_float(0x7f800000);
    best_init(lb[w]);
  }
  u64 ncfg = 0, nfeas = 0, stair_ver = 0;
  int nref = 0;
  const int n = p.n;
  const int ul = p.unit_log2, cl = p.chunk_log2;
  const uint32_t nout = 1u << (2 * (n - 3));  // outer level strings

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
    for (int w = 0; w < WM; w++)
      if (w < p.nw) thr[w] = fminf(thr[w], __uint_as_float(__ldcg(p.thr + w)));
    if (p.want_pareto) stair_sync(stair, p, stair_ver, __ldcg(p.ctr + kCtrStairVer));
    if (lane == 0) {
      dev_unrank(tb, p, s, wp.cfg);
      wp.base = s - wp.cfg.v;
    }
    __syncwarp();
    for (;;) {
      if (p.want_pareto) stair_sync(stair, p, stair_ver, __ldcg(p.ctr + kCtrStairVer));
      const u64 base = wp.base;
      const uint32_t Pn = (uint32_t)wp.cfg.Pn;
      const int k = wp.cfg.k;
      const bool feas = wp.cfg.feasible;
      const uint32_t v0 = s > base ? (uint32_t)(s - base) : 0u;
      const uint32_t v1 = e - base < (u64)Pn ? (uint32_t)(e - base) : Pn;
      if (lane == 0) {
        ncfg += v1 - v0;
        if (feas) nfeas += v1 - v0;
      }
      if (feas) {
        if (k < 3) {
          nref += ct_edge<WM>(tb, *p.gp, stair, wp, thr, lb, v0 + lane, v1, 32);
        } else {
          // tile clients: the highest member of each of the last three blocks
          const uint32_t ma = wp.cfg.mask[k - 3], mb = wp.cfg.mask[k - 2], mc = wp.cfg.mask[k - 1];
          const int x1 = 31 - __clz(ma), x2 = 31 - __clz(mb), x3 = 31 - __clz(mc);
          const uint32_t tmask = (1u << x1) | (1u << x2) | (1u << x3);
          const int s1 = 2 * (n - 1 - x1), s2 = 2 * (n - 1 - x2), s3 = 2 * (n - 1 - x3);
          const uint32_t tbits = (3u << s1) | (3u << s2) | (3u << s3);
          for (uint32_t o = lane; o < nout; o += 32) {
            // outer string o -> levels of the non-tile clients (ascending, most significant first)
            uint32_t lw = 0;  // levels, 2 bits per client (tile clients 0)
            uint32_t vo = 0;  // the outer digits' contribution to the level-vector index
            {
              int sh = 2 * (n - 4);
              for (int i = 0; i < n; i++) {
                if (tmask >> i & 1u) continue;
                const uint32_t d = (o >> sh) & 3u;
                sh -= 2;
                lw |= d << (2 * i);
                vo |= d << (2 * (n - 1 - i));
              }
            }
            // the tile's index span [vo, vo | tbits]: skip it if it misses [v0, v1)
            if ((vo | tbits) < v0 || vo >= v1) continue;
            const bool whole = vo >= v0 && (vo | tbits) < v1;
            float Tp = 0.f, Ep = 0.f;
            for (int g = 0; g < k - 3; g++) {
              float Tg, Eg;
              ct_group32(tb, p, wp.cfg.mask[g], lw, Tg, Eg);
              Tp = fmaxf(Tp, Tg);
              Ep += Eg;
            }
            float At[4], Ae[4], Bt[4], Be[4], Ct[4], Ce[4];
            ct_group32_x4(tb, p, ma, x1, lw, At, Ae);
            ct_group32_x4(tb, p, mb, x2, lw, Bt, Be);
            ct_group32_x4(tb, p, mc, x3, lw, Ct, Ce);
            if (whole) {
              // the tile's 64 configurations, min-reduced to the exact lower corner
              float mT = __int_as_float(0x7f800000), mE = mT;
#pragma unroll
              for (int a = 0; a < 4; a++) {
                const float T1 = fmaxf(Tp, At[a]), E1 = Ep + Ae[a];
#pragma unroll
                for (int b = 0; b < 4; b++) {
                  const float T2 = fmaxf(T1, Bt[b]), E2 = E1 + Be[b];
#pragma unroll
                  for (int c = 0; c < 4; c++) {
                    mT = fminf(mT, fmaxf(T2, Ct[c]));
                    mE = fminf(mE, E2 + Ce[c]);
                  }
                }
              }
              bool hit = false;
#pragma unroll
              for (int w = 0; w < WM; w++) {
                if (w < p.nw) {
                  float q = 1.f;
                  for (int i = 0; i < p.wa[w]; i++) q *= mT;
                  for (int i = 0; i < p.wb[w]; i++) q *= mE;
                  hit |= q <= thr[w] * p.mul[w];
                }
              }
              const bool par = p.want_pareto && !stair_dominated_f(stair, p, __fmul_rd(mT, p.tlb_scale_f), mE);
              if (!hit && !par) continue;
            }
            // slow path: exact fp64 group values of this tile, then every
            // configuration of it inside [v0, v1)
            double Tp64 = 0.0, Ep64 = 0.0;
            for (int g = 0; g < k - 3; g++) {
              double Tg, Eg;
              ct_group64(tb, p, wp.cfg.mask[g], lw, Tg, Eg);
              if (Tg > Tp64) Tp64 = Tg;
              Ep64 = __dadd_rn(Ep64, Eg);
            }
            double A64[4], AE64[4], B64[4], BE64[4], C64[4], CE64[4];
#pragma unroll 1  // rare path: keep the code small (instruction cache)
            for (int l = 0; l < 4; l++) {
              const uint32_t ll = ct_set(ct_set(ct_set(lw, x1, l), x2, l), x3, l);
              ct_group64(tb, p, ma, ll, A64[l], AE64[l]);
              ct_group64(tb, p, mb, ll, B64[l], BE64[l]);
              ct_group64(tb, p, mc, ll, C64[l], CE64[l]);
            }
#pragma unroll 1
            for (int a = 0; a < 4; a++)
#pragma unroll 1
              for (int b = 0; b < 4; b++)
#pragma unroll 1
                for (int c = 0; c < 4; c++) {
                  const uint32_t v = vo | ((uint32_t)a << s1) | ((uint32_t)b << s2) | ((uint32_t)c << s3);
                  if (v < v0 || v >= v1) continue;
                  const float T = fmaxf(fmaxf(fmaxf(Tp, At[a]), Bt[b]), Ct[c]);
                  const float E = ((Ep + Ae[a]) + Be[b]) + Ce[c];
                  nref += ct_check<WM>(p, stair, thr, lb, base + v, T, E, [&](double &T64, double &E64) {
                    T64 = fmax(fmax(fmax(Tp64, A64[a]), B64[b]), C64[c]);
                    E64 = __dadd_rn(__dadd_rn(__dadd_rn(Ep64, AE64[a]), BE64[b]), CE64[c]);
                  });
                }
          }
        }
      }
      __syncwarp();
      if (base + Pn >= e) break;
      if (lane == 0) {
        wp.base = base + Pn;
        dev_successor(tb, p, wp.cfg);
        wp.cfg.Pn = tb.W[wp.cfg.st[p.n - 1]];
        wp.cfg.v = 0;
        cfg_feasibility(tb, p, wp.cfg);
      }
      __syncwarp();
    }
#pragma unroll
    for (int w = 0; w < WM; w++) {
      if (w < p.nw) {
        float t = thr[w];
#pragma unroll
        for (int o = 16; o; o >>= 1) t = fminf(t, __shfl_xor_sync(0xffffffffu, t, o));
        thr[w] = t;
        if (lane == 0 && t < __uint_as_float(__ldcg(p.thr + w))) atomicMin(p.thr + w, __float_as_uint(t));
      }
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
  for (int w = 0; w < WM; w++) {
    if (w < p.nw) {
      warp_best(lb[w]);
      if (lane == 0) red[warp * kMaxW + w] = lb[w];
    }
  }
  __syncthreads();
  if (threadIdx.x < p.nw) {
    const int w = threadIdx.x;
    BestRec b = red[w];
    for (int q = 1; q < kCtWarps; q++) {
      const BestRec x = red[q * kMaxW + w];
      if (x.valid && (!b.valid || better(x.f, x.idx, b.f, b.idx))) b = x;
    }
    ((BestRec *)p.slots)[(size_t)blockIdx.x * p.nw + w] = b;
  }
}

template <int WM>
const void *ctile_fn() {
  return (const void *)k_ctile<WM>;
}

}  // namespace sched
