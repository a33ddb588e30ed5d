// search_ctile2.cuh -- PER_CLIENT tile kernel over per-partition group tables
// (kernel_path 6: PER_CLIENT, L = 4, groups of <= 4 clients, G <= 8; the
// literal per-client reading of c3, "c3-client").
//
// In PER_CLIENT scope a group's tuple (T_g, E_g) depends on the levels of its
// own members only (U, B, sigma, tau and D are sums /
// maxima over the group's members).  So per partition every group g's
// tuples at all 4^|g| member-level vectors are evaluated ONCE (fp32, into a
// per-warp shared-memory table: <= 836 entries for groups of <= 4 clients),
// and the 4^n configurations of the partition are scored from table lookups:
//   T = max_g T_g[var_g],  E = ((E_0[var_0] + E_1[var_1]) + ...) + E_{k-1}
// in block order (the canonical order).  var_g = the member levels of g as a
// base-4 number, lowest member most significant.
//
// Tile: the highest member x of each of the last three groups (A, B, C =
// blocks k-3, k-2, k-1) varies over its 4 levels (x is the least significant
// digit of its group's variant, so A's 4 tuples are 4 consecutive table
// entries); the other n-3 clients' levels form the outer string o.  Lanes
// take o = st * 32 + lane; the warp loop runs over st.  A group's table
// index is additive in the outer digits (idx_g(o) = idxS_g(st) +
// idxL_g(lane)), so per step the warp-uniform part advances by a per-
// partition delta table keyed by the trailing-ones count of st -- no per-
// configuration or per-string group evaluation.  Per step a lane loads the
// 5 fixed-group tuples (blocks 0..k-4; unused slots read a (0, 0) pad) and
// the 3 x 4 varying tuples, then scores the 64 configurations from registers
// exactly like the PER_GPU tile kernel (T max, E add, the tile's exact lower
// corner by min-reduction), screens the corner once against the weights'
// thresholds and the Pareto staircase, and re-checks a tile that is not
// cleared (or that straddles the unit's index range) configuration by
// configuration with exact fp64 group values (refine64 order: bitwise the
// oracle's).
#pragma once
#include "search_ctile.cuh"

namespace sched {

constexpr int kC2Threads = 512;
constexpr int kC2Warps = kC2Threads / 32;
constexpr int kC2Tab = 896;    // table entries per warp: 4 pad + sum_g roundup4(4^|g|) <= 4 + 3*256 + 64
constexpr int kC2Bits = 20;    // bits of st: 4^(n-3) / 32 <= 2^19 for n <= 15
constexpr int kC2Slots = 8;
constexpr int kC2MaxGrid = 256;  // CTAs (1 per SM): bounds the workspace's fp64 T tables    // 5 fixed-group slots + A, B, C; slot 8 of the delta rows = vo

struct C2Warp {
  LaneCfg cfg;
  u64 base, ncfg, nfeas, sver;
  int d[kC2Bits][kC2Slots + 1];   // st -> st + 1 with c trailing ones: delta of idxS[0..7] and voS
  int wb[kC2Bits][kC2Slots + 1];  // contribution of st bit b
  int8_t oc[kMaxN];               // outer digit position t (0 = least significant) -> client
  __align__(16) float2 tab[kC2Tab];  // (T-hat, E-hat) per (group, member-level vector)
};

// group variant (member levels, lowest member most significant) -> level word
__device__ __forceinline__ uint32_t c2_lw(uint32_t m, uint32_t v, int s) {
  uint32_t lw = 0;
  int r = s - 1;
  for (uint32_t mm = m; mm; mm &= mm - 1, r--) lw |= ((v >> (2 * r)) & 3u) << (2 * (__ffs(mm) - 1));
  return lw;
}

// table offsets: off[0] = 4 (entries 0..3: the (0, 0) pad), group g's 4^|g|
// entries from off[g], each table rounded up to a multiple of 4 entries
__device__ __forceinline__ void c2_offsets(const C2Warp &wp, int *off) {
  off[0] = 4;
  for (int g = 0; g < wp.cfg.k; g++) off[g + 1] = off[g] + (((1 << (2 * __popc(wp.cfg.mask[g]))) + 3) & ~3);
}

// per-partition group tables: fp32 (T-hat, E-hat) at every member-level
// vector in shared memory, and the exact canonical fp64 T_g (refine64 order)
// in the warp's global table t64 (read only by the tile's exact-corner
// Pareto check, through L2)
// Returns the partition's fp32 min makespan: max over groups of the group's
// min T-hat over its member-level vectors (every configuration's T-hat is at
// least that: T-hat is a max of these entries).
__device__ __forceinline__ float c2_tables(const Tables &tb, const DevParams &p, C2Warp &wp, int lane,
                                           double *t64) {
  const int k = wp.cfg.k;
  int off[kMaxG + 1];
  c2_offsets(wp, off);
  float gmin[kMaxG];
#pragma unroll
  for (int g = 0; g < kMaxG; g++) gmin[g] = __int_as_float(0x7f800000);
  for (int e = lane; e < off[k]; e += 32) {
    float2 v = make_float2(0.f, 0.f);
    double T64 = 0.0;
    if (e >= 4) {
      int g = 0;
      while (e >= off[g + 1]) g++;
      const uint32_t m = wp.cfg.mask[g];
      const int s = __popc(m);
      const uint32_t var = (uint32_t)(e - off[g]);
      if (var < (1u << (2 * s))) {
        const uint32_t lw = c2_lw(m, var, s);
        ct_group32(tb, p, m, lw, v.x, v.y);
        if (p.want_pareto) {
          double E64;
          ct_group64(tb, p, m, lw, T64, E64);
        }
#pragma unroll
        for (int q = 0; q < kMaxG; q++)
          if (q == g) gmin[q] = fminf(gmin[q], v.x);
      }
    }
    wp.tab[e] = v;
    if (p.want_pareto) __stcg(t64 + e, T64);
  }
  float tmin = 0.f;
#pragma unroll
  for (int g = 0; g < kMaxG; g++) {
    float m = gmin[g];
#pragma unroll
    for (int o = 16; o; o >>= 1) m = fminf(m, __shfl_xor_sync(0xffffffffu, m, o));
    if (g < k) tmin = fmaxf(tmin, m);
  }
  __threadfence_block();
  __syncwarp();
  return tmin;
}

// per-partition tile setup (k >= 3): outer digit map, delta / contribution
// rows; every lane returns its own idxL[8] (table offsets folded in) and voL
__device__ __forceinline__ void c2_setup(const DevParams &p, C2Warp &wp, int lane, int *idxL, uint32_t &voL,
                                         uint32_t &tbits) {
  const int n = p.n, k = wp.cfg.k;
  int off[kMaxG + 1];
  c2_offsets(wp, off);
  // tile clients and the outer digit map (the non-tile clients, highest first)
  const int x1 = 31 - __clz(wp.cfg.mask[k - 3]), x2 = 31 - __clz(wp.cfg.mask[k - 2]),
            x3 = 31 - __clz(wp.cfg.mask[k - 1]);
  const uint32_t tmask = (1u << x1) | (1u << x2) | (1u << x3);
  tbits = (3u << (2 * (n - 1 - x1))) | (3u << (2 * (n - 1 - x2))) | (3u << (2 * (n - 1 - x3)));
  const int nout = n - 3;
  if (lane == 0) {
    int t = 0;
    for (int i = n - 1; i >= 0; i--)
      if (!(tmask >> i & 1u)) wp.oc[t++] = (int8_t)i;
  }
  __syncwarp();
  // slot / weight of a client: slot(g) = g for fixed groups, 5 + (g - (k-3)) for A, B, C;
  // weight 4^(members of g above i)
  auto slot_w = [&](int i, int &slot, int &w) {
    const int g = wp.cfg.a[i];
    slot = g < k - 3 ? g : 5 + (g - (k - 3));
    w = 1 << (2 * __popc(wp.cfg.mask[g] >> (i + 1)));
  };
  // lane part: o bits 0..4 = digit 0, digit 1, low bit of digit 2
#pragma unroll
  for (int q = 0; q < kC2Slots; q++) {  // slot q -> group (fixed slots beyond k-4: the pad, index 0)
    const int g = q < 5 ? q : (k - 3) + (q - 5);
    idxL[q] = (q < 5 && q >= k - 3) ? 0 : off[g];
  }
  voL = 0;
  for (int t = 0; t < 3 && t < nout; t++) {
    const uint32_t dgt = t < 2 ? ((uint32_t)lane >> (2 * t)) & 3u : ((uint32_t)lane >> 4) & 1u;
    int sl, w;
    const int i = wp.oc[t];
    slot_w(i, sl, w);
#pragma unroll
    for (int q = 0; q < kC2Slots; q++)
      if (q == sl) idxL[q] += (int)dgt * w;
    voL += dgt << (2 * (n - 1 - i));
  }
  // st bit b = o bit b + 5: digit t = (b + 5) / 2, value 1 << ((b + 5) & 1)
  if (lane < kC2Bits) {
    const int b = lane, ob = b + 5, t = ob >> 1;
#pragma unroll
    for (int q = 0; q <= kC2Slots; q++) wp.wb[b][q] = 0;
    if (t < nout) {
      const int i = wp.oc[t], val = 1 << (ob & 1);
      int sl, w;
      slot_w(i, sl, w);
      wp.wb[b][sl] = val * w;
      wp.wb[b][kC2Slots] = (int)((uint32_t)val << (2 * (n - 1 - i)));
    }
  }
  __syncwarp();
  if (lane < kC2Bits) {
    const int c = lane;
#pragma unroll
    for (int q = 0; q <= kC2Slots; q++) {
      int dd = wp.wb[c][q];
      for (int b = 0; b < c; b++) dd -= wp.wb[b][q];
      wp.d[c][q] = dd;
    }
  }
  __syncwarp();
}

// index of outer string o's configurations with tile digits 0 (vo) -- the
// non-tile clients' digits at their index positions (client 0 most significant)
__device__ __forceinline__ uint32_t c2_vo(const C2Warp &wp, int n, uint32_t o) {
  uint32_t vo = 0;
  for (int t = 0; t < n - 3; t++) vo |= ((o >> (2 * t)) & 3u) << (2 * (n - 1 - wp.oc[t]));
  return vo;
}

// Slow path of one tile (outer string o): exact fp64 group values, then every
// configuration of the tile inside [v0, v1) through ct_check.
template <int WM>
__device__ __noinline__ int c2_tile_slow(const Tables &tb, const DevParams &p, const Stair &stair, const C2Warp &wp,
                                         float *thr, BestRec *lb, uint32_t o, uint32_t vo, uint32_t v0, uint32_t v1,
                                         float Tp, float Ep, const float *At, const float *Ae, const float *Bt,
                                         const float *Be, const float *Ct, const float *Ce) {
  const int n = p.n, k = wp.cfg.k;
  uint32_t lw = 0;
  for (int t = 0; t < n - 3; t++) lw |= ((o >> (2 * t)) & 3u) << (2 * wp.oc[t]);
  const uint32_t ma = wp.cfg.mask[k - 3], mb = wp.cfg.mask[k - 2], mc = wp.cfg.mask[k - 1];
  const int x1 = 31 - __clz(ma), x2 = 31 - __clz(mb), x3 = 31 - __clz(mc);
  const int s1 = 2 * (n - 1 - x1), s2 = 2 * (n - 1 - x2), s3 = 2 * (n - 1 - x3);
  double Tp64 = 0.0, Ep64 = 0.0;
  for (int g = 0; g < k - 3; g++) {
    double Tg, Eg;
    ct_group64(tb, p, wp.cfg.mask[g], lw, Tg, Eg);
    if (Tg > Tp64) Tp64 = Tg;
    Ep64 = __dadd_rn(Ep64, Eg);
  }
  double A64[4], AE64[4], B64[4], BE64[4], C64[4], CE64[4];
#pragma unroll 1
  for (int l = 0; l < 4; l++) {
    const uint32_t ll = ct_set(ct_set(ct_set(lw, x1, l), x2, l), x3, l);
    ct_group64(tb, p, ma, ll, A64[l], AE64[l]);
    ct_group64(tb, p, mb, ll, B64[l], BE64[l]);
    ct_group64(tb, p, mc, ll, C64[l], CE64[l]);
  }
  int nref = 0;
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
        nref += ct_check<WM>(p, stair, thr, lb, wp.base + v, T, E, [&](double &T64, double &E64) {
          T64 = fmax(fmax(fmax(Tp64, A64[a]), B64[b]), C64[c]);
          E64 = __dadd_rn(__dadd_rn(__dadd_rn(Ep64, AE64[a]), BE64[b]), CE64[c]);
        });
      }
  return nref;
}

// Per-configuration path for a partition with k < 3 groups (no tile):
// scores from the group tables, exact values by refine64.
template <int WM>
__device__ __noinline__ int c2_small(const Tables &tb, const DevParams &p, const Stair &stair, const C2Warp &wp,
                                     float *thr, BestRec *lb, uint32_t v0, uint32_t v1, int lane) {
  const int n = p.n, k = wp.cfg.k;
  int off[kMaxG + 1];
  c2_offsets(wp, off);
  int nref = 0;
  int lam[kMaxN];
  for (uint32_t v = v0 + lane; v < v1; v += 32) {
    for (int i = 0; i < n; i++) lam[i] = (int)(v >> (2 * (n - 1 - i))) & 3;
    float T = 0.f, E = 0.f;
    for (int g = 0; g < k; g++) {
      uint32_t var = 0;
      for (uint32_t mm = wp.cfg.mask[g]; mm; mm &= mm - 1) var = var * 4 + (uint32_t)lam[__ffs(mm) - 1];
      const float2 te = wp.tab[off[g] + (int)var];
      T = fmaxf(T, te.x);
      E += te.y;
    }
    nref += ct_check<WM>(p, stair, thr, lb, wp.base + v, T, E, [&](double &T64, double &E64) {
      refine64(tb, p, wp.cfg.mask, k, lam, &T64, &E64);
    });
  }
  return nref;
}

template <int WM>
__global__ void __launch_bounds__(kC2Threads, 1) k_ctile2(const DevParams p) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned char *after = sm + ((p.blob_bytes + 15) & ~15u);
  Stair stair = stair_at(after);
  const StairSm ss = stair_sm(stair);
  C2Warp *wps = (C2Warp *)(after + kStairSmem);
  C2Warp &wp = wps[warp];
  BestRec *red = (BestRec *)(wps + kC2Warps);
  stair_init(stair);
  if (lane == 0) {
    wp.ncfg = 0;
    wp.nfeas = 0;
    wp.sver = 0;
  }
  __syncthreads();

  float thr[WM];
  BestRec lb[WM];
#pragma unroll
  for (int w = 0; w < WM; w++) {
    thr[w] = __int_as_float(0x7f800000);
    best_init(lb[w]);
  }
  int nref = 0;
  const int n = p.n;
  const int ul = p.unit_log2, cl = p.chunk_log2;
  double *t64 = p.c2t64 + ((size_t)blockIdx.x * kC2Warps + warp) * kC2Tab;

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
    if (lane == 0) {
      dev_unrank(tb, p, s, wp.cfg);
      wp.base = s - wp.cfg.v;
    }
    __syncwarp();
    for (;;) {
      if (p.want_pareto) {
        u64 sv = wp.sver;
        stair_sync(stair, p, sv, __ldcg(p.ctr + kCtrStairVer));
        __syncwarp();
        if (lane == 0) wp.sver = sv;
      }
      const u64 base = wp.base;
      const uint32_t Pn = (uint32_t)wp.cfg.Pn;
      const int k = wp.cfg.k;
      const bool feas = wp.cfg.feasible;
      const uint32_t v0 = s > base ? (uint32_t)(s - base) : 0u;
      const uint32_t v1 = e - base < (u64)Pn ? (uint32_t)(e - base) : Pn;
      __syncwarp();  // every lane has read the partition descriptor before lane 0 updates the warp's counters
      if (lane == 0) {
        wp.ncfg += v1 - v0;
        if (feas) wp.nfeas += v1 - v0;
      }
      if (feas) {
        int idxL[kC2Slots];
        uint32_t voL, tbits;
        const float ptmin = c2_tables(tb, p, wp, lane, t64);
        // the partition-wide staircase bound (as in the tile kernel)
        const unsigned int pmp = p.want_pareto ? stair_pm_at(ss, p, __fmul_rd(ptmin, p.tlb_scale_f)) : 0xffffffffu;
        if (k < 3) {
          nref += c2_small<WM>(tb, *p.gp, stair, wp, thr, lb, v0, v1, lane);
        } else {
          c2_setup(p, wp, lane, idxL, voL, tbits);
          const uint32_t nout = 1u << (2 * (n - 3));
          // outer strings whose tiles can meet [v0, v1): monotone in o for fixed
          // tile digits, so [first o with vo|tbits >= v0, last o with vo < v1]
          uint32_t o_lo = 0, o_hi = nout;  // [o_lo, o_hi)
          if (v0 > 0 || v1 < Pn) {
            uint32_t lo = 0, hi = nout;
            while (lo < hi) {
              const uint32_t mid = (lo + hi) >> 1;
              if ((c2_vo(wp, n, mid) | tbits) >= v0) hi = mid;
              else lo = mid + 1;
            }
            o_lo = lo;
            lo = o_lo;
            hi = nout;
            while (lo < hi) {
              const uint32_t mid = (lo + hi) >> 1;
              if (c2_vo(wp, n, mid) < v1) lo = mid + 1;
              else hi = mid;
            }
            o_hi = lo;
          }
          // seed pass (p.c2_seed_tiles): the unit's index range only picks a
          // place in the partition; from there 32 whole steps of tiles are
          // sampled (32 x 32 tiles = 2^16 configurations, as many as the
          // unit) -- a 2^16-index range cuts every tile whose clients carry
          // high index digits, which sent the seed pass configuration by
          // configuration (56 of 213 ms of a c3-client slice)
          uint32_t tv0 = v0, tv1 = v1;
          if (p.c2_seed_tiles) {
            o_lo &= ~31u;
            o_hi = min(nout, o_lo + 32u * 32u);
            tv0 = 0;
            tv1 = Pn;
          }
          const uint32_t st_lo = o_lo >> 5, st_hi = (o_hi + 31) >> 5;
          const bool inner = tv0 == 0 && tv1 == Pn && o_lo == 0 && o_hi == nout && (nout & 31u) == 0;
          // warp-uniform part of the table indices at st_lo
          int idxS[kC2Slots];
          uint32_t voS = 0;
#pragma unroll
          for (int q = 0; q < kC2Slots; q++) idxS[q] = 0;
          for (int b = 0; b < kC2Bits; b++)
            if (st_lo >> b & 1u) {
#pragma unroll
              for (int q = 0; q < kC2Slots; q++) idxS[q] += wp.wb[b][q];
              voS += (uint32_t)wp.wb[b][kC2Slots];
            }
          for (uint32_t st = st_lo; st < st_hi; st++) {
            // seed pass: thresholds and staircase refreshed every 4 steps (the
            // pass starts from nothing; every lane's first tiles are re-checked
            // configuration by configuration until they are)
            if (p.c2_seed_tiles && ((st - st_lo) & 3u) == 3u) {
#pragma unroll
              for (int w = 0; w < WM; w++) {
                if (w < p.nw) {  // publish the warp's minimum, take the global one
                  float m = thr[w];
#pragma unroll
                  for (int o = 16; o; o >>= 1) m = fminf(m, __shfl_xor_sync(0xffffffffu, m, o));
                  if (lane == 0 && m < __uint_as_float(__ldcg(p.thr + w))) atomicMin(p.thr + w, __float_as_uint(m));
                  thr[w] = fminf(thr[w], __uint_as_float(__ldcg(p.thr + w)));
                }
              }
              if (p.want_pareto) {
                u64 sv = wp.sver;
                stair_sync(stair, p, sv, __ldcg(p.ctr + kCtrStairVer));
                __syncwarp();
                if (lane == 0) wp.sver = sv;
              }
            }
            if (st > st_lo) {  // st - 1 -> st: delta row of its trailing-ones count
              const int c = __ffs(~(st - 1)) - 1;
#pragma unroll
              for (int q = 0; q < kC2Slots; q++) idxS[q] += wp.d[c][q];
              voS += (uint32_t)wp.d[c][kC2Slots];
            }
            const uint32_t o = (st << 5) | (uint32_t)lane;
            const uint32_t vo = voS + voL;
            // a unit covering the whole partition (the main pass: units of a
            // partition's 4^n configurations) needs no per-tile range checks
            bool whole = true;
            if (!inner) {
              if (o < o_lo || o >= o_hi || (vo | tbits) < tv0 || vo >= tv1) continue;
              whole = vo >= tv0 && (vo | tbits) < tv1;
            }
            float Tp = 0.f, Ep = 0.f;
#pragma unroll
            for (int q = 0; q < 5; q++) {
              const float2 te = wp.tab[idxS[q] + idxL[q]];
              Tp = fmaxf(Tp, te.x);
              Ep += te.y;
            }
            float At[4], Ae[4], Bt[4], Be[4], Ct[4], Ce[4];
            {
              const float4 *ta = (const float4 *)&wp.tab[idxS[5] + idxL[5]];
              const float4 *tbb = (const float4 *)&wp.tab[idxS[6] + idxL[6]];
              const float4 *tc = (const float4 *)&wp.tab[idxS[7] + idxL[7]];
              const float4 a0 = ta[0], a1 = ta[1], b0 = tbb[0], b1 = tbb[1], c0 = tc[0], c1 = tc[1];
              At[0] = a0.x; Ae[0] = a0.y; At[1] = a0.z; Ae[1] = a0.w;
              At[2] = a1.x; Ae[2] = a1.y; At[3] = a1.z; Ae[3] = a1.w;
              Bt[0] = b0.x; Be[0] = b0.y; Bt[1] = b0.z; Be[1] = b0.w;
              Bt[2] = b1.x; Be[2] = b1.y; Bt[3] = b1.z; Be[3] = b1.w;
              Ct[0] = c0.x; Ce[0] = c0.y; Ct[1] = c0.z; Ce[1] = c0.w;
              Ct[2] = c1.x; Ce[2] = c1.y; Ct[3] = c1.z; Ce[3] = c1.w;
            }
            if (whole) {
              // the tile's 64 configurations, min-reduced to the exact lower corner
              float mT = __int_as_float(0x7f800000), mE = mT;
#pragma unroll
              for (int a = 0; a < 4; a++) {
                const float T1 = fmaxf(Tp, At[a]), E1 = Ep + Ae[a];
#pragma unroll
                for (int b = 0; b < 4; b++) {
                  const float E2 = E1 + Be[b];
#pragma unroll
                  for (int c = 0; c < 4; c++) {
                    mT = fminf(mT, fmax3f(T1, Bt[b], Ct[c]));  // T: one FMNMX3 per configuration
                    mE = fminf(mE, E2 + Ce[c]);
                  }
                }
              }
              // the fp32 staircase screen first: a corner it discards is
              // dominated by a verified configuration with margin (E > E_p
              // (1 + 4u)), so when every weight has b >= 1
              // no configuration of the tile reaches or ties any weight's
              // optimum and the weight screen is skipped
              const bool fdom = p.want_pareto && (__float_as_uint(mE) > pmp ||
                                                  stair_dominated_fs(ss, p, __fmul_rd(mT, p.tlb_scale_f), mE));
              bool hit = false;
              if (!(fdom && p.wb_pos)) {
#pragma unroll
                for (int w = 0; w < WM; w++) {
                  if (w < p.nw) {
                    float q = 1.f;
                    for (int i = 0; i < p.wa[w]; i++) q *= mT;
                    for (int i = 0; i < p.wb[w]; i++) q *= mE;
                    hit |= q <= thr[w] * p.mul[w];
                  }
                }
              }
              bool par = p.want_pareto && !fdom;
              if (par) {  // the fp32 screen cannot decide: the tile's exact fp64 corner makespan
                double c = 0.0;
#pragma unroll
                for (int q = 0; q < 5; q++) c = fmax(c, __ldcg(t64 + idxS[q] + idxL[q]));
#pragma unroll
                for (int q = 5; q < 8; q++) {
                  const double *tq = t64 + idxS[q] + idxL[q];
                  c = fmax(c, fmin(fmin(__ldcg(tq), __ldcg(tq + 1)), fmin(__ldcg(tq + 2), __ldcg(tq + 3))));
                }
                par = !stair_dominated(stair, p, c, mE);
              }
              if (!hit && !par) continue;
            }
            nref += c2_tile_slow<WM>(tb, *p.gp, stair, wp, thr, lb, o, vo, tv0, tv1, Tp, Ep, At, Ae, Bt, Be, Ct, Ce);
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
  for (int o = 16; o; o >>= 1) nref64 += __shfl_xor_sync(0xffffffffu, nref64, o);
  __syncwarp();
  if (lane == 0) {
    atomicAdd(p.ctr + kCtrConfigs, wp.ncfg);
    atomicAdd(p.ctr + kCtrFeasible, wp.nfeas);
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
  if ((int)threadIdx.x < p.nw) {
    const int w = threadIdx.x;
    BestRec b = red[w];
    for (int q = 1; q < kC2Warps; q++) {
      const BestRec x = red[q * kMaxW + w];
      if (x.valid && (!b.valid || better(x.f, x.idx, b.f, b.idx))) b = x;
    }
    ((BestRec *)p.slots)[(size_t)blockIdx.x * p.nw + w] = b;
  }
}

template <int WM>
const void *ctile2_fn() {
  return (const void *)k_ctile2<WM>;
}

}  // namespace sched
