// search_sfx.cuh -- L = 1 suffix kernel (c5 fast path), lane-parallel.
//
// With one MPS level every configuration is a set partition (RGS) and the
// score decomposes over groups:
//   T = max_g T_g,  E = sum_g E_g.
// A warp walks *prefixes*: partitions of workflows 0..n-M-1 (the first
// n-M entries of the RGS).  The completions of a prefix -- the placements of
// the last M workflows x_0..x_{M-1} (the "suffix") in lexicographic RGS
// order -- are consecutive indices [base, base + W_prefix).  Per prefix:
//   * the warp fills a table row per group r (prefix group P_r, or an empty
//     "new group" row) over every suffix subset S: (t, de) =
//       ( T(P_r u S) / T_seq ,  (E(P_r u S) - E(P_r u S \ max S)) / E_seq )
//     from the exact fp64 group tuples (k_groups table, L2-resident), each
//     rounded once to fp32.  Rows are rebuilt only when the prefix group
//     changes (consecutive prefixes share most groups).
//   * the prefix's completions are split into 32 equal ordinal ranges; each
//     lane unranks its start through the DP count table and enumerates its
//     range in lexicographic order with M nested loops.  Placing x_i in group
//     j reads one table entry (S_j | bit i) and updates
//       T <- max(T, t),  E <- E + de
//     (exact chain: adding the highest-numbered member appends one term to
//     every ascending sum of the canonical group score, so T_g is monotone
//     and the running max equals the max over the final groups; E
//     telescopes).  Every configuration's (T, E) is computed and
//     min-reduced per lane (4 fp32 ops per configuration).
//   * the lane's exact lower corner (min T, min E) is screened once against
//     the per-weight thresholds (q_w is monotone in T and E) and the Pareto
//     staircase; a lane that is not cleared re-enumerates its range checking
//     every configuration (fp32 screens, fp64 canonical re-score from the
//     exact group tuples, lowest-index ties), like the other kernels.
// fp32 error: T carries <= 2u, E <= (kp + M + 2)u (sum of non-negative terms
// each within 2u), inside the host's eps_T / eps_E (host_core.cpp), so the
// screens of DESIGN.md section 5 stay complete.
#pragma once
#include "device_common.cuh"
#include "search_tile.cuh"

namespace sched {

#ifndef SCHED_SFX_THREADS
#define SCHED_SFX_THREADS 512  // one 512-thread CTA per SM (c5: 485 ms vs 500 at 256 x 2; M = 7 tables need it)
#endif
#ifndef SCHED_SFX_MINB
#define SCHED_SFX_MINB 1
#endif
constexpr int kSfxThreads = SCHED_SFX_THREADS;
constexpr int kSfxWarps = kSfxThreads / 32;
constexpr int kSfxMaxG = 8;

template <int M>
struct SfxWarp {
  static constexpr int RS = (1 << M) + 1;  // row stride (float2): +1 staggers the banks of rows
  LaneCfg cfg;                             // the prefix (workflows 0..n-M-1), lane 0 owns it
  u64 base;                                // index of the prefix's first completion
  uint32_t key[kSfxMaxG];                  // row content: prefix group mask, 0 = new-group row
  int flag;
  float2 tab[kSfxMaxG * RS];               // (t, de) per (row, suffix subset)
};

struct SfxLane {   // per-lane suffix state (registers)
  u64 gi;          // byte j: suffix subset S_j placed in group j
  uint32_t rr;     // nibble j: remaining room of group j (C - size, saturated at 15)
  uint32_t rm;     // bit j: group j has room
  int kc;          // open groups
  float T, E;      // fp32 normalised makespan / energy so far
};

struct SfxHot {    // fast-pass accumulators (registers)
  float mT, mE;
  int nf, cnt;
  uint32_t ord;    // ordinal of the next configuration within the prefix
};

struct SfxCold {   // slow-pass state (local memory)
  float thr[kMaxW];
  BestRec lb[kMaxW];
  int nref;
};

struct SfxCtx {    // read-only per-prefix context
  const float2 *tab;
  int G, C, start[8];
  int kp, off;     // prefix groups, suffix bit offset (n - M)
  u64 base;
  const uint32_t *pmask;  // prefix group masks (shared)
};

__device__ __forceinline__ uint32_t sfx_opts(const SfxLane &s, int G) {
  return s.rm | (s.kc < G ? 1u << s.kc : 0u);
}

__device__ __forceinline__ void sfx_apply(SfxLane &s, int j, uint32_t bi, float2 v, int C) {
  s.T = fmaxf(s.T, v.x);
  s.E = s.E + v.y;
  // branchless: a new group (j == kc) gets room min(C-1, 15) in its (zero)
  // nibble, an existing one loses one unit of room
  const bool nw = j == s.kc;
  const uint32_t room = (uint32_t)(C - 1 < 15 ? C - 1 : 15);
  s.kc += nw ? 1 : 0;
  s.rr += (nw ? room : 0xffffffffu) << (4 * j);
  const uint32_t has = ((s.rr >> (4 * j)) & 15u) ? 1u : 0u;
  s.rm = (s.rm & ~(1u << j)) | (has << j);
  s.gi |= (u64)bi << (8 * j);
}

// One configuration of the slow pass: fp32 screens, fp64 canonical re-score
// (T = max of exact group T_g, E = sum of exact E_g in block order), record.
static __device__ __noinline__ void sfx_check(const DevParams &p, const Stair &stair, const SfxCtx &x, SfxCold *cold,
                                       u64 gi, int kc, float T, float E, u64 idx) {
  if (!(T < __int_as_float(0x7f800000))) return;  // memory-infeasible
  unsigned need = 0;
#pragma unroll
  for (int w = 0; w < kMaxW; w++) {
    if (w < p.nw) {
      float q = 1.f;
      for (int i = 0; i < p.wa[w]; i++) q *= T;
      for (int i = 0; i < p.wb[w]; i++) q *= E;
      if (q <= fminf(cold->thr[w], q) * p.mul[w]) need |= 1u << w;
      cold->thr[w] = fminf(cold->thr[w], q);
    }
  }
  const bool par = p.want_pareto && !stair_dominated_f(stair, p, __fmul_rd(T, p.tlb_scale_f), E);
  if (!need && !par) return;
  const GroupRec *gtab = (const GroupRec *)p.gtab;
  double T64 = 0.0, E64 = 0.0;
  for (int g = 0; g < kc; g++) {
    const uint32_t m = (g < x.kp ? x.pmask[g] : 0u) | ((uint32_t)((gi >> (8 * g)) & 0xffu) << x.off);
    const GroupRec r = gtab[m];
    T64 = fmax(T64, r.t64);
    E64 = __dadd_rn(E64, r.e64);
  }
  // weights with b = 0 (F = X^a depends on T alone): a best with makespan
  // <= T64 at a lower index cannot be replaced (F <= its F, index higher) --
  // exact early reject that stops the (1,0) tie flood
#pragma unroll
  for (int w = 0; w < kMaxW; w++)
    if (w < p.nw && (need >> w & 1u) && p.wb[w] == 0 && cold->lb[w].valid && T64 >= cold->lb[w].t &&
        idx > cold->lb[w].idx)
      need &= ~(1u << w);
  if (!need && !par) return;
  cold->nref++;
#pragma unroll
  for (int w = 0; w < kMaxW; w++) {
    if (w < p.nw && (need >> w & 1u)) {
      const double F = objective64(p, T64, E64, p.wa[w], p.wb[w]);
      BestRec &b = cold->lb[w];
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
  if (par && !stair_dominated(stair, p, T64, __double2float_rd(__ddiv_rd(E64, p.eseq))) &&
      !stair_dominated_exact(stair, p, T64, E64))
    emit_candidate(p, stair, idx, T64, E64, T, E);
}

// The last level (suffix element M-1) over the option set `opts` of state
// st: every option is one configuration.  FAST: (T, E) and the lane's
// min-reduction (the loop carries no count or order bookkeeping; options
// are taken highest first); CHECK: ascending (lexicographic) order with the
// exact ordinal, per-configuration screens.  lim bounds the number taken.
template <int M, bool CHECK>
__device__ __forceinline__ void sfx_last(const DevParams &p, const Stair &stair, const SfxCtx &x, SfxHot &h,
                                         SfxCold *cold, const SfxLane &st, uint32_t opts) {
  constexpr int RS = SfxWarp<M>::RS;
  constexpr uint32_t bl = 1u << (M - 1);
  if constexpr (!CHECK) {
    float mT = h.mT, mE = h.mE;
    int nf = h.nf;
    while (opts) {
      uint32_t j;
      asm("bfind.u32 %0, %1;" : "=r"(j) : "r"(opts));
      opts ^= 1u << j;
      const float2 v = x.tab[j * RS + (((uint32_t)(st.gi >> (8 * j)) & 0xffu) | bl)];
      const float T = fmaxf(st.T, v.x), E = st.E + v.y;
      mT = fminf(mT, T);
      mE = fminf(mE, E);
      nf += (int)((__float_as_uint(T) - 0x7f800000u) >> 31);  // T < +inf (T >= 0)
    }
    h.mT = mT;
    h.mE = mE;
    h.nf = nf;
  } else {
    while (opts) {
      const int j = __ffs(opts) - 1;
      opts &= opts - 1;
      const float2 v = x.tab[j * RS + (((uint32_t)(st.gi >> (8 * j)) & 0xffu) | bl)];
      const float T = fmaxf(st.T, v.x), E = st.E + v.y;
      const int kc = st.kc + (j == st.kc ? 1 : 0);
      sfx_check(p, stair, x, cold, st.gi | ((u64)bl << (8 * j)), kc, T, E, x.base + h.ord);
      h.ord++;
    }
  }
}

// m without its `lim` lowest set bits
__device__ __forceinline__ uint32_t strip_low(uint32_t m, int lim) {
  for (; lim > 0 && m; lim--) m &= m - 1;
  return m;
}

// Level I < M-1 of the lexicographic enumeration (placement of suffix
// element I).  first: still on the first descent (start at the unranked
// choice start[I]).  h.cnt = configurations left in the lane's range; the
// level above the last checks it once per option, so the last level runs
// without bookkeeping.
template <int M, int I, bool CHECK>
__device__ __forceinline__ void sfx_level(const DevParams &p, const Stair &stair, const SfxCtx &x, SfxHot &h,
                                          SfxCold *cold, const SfxLane &st, bool first) {
  constexpr int RS = SfxWarp<M>::RS;
  uint32_t opts = sfx_opts(st, x.G);
  if (first) opts &= ~0u << x.start[I];
  const uint32_t bi = 1u << I;
  while (opts) {
    const int j = __ffs(opts) - 1;
    opts &= opts - 1;
    const float2 v = x.tab[j * RS + (((uint32_t)(st.gi >> (8 * j)) & 0xffu) | bi)];
    SfxLane s2 = st;
    sfx_apply(s2, j, bi, v, x.C);
    if constexpr (I == M - 2) {
      uint32_t o2 = sfx_opts(s2, x.G);
      if (first) o2 &= ~0u << x.start[M - 1];
      const int n2 = __popc(o2);
      if (h.cnt > n2) {
        sfx_last<M, CHECK>(p, stair, x, h, cold, s2, o2);
        h.cnt -= n2;
      } else {  // the lane's range ends inside this option set
        sfx_last<M, CHECK>(p, stair, x, h, cold, s2, o2 & ~strip_low(o2, h.cnt));
        h.cnt = 0;
        return;
      }
    } else {
      sfx_level<M, I + 1, CHECK>(p, stair, x, h, cold, s2, first);
      if (h.cnt == 0) return;
    }
    first = false;
  }
}

// ---- fast pass: converged per-parent loop ----
// A parent is a state after x_0..x_{M-2}; its configurations are the options
// of the last element.  sfx_slots evaluates them over the 8 row slots
// without branches: a full group's entry (|S| > cap) is (+inf, +inf); rows
// >= G hold (+inf, +inf); slots kc+1 .. G-1 are empty "new" rows whose entry
// repeats the new-group configuration of slot kc (mins unchanged, the
// feasible count is corrected).  Every lane runs the same instructions.
template <int M>
__device__ __forceinline__ void sfx_slots(const float2 *tab, const SfxLane &s, int G, float &mT, float &mE,
                                          int &nf) {
  constexpr int RS = SfxWarp<M>::RS;
  constexpr uint32_t bl = 1u << (M - 1);
  const uint32_t lo = (uint32_t)s.gi, hi = (uint32_t)(s.gi >> 32);
  int c = 0;
#pragma unroll
  for (int j = 0; j < kSfxMaxG; j++) {
    const uint32_t S = __byte_perm(j < 4 ? lo : hi, 0u, 0x4440u | (uint32_t)(j & 3));
    const float2 v = tab[j * RS + bl + S];  // S | bl == S + bl
    const float T = fmaxf(s.T, v.x), E = s.E + v.y;
    mT = fminf(mT, T);
    mE = fminf(mE, E);
    c += (int)((__float_as_uint(T) - 0x7f800000u) >> 31);
  }
  if (s.kc < G - 1) {  // duplicates of the new-group configuration
    const float T = fmaxf(s.T, tab[(G - 1) * RS + bl].x);
    c -= (G - 1 - s.kc) * (int)((__float_as_uint(T) - 0x7f800000u) >> 31);
  }
  nf += c;
}

// next option at level I (I <= M-2) and the first parent below it; false
// when level I is exhausted.  st[I] = state before x_I, rem[I] = options left.
template <int M, int I>
__device__ __forceinline__ bool sfx_adv(const SfxCtx &x, SfxLane (&st)[M - 1], uint32_t (&rem)[M - 1],
                                        SfxLane &par) {
  constexpr int RS = SfxWarp<M>::RS;
  while (rem[I]) {
    const int j = __ffs(rem[I]) - 1;
    rem[I] &= rem[I] - 1;
    const float2 v = x.tab[j * RS + (((uint32_t)(st[I].gi >> (8 * j)) & 0xffu) | (1u << I))];
    SfxLane s = st[I];
    sfx_apply(s, j, 1u << I, v, x.C);
    if constexpr (I == M - 2) {
      par = s;
      return true;
    } else {
      st[I + 1] = s;
      rem[I + 1] = sfx_opts(s, x.G);
      if (sfx_adv<M, I + 1>(x, st, rem, par)) return true;
    }
  }
  return false;
}

template <int M, int I>
__device__ __forceinline__ bool sfx_next(const SfxCtx &x, SfxLane (&st)[M - 1], uint32_t (&rem)[M - 1],
                                         SfxLane &par) {
  if (sfx_adv<M, I>(x, st, rem, par)) return true;
  if constexpr (I == 0) {
    return false;
  } else {
    return sfx_next<M, I - 1>(x, st, rem, par);
  }
}

// Fast pass over the lane range starting at the unranked choices x.start
// (state s0 before x_0), cnt configurations.
template <int M>
__device__ __forceinline__ void sfx_fast(const DevParams &p, const Stair &stair, const SfxCtx &x, SfxHot &h,
                                         const SfxLane &s0, int cnt) {
  constexpr int RS = SfxWarp<M>::RS;
  SfxLane st[M - 1], par;
  uint32_t rem[M - 1];
  st[0] = s0;
#pragma unroll
  for (int I = 0; I < M - 1; I++) {
    const int j = x.start[I];
    rem[I] = sfx_opts(st[I], x.G) & (~1u << j);  // options after the start choice
    const float2 v = x.tab[j * RS + (((uint32_t)(st[I].gi >> (8 * j)) & 0xffu) | (1u << I))];
    SfxLane s = st[I];
    sfx_apply(s, j, 1u << I, v, x.C);
    if (I < M - 2) st[I + 1] = s;
    else par = s;
  }
  uint32_t o = sfx_opts(par, x.G) & (~0u << x.start[M - 1]);
  for (;;) {
    const int n = __popc(o);
    if (cnt <= n) {  // the lane's range ends in this parent
      sfx_last<M, false>(p, stair, x, h, nullptr, par, o & ~strip_low(o, cnt));
      return;
    }
    if (o == sfx_opts(par, x.G)) sfx_slots<M>(x.tab, par, x.G, h.mT, h.mE, h.nf);
    else sfx_last<M, false>(p, stair, x, h, nullptr, par, o);  // the partial first parent
    cnt -= n;
    if (!sfx_next<M, M - 2>(x, st, rem, par)) return;
    o = sfx_opts(par, x.G);
  }
}

// ---- fast pass over grandparents (SCHED_SFX_PAIRS, default) ----
// A grandparent is a state after x_0..x_{M-3}; its configurations are the
// placements (j1, j2) of the last two elements x_{M-2}, x_{M-1}.  sfx_pairs
// evaluates them as a register tile: the 8 slots of x_{M-1} (B entries: the
// row's suffix subset S_j plus x_{M-1}; rows above the grandparent's kc read
// +inf, full groups read +inf from the table itself) for every option j1 of
// x_{M-2} (A entry: S_j1 plus x_{M-2}), and both in the same group (D entry:
// S_j1 plus both); the placement in two new groups (kc, kc + 1) is evaluated
// on its own.  Per configuration T = max(T_g, t_A, t_B), E = (E_g + e_A) + e_B
// (the chain order of sfx_apply), min-reduced; the feasible count comes from
// the finite masks of A, B, D (no per-configuration count).
template <int M>
__device__ __forceinline__ void sfx_pairs(const float2 *tab, const SfxLane &g, int G, float &mT, float &mE, int &nf) {
  constexpr int RS = SfxWarp<M>::RS;
  constexpr uint32_t bA = 1u << (M - 2), bB = 1u << (M - 1);
  const float inf = __int_as_float(0x7f800000);
  const uint32_t lo = (uint32_t)g.gi, hi = (uint32_t)(g.gi >> 32);
  // B: x_{M-1} alone in slot j2 (rows above kc unused: +inf)
  float tB[kSfxMaxG], eB[kSfxMaxG];
  uint32_t fB = 0;
#pragma unroll
  for (int j = 0; j < kSfxMaxG; j++) {
    const uint32_t S = __byte_perm(j < 4 ? lo : hi, 0u, 0x4440u | (uint32_t)(j & 3));
    const float2 b = tab[j * RS + (S | bB)];
    const bool used = j <= g.kc;
    tB[j] = used ? b.x : inf;
    eB[j] = used ? b.y : inf;
    fB |= (tB[j] < inf ? 1u : 0u) << j;
  }
  float lT = mT, lE = mE;
  uint32_t fA = 0, fD = 0;
  // x_{M-2} over its options j1 (existing groups with room, the new group kc)
  for (uint32_t oa = sfx_opts(g, G); oa;) {
    const int j1 = __ffs(oa) - 1;
    oa &= oa - 1;
    const uint32_t S = (uint32_t)(g.gi >> (8 * j1)) & 0xffu;
    const float2 a = tab[j1 * RS + (S | bA)], d = tab[j1 * RS + (S | bA | bB)];
    fA |= (a.x < inf ? 1u : 0u) << j1;
    fD |= (d.x < inf ? 1u : 0u) << j1;
    const float T1 = fmaxf(g.T, a.x), E1 = g.E + a.y;
    // the 8 slots of x_{M-1} with B entries, slot j1 included: that one is
    // not a configuration (x_{M-1} in j1 without x_{M-2}), its (T, E) only
    // lowers the min-reduced corner -- still a lower bound of every real
    // configuration's -- so the screen stays complete; the real placement
    // (both in j1) is the D entry
#pragma unroll
    for (int j2 = 0; j2 < kSfxMaxG; j2++) {
      lT = fminf(lT, fmaxf(T1, tB[j2]));
      lE = fminf(lE, E1 + eB[j2]);
    }
    lT = fminf(lT, fmaxf(T1, d.x));
    lE = fminf(lE, E1 + d.y);
  }
  // x_{M-2} in the new group kc, x_{M-1} in a second new group kc + 1
  int ext = 0;
  if (g.kc + 1 < G) {
    const float2 a = tab[g.kc * RS + bA], b = tab[(g.kc + 1) * RS + bB];
    const float T = fmaxf(fmaxf(g.T, a.x), b.x), E = (g.E + a.y) + b.y;
    lT = fminf(lT, T);
    lE = fminf(lE, E);
    ext = T < inf ? 1 : 0;
  }
  mT = lT;
  mE = lE;
  if (g.T < inf) nf += __popc(fA) * __popc(fB) - __popc(fA & fB) + __popc(fA & fD) + ext;
}

// configurations under a grandparent: sum over the options j1 of x_{M-2} of
// the option count of x_{M-1} (r existing groups with room, `one` of them
// with room 1, the new group if kc < G)
__device__ __forceinline__ int sfx_pairs_count(const SfxLane &g, int G, int C) {
  const int r = __popc(g.rm);
  const int na = g.kc < G ? 1 : 0;
  // groups (< kc) whose room nibble is exactly 1
  const uint32_t x = g.rr ^ 0x11111111u;                 // nibble == 1 -> 0
  const uint32_t z = ~(((x & 0x77777777u) + 0x77777777u) | x) & 0x88888888u;  // high bit of each zero nibble
  const uint32_t km = g.kc >= 8 ? 0xffffffffu : ((1u << (4 * g.kc)) - 1u);
  const int one = __popc(z & km);
  return r * (r + na) - one + na * (r + (C > 1 ? 1 : 0) + (g.kc + 1 < G ? 1 : 0));
}

// next option at level I (I <= M-3) and the first grandparent below it
template <int M, int I>
__device__ __forceinline__ bool sfx_gadv(const SfxCtx &x, SfxLane (&st)[M - 2], uint32_t (&rem)[M - 2],
                                         SfxLane &gp) {
  constexpr int RS = SfxWarp<M>::RS;
  while (rem[I]) {
    const int j = __ffs(rem[I]) - 1;
    rem[I] &= rem[I] - 1;
    const float2 v = x.tab[j * RS + (((uint32_t)(st[I].gi >> (8 * j)) & 0xffu) | (1u << I))];
    SfxLane s = st[I];
    sfx_apply(s, j, 1u << I, v, x.C);
    if constexpr (I == M - 3) {
      gp = s;
      return true;
    } else {
      st[I + 1] = s;
      rem[I + 1] = sfx_opts(s, x.G);
      if (sfx_gadv<M, I + 1>(x, st, rem, gp)) return true;
    }
  }
  return false;
}

template <int M, int I>
__device__ __forceinline__ bool sfx_gnext(const SfxCtx &x, SfxLane (&st)[M - 2], uint32_t (&rem)[M - 2],
                                          SfxLane &gp) {
  if (sfx_gadv<M, I>(x, st, rem, gp)) return true;
  if constexpr (I == 0) {
    return false;
  } else {
    return sfx_gnext<M, I - 1>(x, st, rem, gp);
  }
}

// the parents of grandparent gp whose x_{M-2} option is in remA, parent by
// parent (the first one's x_{M-1} options masked by ofirst); returns true
// when the lane's range (cnt) ends inside
template <int M>
__device__ __forceinline__ bool sfx_gp_parents(const DevParams &p, const Stair &stair, const SfxCtx &x, SfxHot &h,
                                               const SfxLane &gp, uint32_t remA, uint32_t ofirst, int &cnt) {
  constexpr int RS = SfxWarp<M>::RS;
  constexpr uint32_t bA = 1u << (M - 2);
  while (remA) {
    const int j = __ffs(remA) - 1;
    remA &= remA - 1;
    const float2 v = x.tab[j * RS + (((uint32_t)(gp.gi >> (8 * j)) & 0xffu) | bA)];
    SfxLane par = gp;
    sfx_apply(par, j, bA, v, x.C);
    const uint32_t oall = sfx_opts(par, x.G);
    const uint32_t o = oall & ofirst;
    ofirst = 0xffffffffu;
    const int n = __popc(o);
    if (cnt <= n) {
      sfx_last<M, false>(p, stair, x, h, nullptr, par, o & ~strip_low(o, cnt));
      cnt = 0;
      return true;
    }
    if (o == oall) sfx_slots<M>(x.tab, par, x.G, h.mT, h.mE, h.nf);
    else sfx_last<M, false>(p, stair, x, h, nullptr, par, o);
    cnt -= n;
  }
  return false;
}

// Fast pass over the lane range by grandparents: the first (partial) and the
// last (partial) grandparent parent by parent, the whole ones in between as
// pair tiles.
template <int M>
__device__ __forceinline__ void sfx_fast_pairs(const DevParams &p, const Stair &stair, const SfxCtx &x, SfxHot &h,
                                               const SfxLane &s0, int cnt) {
  constexpr int RS = SfxWarp<M>::RS;
  SfxLane st[M - 2], gp;
  uint32_t rem[M - 2];
  st[0] = s0;
#pragma unroll
  for (int I = 0; I < M - 2; I++) {
    const int j = x.start[I];
    rem[I] = sfx_opts(st[I], x.G) & (~1u << j);  // options after the start choice
    const float2 v = x.tab[j * RS + (((uint32_t)(st[I].gi >> (8 * j)) & 0xffu) | (1u << I))];
    SfxLane s = st[I];
    sfx_apply(s, j, 1u << I, v, x.C);
    if (I < M - 3) st[I + 1] = s;
    else gp = s;
  }
  if (sfx_gp_parents<M>(p, stair, x, h, gp, sfx_opts(gp, x.G) & (~0u << x.start[M - 2]), ~0u << x.start[M - 1],
                        cnt))
    return;
  for (;;) {
    if (!sfx_gnext<M, M - 3>(x, st, rem, gp)) return;
    const int np = sfx_pairs_count(gp, x.G, x.C);
    if (cnt <= np) {  // the lane's range ends in this grandparent
      sfx_gp_parents<M>(p, stair, x, h, gp, sfx_opts(gp, x.G), 0xffffffffu, cnt);
      return;
    }
    sfx_pairs<M>(x.tab, gp, x.G, h.mT, h.mE, h.nf);
    cnt -= np;
  }
}

// Slow pass over a lane range (out of line: keeps the fast pass's registers).
template <int M>
static __device__ __noinline__ void sfx_slow(const DevParams &p, const Stair &stair, const SfxCtx &x,
                                             SfxCold *cold, const SfxLane &s0, uint32_t l0, int cnt) {
  SfxHot h;
  h.mT = h.mE = 0.f;
  h.nf = 0;
  h.cnt = cnt;
  h.ord = l0;
  sfx_level<M, 0, true>(p, stair, x, h, cold, s0, true);
}

// lane start: unrank ordinal r within the prefix's completions (DP table),
// writing the first-descent choices into x.start
template <int M>
__device__ __forceinline__ void sfx_unrank(const Tables &tb, const DevParams &p, SfxCtx &x, const SfxLane &s0,
                                           int st0, uint32_t r) {
  SfxLane s = s0;
  int st = st0;
#pragma unroll
  for (int I = 0; I < M; I++) {
    uint32_t opts = sfx_opts(s, x.G);
    int jc = 0;
    while (opts) {
      const int j = __ffs(opts) - 1;
      opts &= opts - 1;
      int col;
      if (j == s.kc) col = 0;
      else col = p.capped ? x.C - (int)((s.rr >> (4 * j)) & 15u) : 1;
      const uint16_t s2 = tb.trans[st * p.tc + col];
      const u64 wv = s2 == kNoState ? 0ull : tb.W[s2];
      jc = j;
      if ((u64)r < wv) {
        st = s2;
        break;
      }
      r -= (uint32_t)wv;
    }
    x.start[I] = jc;
    sfx_apply(s, jc, 1u << I, make_float2(0.f, 0.f), x.C);
  }
}

// index -> prefix (RGS of workflows 0..plen-1) and the ordinal of idx among
// the prefix's completions
static __device__ uint32_t sfx_unrank_prefix(const Tables &tb, const DevParams &p, u64 idx, LaneCfg &c, int plen) {
  u64 r = idx;
  int s = p.root;
  c.k = 0;
  place(c, 0, 0);
  c.st[0] = (uint16_t)s;
  for (int i = 1; i < plen; i++) {
    int chosen = -1;
    for (int j = 0; j <= c.k; j++) {
      const int col = col_for(p, j, c.k, c.sz);
      if (col < 0) {
        if (j == c.k) break;
        continue;
      }
      const uint16_t s2 = tb.trans[s * p.tc + col];
      if (s2 == kNoState) continue;
      const u64 w = tb.W[s2];
      if (r < w) {
        chosen = j;
        s = s2;
        break;
      }
      r -= w;
    }
    if (chosen < 0) return 0;
    place(c, i, chosen);
    c.st[i] = (uint16_t)s;
  }
  return (uint32_t)r;
}

// next prefix in lexicographic order among completable ones (W > 0)
__device__ __forceinline__ bool sfx_prefix_successor(const Tables &tb, const DevParams &p, LaneCfg &c, int last) {
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

// (t, de) of one table entry: group = key | S (suffix bits at `off`)
// (values scaled by 1/T_seq, 1/E_seq: multiplication by a positive constant
// is monotone, so T stays monotone along every chain; relative error <= 2u)
__device__ __forceinline__ float2 sfx_entry(const DevParams &p, const GroupRec *gtab, uint32_t key, uint32_t S,
                                            int off, int cap, double its, double ies) {
  const float inf = __int_as_float(0x7f800000);
  if (S == 0u) {
    if (key == 0u) return make_float2(0.f, 0.f);
    const GroupRec g = gtab[key];
    if (!(g.t32 < inf)) return make_float2(inf, inf);
    return make_float2(__double2float_rn(__dmul_rn(g.t64, its)), __double2float_rn(__dmul_rn(g.e64, ies)));
  }
  if (__popc(S) > cap) return make_float2(inf, inf);
  const GroupRec cur = gtab[key | (S << off)];
  if (!(cur.t32 < inf)) return make_float2(inf, inf);
  const uint32_t Sp = S & ~(1u << (31 - __clz(S)));
  const uint32_t mp = key | (Sp << off);
  const double ep = mp ? gtab[mp].e64 : 0.0;
  return make_float2(__double2float_rn(__dmul_rn(cur.t64, its)),
                     __double2float_rn(__dmul_rn(__dsub_rn(cur.e64, ep), ies)));
}

template <int M>
__global__ void __launch_bounds__(kSfxThreads, SCHED_SFX_MINB) k_sfx(const DevParams p) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  constexpr int RS = SfxWarp<M>::RS;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned char *after = sm + ((p.blob_bytes + 15) & ~15u);
  Stair stair = stair_at(after);
  SfxWarp<M> *wps = (SfxWarp<M> *)(after + kStairSmem);
  SfxWarp<M> &w = wps[warp];
  stair_init(stair);
  if (lane < kSfxMaxG) w.key[lane] = 0xffffffffu;
  for (int i = p.g * RS + lane; i < kSfxMaxG * RS; i += 32)  // rows >= G: no group
    w.tab[i] = make_float2(__int_as_float(0x7f800000), __int_as_float(0x7f800000));
  __syncthreads();

  const GroupRec *gtab = (const GroupRec *)p.gtab;
  const int plen = p.n - M, off = p.n - M;
  const float inf = __int_as_float(0x7f800000);
  const double its = 1.0 / p.tseq, ies = 1.0 / p.eseq;
  SfxCold cold;
#pragma unroll
  for (int q = 0; q < kMaxW; q++) {
    cold.thr[q] = inf;
    best_init(cold.lb[q]);
  }
  cold.nref = 0;
  u64 ncfg = 0, nfeas = 0, stair_ver = 0;
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
    for (int q = 0; q < kMaxW; q++)
      if (q < p.nw) cold.thr[q] = fminf(cold.thr[q], __uint_as_float(__ldcg(p.thr + q)));
    if (p.want_pareto) stair_sync(stair, p, stair_ver, __ldcg(p.ctr + kCtrStairVer));
    if (lane == 0) {
      const uint32_t r = sfx_unrank_prefix(tb, p, s, w.cfg, plen);
      w.base = s - r;
    }
    __syncwarp();
    u64 ver_pref = p.want_pareto ? __shfl_sync(0xffffffffu, __ldcg(p.ctr + kCtrStairVer), 0) : 0;
    for (;;) {
      if (p.want_pareto) {
        stair_sync(stair, p, stair_ver, ver_pref);
        ver_pref = __shfl_sync(0xffffffffu, __ldcg(p.ctr + kCtrStairVer), 0);
      }
      const int kp = w.cfg.k;
      // ---- table rows whose group changed (warp-uniform loop) ----
      for (int r = 0; r < p.g; r++) {
        const uint32_t key = r < kp ? w.cfg.mask[r] : 0u;
        if (w.key[r] == key) continue;
        const int cap = key ? p.c - __popc(key) : p.c;
        for (int S = lane; S < (1 << M); S += 32) w.tab[r * RS + S] = sfx_entry(p, gtab, key, (uint32_t)S, off, cap, its, ies);
        __syncwarp();
        if (lane == 0) w.key[r] = key;
      }
      __syncwarp();
      // ---- prefix aggregates ----
      float Tp = 0.f, Ep = 0.f;
      if (lane < kp) {
        const float2 v = w.tab[lane * RS];
        Tp = v.x;
        Ep = v.y;
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        Tp = fmaxf(Tp, __shfl_xor_sync(0xffffffffu, Tp, o));
        Ep += __shfl_xor_sync(0xffffffffu, Ep, o);
      }
      const u64 base = w.base;
      const u64 Wp = tb.W[w.cfg.st[plen - 1]];
      const u64 o0 = s > base ? s - base : 0ull;
      const u64 o1 = e - base < Wp ? e - base : Wp;
      if (lane == 0) ncfg += o1 - o0;
      if (Tp < inf && o1 > o0) {
        // lane ranges: equal shares of [o0, o1)
        const uint32_t tot = (uint32_t)(o1 - o0), q = (tot + 31) >> 5;
        const uint32_t l0 = (uint32_t)o0 + min((uint32_t)lane * q, tot);
        const uint32_t l1 = (uint32_t)o0 + min((uint32_t)(lane + 1) * q, tot);
        if (l1 > l0) {
          SfxCtx x;
          x.tab = w.tab;
          x.G = p.g;
          x.C = p.c;
          x.kp = kp;
          x.off = off;
          x.base = base;
          x.pmask = w.cfg.mask;
          SfxLane s0;
          s0.gi = 0ull;
          s0.rr = 0u;
          s0.rm = 0u;
          s0.kc = kp;
          s0.T = Tp;
          s0.E = Ep;
          for (int r = 0; r < kp; r++) {
            const int room = min(p.c - (int)w.cfg.sz[r], 15);
            s0.rr |= (uint32_t)room << (4 * r);
            if (room > 0) s0.rm |= 1u << r;
          }
          sfx_unrank<M>(tb, p, x, s0, w.cfg.st[plen - 1], l0);
          SfxHot h;
          h.mT = inf;
          h.mE = inf;
          h.nf = 0;
          h.cnt = (int)(l1 - l0);
          h.ord = l0;
#ifdef SCHED_SFX_PARENTS  // A/B: round 1's parent-by-parent fast pass
          sfx_fast<M>(p, stair, x, h, s0, (int)(l1 - l0));
#else
          sfx_fast_pairs<M>(p, stair, x, h, s0, (int)(l1 - l0));
#endif
          nfeas += (u64)h.nf;
          if (h.nf) {
            bool hit = false;
#pragma unroll
            for (int q2 = 0; q2 < kMaxW; q2++) {
              if (q2 < p.nw) {
                float qq = 1.f;
                for (int i = 0; i < p.wa[q2]; i++) qq *= h.mT;
                for (int i = 0; i < p.wb[q2]; i++) qq *= h.mE;
                hit |= qq <= cold.thr[q2] * p.mul[q2];
              }
            }
            if (!hit && p.want_pareto) hit = !stair_dominated_f(stair, p, __fmul_rd(h.mT, p.tlb_scale_f), h.mE);
            if (hit) sfx_slow<M>(*p.gp, stair, x, &cold, s0, l0, (int)(l1 - l0));
          }
        }
      }
      __syncwarp();
      if (base + Wp >= e) break;
      if (lane == 0) {
        w.base = base + Wp;
        w.flag = sfx_prefix_successor(tb, p, w.cfg, plen - 1) ? 1 : 0;
      }
      __syncwarp();
      if (!w.flag) break;
    }
#pragma unroll
    for (int q = 0; q < kMaxW; q++) {
      if (q < p.nw) {
        float t = cold.thr[q];
#pragma unroll
        for (int o = 16; o; o >>= 1) t = fminf(t, __shfl_xor_sync(0xffffffffu, t, o));
        cold.thr[q] = t;
        if (lane == 0 && t < __uint_as_float(__ldcg(p.thr + q))) atomicMin(p.thr + q, __float_as_uint(t));
      }
    }
  }
  u64 nref64 = (u64)cold.nref;
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
  // per-warp best slots (slot = CTA * kSfxWarps + warp; k_best_final reduces
  // them): no block barrier after the warps' independent unit loops
#pragma unroll
  for (int q = 0; q < kMaxW; q++) {
    if (q < p.nw) {
      warp_best(cold.lb[q]);
      if (lane == 0) ((BestRec *)p.slots)[((size_t)blockIdx.x * kSfxWarps + warp) * p.nw + q] = cold.lb[q];
    }
  }
}

template <int M>
const void *sfx_fn();

}  // namespace sched
