// dp_front.cu -- exact Pareto front and optimum by a subset DP on the device
// (SURVEY 8(f) N1): spaces too large to enumerate, in particular the literal
// per-client reading of c4 (BASELINE.json "per-client active-thread
// percentage": 16 workflows x 8 GPUs x 4 levels per CLIENT = 4.05e19
// configurations, more than 2^64).
//
// A configuration is a sequence of groups in block order (group j holds the
// smallest workflow not in groups 0..j-1) with a level vector per group;
// T = max_g T_g and E = ((0 + E_0) + E_1) + ... in that order (DESIGN.md
// section 2).  Both maps are monotone under IEEE rounding, so dominated
// partial results can be dropped without losing a final Pareto point:
//   phase 1 (k_pf_items, k_pf_merge): for every feasible group B the Pareto
//     front PF(B) of its exact canonical fp64 (T_B, E_B) over all level
//     vectors (L^|B| PER_CLIENT, L PER_GPU);
//   phase 2 (k_dp_level, one launch per |S|): Front[S][k] = Pareto front of
//     { (max(T, T_b), E + E_b) : (T, E) in Front[S \ B][k-1], b in PF(B) }
//     over the last groups B of S (B holds an element below min(~S));
//   phase 3 (k_dp_final): the front of the whole set over k <= G, the best
//     point per weight (max F = X^a Y^b, first in T order on ties) and a
//     witness configuration per point traced through back-pointers.
// Everything is exact fp64 in the canonical order; the result equals the
// oracle's O4/O3 certificate (oracle/dpcert.c) bitwise.  Values and one
// witness per point; ties between distinct configurations of equal (T, E)
// are not resolved to the lowest index (the literal space has no u64 index).
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <vector>

#include "device_common.cuh"
#include "event_guard.hpp"

namespace sched {

#ifndef SCHED_PF_MINB
#define SCHED_PF_MINB 2  // k_pf_items CTAs per SM the register budget is sized for (1: 3.97 s, 2: 2.66 s)
#endif

constexpr int kLF = 16;     // lane-local front capacity (phase 1)
constexpr int kOF = 16;     // per work item / per group front capacity
constexpr int kFM = 32;     // per DP state front capacity
constexpr int kItemLog2 = 18;  // level vectors per phase-1 work item

struct PPt {  // a group tuple: exact (T_B, E_B) of level vector v
  double t, e;
  uint32_t v, pad;
};

struct DPt {  // a DP state point and its back-pointer
  double t, e;
  uint32_t B;     // last group
  uint8_t i, q;   // point in Front[S \ B][k-1] (0xff: S == B), point in PF(B)
  uint16_t pad;
};

enum { kDpItem = 0, kDpErr = 1, kDpN = 4 };

struct DpParams {
  DevParams p;                 // tables (blob), scope, L, G, C, model, ps
  int n, ns, nfull;            // workflows, subsets, n_items (phase 1)
  const uint32_t *smask;       // [ns] subsets (ascending)
  const unsigned long long *ioff;  // [ns + 1] item offsets
  const int *sid;              // [2^n] subset id of a mask, -1 if none
  PPt *items;                  // [n_items][kOF]
  int *icnt;                   // [n_items]
  PPt *pf;                     // [ns][kOF]
  int *pfcnt;                  // [ns]
  DPt *fr;                     // [2^(n-1)][G+1][kFM] (states contain workflow 0)
  int *frcnt;                  // [2^(n-1)][G+1]
  unsigned long long *ctr;     // [kDpN]
};

__device__ __forceinline__ bool dom(double t1, double e1, double t2, double e2) {  // (1) dominates (2)
  return t1 <= t2 && e1 <= e2 && (t1 < t2 || e1 < e2);
}

// insert into a small front (local memory); returns false on overflow
template <int CAP, class P>
__device__ __forceinline__ bool front_insert(P *f, int &n, const P &x) {
  for (int j = 0; j < n; j++)
    if (f[j].t <= x.t && f[j].e <= x.e) return true;  // dominated or equal: keep the first
  int w = 0;
  for (int j = 0; j < n; j++)
    if (!(x.t <= f[j].t && x.e <= f[j].e)) f[w++] = f[j];
  n = w;
  if (n >= CAP) return false;
  f[n++] = x;
  return true;
}

// exact canonical fp64 (T_B, E_B) of group B with per-member level digits
// lev[i] (digit of workflow i); false if infeasible (R27)
// the group term the DP adds up: E_g = P_s T_g + D_g (canonical), or D_g
// alone under COUNT_IDLE (R26: E = G P_s T + sum_g D_g; k_dp_final adds the
// idle term to the whole-set front, E is monotone in (T, sum D), so the
// (T, sum D) front holds every (T, E) front point)
__device__ __forceinline__ double dp_eg(const DevParams &p, double Tg, double D) {
  return (p.model & SCHED_MODEL_COUNT_IDLE) ? D : __dadd_rn(__dmul_rn(p.ps, Tg), D);
}

__device__ __forceinline__ bool group64(const Tables &tb, const DevParams &p, uint32_t B, const int *lev,
                                        double &Tout, double &Eout) {
  const double ps = p.ps;
  double U = 0.0, Bw = 0.0;
  for (uint32_t m = B; m; m &= m - 1) {
    const int i = __ffs(m) - 1, r = i * p.L + lev[i];
    U = __dadd_rn(U, (double)tb.u[r]);
    Bw = __dadd_rn(Bw, (double)tb.bw[r]);
  }
  if ((p.model & SCHED_MODEL_NO_INTERFERENCE) && (U > 1.0 || Bw > 1.0)) return false;
  double c = 1.0;
  if (U > c) c = U;
  if (Bw > c) c = Bw;
  double Tg = 0.0;
  for (uint32_t m = B; m; m &= m - 1) {
    const int i = __ffs(m) - 1, ri = i * p.L + lev[i];
    double sigma = 1.0;
    for (uint32_t m2 = B & ~(1u << i); m2; m2 &= m2 - 1) {
      const int j = __ffs(m2) - 1;
      sigma = __dadd_rn(sigma, (double)tb.d[ri * p.ds + j * p.L + lev[j]]);
    }
    const double tau = __dmul_rn(__dmul_rn((double)tb.traw[ri], sigma), c);
    if (tau > Tg) Tg = tau;
  }
  double D = 0.0;
  for (uint32_t m = B; m; m &= m - 1) {
    const int i = __ffs(m) - 1, r = i * p.L + lev[i];
    D = __dadd_rn(D, __dmul_rn(__dsub_rn((double)tb.praw[r], ps), (double)tb.traw[r]));
  }
  if (p.model & SCHED_MODEL_POWER_CAP) {
    const double tcap = __ddiv_rn(D, p.capd);
    if (tcap > Tg) Tg = tcap;
  }
  Tout = Tg;
  Eout = dp_eg(p, Tg, D);
  return true;
}

// level digits of vector v for group B: PER_CLIENT the members' digits in
// base L, most significant = lowest member; PER_GPU one digit for all
__device__ __forceinline__ void decode_vec(const DevParams &p, uint32_t B, uint32_t v, int *lev) {
  if (p.scope == SCHED_PER_GPU) {
    for (uint32_t m = B; m; m &= m - 1) lev[__ffs(m) - 1] = (int)v;
    return;
  }
  uint32_t x = v;
  for (int i = 31; i >= 0; i--)
    if (B >> i & 1u) {
      lev[i] = (int)(x % (uint32_t)p.L);
      x /= (uint32_t)p.L;
    }
}

// Split evaluation of a PER_CLIENT group's level vectors (L <= 4, |B| > kH):
// the vector's digits split into the members' high part (all but the last kH
// members, the most significant digits) and the low part (the last kH
// members, highest workflow indices).  Every canonical sum runs over members
// in ascending order, so the low members' terms come LAST: per high
// assignment the high prefixes (U, B, D, each high member's sigma over the
// other high members, each low member's sigma prefix over the high members
// for each of its levels) are summed once, and each of the L^kH low vectors
// only appends its terms -- the same additions in the same order as the
// from-scratch evaluation (group64), hence the same fp64 bits.  T uses
// max_i fl(fl(t_i s_i) c) = fl(c * max_i fl(t_i s_i)) (rounding is monotone).
constexpr int kMS = 16;  // largest group on the split path
constexpr int kH = 3;    // low members

// Table accessors of the split evaluation (values widened to fp64 exactly;
// dyn = fl(fl(p - P_s) * t) as in group64): straight from the staged fp32
// blob, or from fp64 copies staged once per CTA in shared memory (no
// per-use F2F conversion in the hot loops).
struct Acc32 {
  Tables tb;
  double ps;
  __device__ __forceinline__ double dd(int i) const { return (double)tb.d[i]; }
  __device__ __forceinline__ double t(int r) const { return (double)tb.traw[r]; }
  __device__ __forceinline__ double uu(int r) const { return (double)tb.u[r]; }
  __device__ __forceinline__ double bb(int r) const { return (double)tb.bw[r]; }
  __device__ __forceinline__ double dyn(int r) const {
    return __dmul_rn(__dsub_rn((double)tb.praw[r], ps), (double)tb.traw[r]);
  }
};
struct Acc64 {
  const double *d, *tt, *u, *bw, *dy;
  __device__ __forceinline__ double dd(int i) const { return d[i]; }
  __device__ __forceinline__ double t(int r) const { return tt[r]; }
  __device__ __forceinline__ double uu(int r) const { return u[r]; }
  __device__ __forceinline__ double bb(int r) const { return bw[r]; }
  __device__ __forceinline__ double dyn(int r) const { return dy[r]; }
};
// fp64 shared-memory tables: d [R * ds] then t, u, bw, dyn [R] (R = n L rows)
__host__ __device__ inline size_t acc64_bytes(const DevParams &p) {
  const size_t R = (size_t)p.n * p.L;
  return 8 * (R * p.ds + 4 * R);
}
constexpr size_t kAcc64Max = 40 << 10;  // staged only if it fits beside 4 CTAs per SM

// per-warp scratch of the block-corner bounds (one group per warp item):
// MD[(k*4 + level of high member k)*3 + j] = min over the levels of low member
// j of d[high k][low j]; ML[(j*4 + l)*3 + j2] = min over the levels of j2 of
// d[low j at l][low j2]; then the minima of u, bw, dyn of each low member
constexpr int kScrMD = (kMS - kH) * 4 * kH, kScrML = kH * 4 * kH, kScr = kScrMD + kScrML + 3 * kH;

template <class A>
__device__ __forceinline__ void pf_split(const A &tb, const DevParams &p, uint32_t B, int s, uint64_t v0,
                                         uint64_t v1, int lane, PPt *f, int &nf, bool &ok, double *scr) {
  const int L = p.L, nh = s - kH;
  const uint32_t Lh = (uint32_t)(L * L * L);
  int mw[kMS];
  {
    int k = 0;
#pragma unroll
    for (int b = 0; b < 32; b++)
      if (B >> b & 1u) {
        if (k < kMS) mw[k] = b;
        k++;
      }
  }
  const double ps = p.ps;
  {  // the group's corner-bound tables, once per item, lanes cooperating
    for (int e = lane; e < kScr; e += 32) {
      double v = 0.0;
      if (e < kScrMD) {
        const int k = e / (4 * kH), lk = (e / kH) % 4, j = e % kH;
        if (k < nh && lk < L) {
          const int rk = mw[k] * L + lk, rj = mw[nh + j] * L;
          v = tb.dd(rk * p.ds + rj);
          for (int l = 1; l < L; l++) v = fmin(v, tb.dd(rk * p.ds + rj + l));
        }
      } else if (e < kScrMD + kScrML) {
        const int x = e - kScrMD, j = x / (4 * kH), l = (x / kH) % 4, j2 = x % kH;
        if (l < L && j2 != j) {
          const int rj = mw[nh + j] * L + l, r2 = mw[nh + j2] * L;
          v = tb.dd(rj * p.ds + r2);
          for (int l2 = 1; l2 < L; l2++) v = fmin(v, tb.dd(rj * p.ds + r2 + l2));
        }
      } else {
        const int x = e - kScrMD - kScrML, what = x / kH, j = x % kH, rj = mw[nh + j] * L;
        v = what == 0 ? tb.uu(rj) : what == 1 ? tb.bb(rj) : tb.dyn(rj);
        for (int l = 1; l < L; l++)
          v = fmin(v, what == 0 ? tb.uu(rj + l) : what == 1 ? tb.bb(rj + l) : tb.dyn(rj + l));
      }
      scr[e] = v;
    }
    __syncwarp();
  }
  const double kInf = __longlong_as_double(0x7ff0000000000000ll);
  double lt = kInf, le = kInf;  // the lane's last inserted point
  double bt = kInf, be = kInf;  // the lane's lowest-(T, E) evaluated point
  // every lane runs the same number of blocks: the warp can share its best point
  const bool uni = v0 % Lh == 0 && (v1 - v0) % (32ull * Lh) == 0;
  for (uint64_t hv = v0 / Lh + lane; hv * Lh < v1; hv += 32) {
    double wt = kInf, we = kInf;  // the warp's lowest-(T, E) evaluated point (a real point of B)
    if (uni) {
      wt = bt;
      we = be;
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        const double t2 = __shfl_xor_sync(0xffffffffu, wt, o), e2 = __shfl_xor_sync(0xffffffffu, we, o);
        if (t2 < wt || (t2 == wt && e2 < we)) {
          wt = t2;
          we = e2;
        }
      }
    }
    int rh[kMS - kH];
    double sg[kMS - kH];
    double U = 0.0, Bw = 0.0, D = 0.0;
    {
      uint64_t x = hv;
#pragma unroll
      for (int k = kMS - kH - 1; k >= 0; k--)
        if (k < nh) {
          rh[k] = mw[k] * L + (int)((uint32_t)x % (uint32_t)L);  // hv < 4^13: 32-bit
          x = (uint32_t)x / (uint32_t)L;
        }
    }
#pragma unroll
    for (int k = 0; k < kMS - kH; k++)
      if (k < nh) {
        const int r = rh[k];
        U = __dadd_rn(U, tb.uu(r));
        Bw = __dadd_rn(Bw, tb.bb(r));
        D = __dadd_rn(D, tb.dyn(r));
      }
    // sigma prefixes over the high members (ascending q, one rolled loop
    // with the member's row recomputed from hv: small code), and for each
    // low member and level the sum over the high members
    double Q[kH][4];
#pragma unroll
    for (int k = 0; k < kMS - kH; k++) sg[k] = 1.0;
#pragma unroll
    for (int j = 0; j < kH; j++)
#pragma unroll
      for (int l = 0; l < 4; l++) Q[j][l] = 1.0;
    {
      uint32_t pw = 1;
      for (int q = 1; q < nh; q++) pw *= (uint32_t)L;  // L^(nh-1): weight of member 0's digit
#pragma unroll 1
      for (int q = 0; q < nh; q++, pw /= (uint32_t)L) {
        const int rq = mw[q] * L + (int)(((uint32_t)hv / pw) % (uint32_t)L);
#pragma unroll
        for (int k = 0; k < kMS - kH; k++)
          if (k < nh && k != q) sg[k] = __dadd_rn(sg[k], tb.dd(rh[k] * p.ds + rq));
#pragma unroll
        for (int j = 0; j < kH; j++)
#pragma unroll
          for (int l = 0; l < 4; l++)
            if (l < L) Q[j][l] = __dadd_rn(Q[j][l], tb.dd((mw[nh + j] * L + l) * p.ds + rq));
      }
    }
    const uint64_t base = hv * Lh;
    const uint32_t lv0 = (uint32_t)(v0 > base ? v0 - base : 0), lv1 = (uint32_t)(v1 - base < Lh ? v1 - base : Lh);
    if (lv0 == 0 && lv1 == Lh) {
      // Whole low block, nested over the low members' digits (d0 most
      // significant, as the index): every partial sum that does not involve
      // a deeper low member is formed once at its loop level -- the same
      // additions in the same ascending-member order as below.
      const int r0b = mw[nh] * L, r1b = mw[nh + 1] * L, r2b = mw[nh + 2] * L;
      if (nf > 0 || wt != kInf) {
        // Block lower corner: every canonical sum with each low member's term
        // replaced by its minimum over the levels (same order; rounding is
        // monotone, all terms >= 0), so T >= Tmin and E >= Emin for every
        // vector of the block.  A point of B at or below the corner (the
        // lane's front, or the warp's best evaluated point) dominates or
        // equals all 64 vectors: skip the block.
        const int rb[kH] = {r0b, r1b, r2b};
        const double *MD = scr, *ML = scr + kScrMD, *MX = scr + kScrMD + kScrML;
        double Umin = U, Bmin = Bw, Dmin = D;
#pragma unroll
        for (int j = 0; j < kH; j++) {
          Umin = __dadd_rn(Umin, MX[j]);
          Bmin = __dadd_rn(Bmin, MX[kH + j]);
          Dmin = __dadd_rn(Dmin, MX[2 * kH + j]);
        }
        if ((p.model & SCHED_MODEL_NO_INTERFERENCE) && (Umin > 1.0 || Bmin > 1.0)) continue;  // all infeasible
        double cmin = 1.0;
        if (Umin > cmin) cmin = Umin;
        if (Bmin > cmin) cmin = Bmin;
        double mx = 0.0;
#pragma unroll
        for (int k = 0; k < kMS - kH; k++)
          if (k < nh) {
            const double *md = MD + (k * 4 + (rh[k] - mw[k] * L)) * kH;
            const double a = __dadd_rn(__dadd_rn(__dadd_rn(sg[k], md[0]), md[1]), md[2]);
            const double ts = __dmul_rn(tb.t(rh[k]), a);
            if (ts > mx) mx = ts;
          }
#pragma unroll
        for (int j = 0; j < kH; j++) {
          double tj = 0.0;  // min over the member's own level of its bound
          for (int l = 0; l < L; l++) {
            double a = Q[j][l];
#pragma unroll
            for (int j2 = 0; j2 < kH; j2++)
              if (j2 != j) a = __dadd_rn(a, ML[(j * 4 + l) * kH + j2]);
            const double ts = __dmul_rn(tb.t(rb[j] + l), a);
            tj = l == 0 ? ts : fmin(tj, ts);
          }
          if (tj > mx) mx = tj;
        }
        double Tmin = __dmul_rn(mx, cmin);
        if (p.model & SCHED_MODEL_POWER_CAP) {
          const double tcap = __ddiv_rn(Dmin, p.capd);
          if (tcap > Tmin) Tmin = tcap;
        }
        const double Emin = dp_eg(p, Tmin, Dmin);
        bool skip = wt <= Tmin && we <= Emin;
        for (int i = 0; i < nf && !skip; i++)
          if (f[i].t <= Tmin && f[i].e <= Emin) {
            skip = true;
            break;
          }
        if (skip) continue;
      }
      for (int d0 = 0; d0 < L; d0++) {
        const int r0 = r0b + d0;
        const double U0 = __dadd_rn(U, tb.uu(r0)), B0 = __dadd_rn(Bw, tb.bb(r0));
        const double D0 = __dadd_rn(D, tb.dyn(r0));
        for (int d1 = 0; d1 < L; d1++) {
          const int r1 = r1b + d1;
          const double U1 = __dadd_rn(U0, tb.uu(r1)), B1 = __dadd_rn(B0, tb.bb(r1));
          const double D1 = __dadd_rn(D0, tb.dyn(r1));
          double a1[kMS - kH];
#pragma unroll
          for (int k = 0; k < kMS - kH; k++)
            if (k < nh)  // (sg + d[k][low 0]) + d[k][low 1]: the a0 partial re-formed per d1 (fewer live registers)
              a1[k] = __dadd_rn(__dadd_rn(sg[k], tb.dd(rh[k] * p.ds + r0)), tb.dd(rh[k] * p.ds + r1));
          const double s0p = __dadd_rn(Q[0][d0], tb.dd(r0 * p.ds + r1));  // low 0: + low 1
          const double s1p = __dadd_rn(Q[1][d1], tb.dd(r1 * p.ds + r0));  // low 1: + low 0
          for (int d2 = 0; d2 < L; d2++) {
            const int r2 = r2b + d2;
            const double Ul = __dadd_rn(U1, tb.uu(r2)), Bl = __dadd_rn(B1, tb.bb(r2));
            const double Dl =
                __dadd_rn(D1, tb.dyn(r2));
            if ((p.model & SCHED_MODEL_NO_INTERFERENCE) && (Ul > 1.0 || Bl > 1.0)) continue;
            double c = 1.0;
            if (Ul > c) c = Ul;
            if (Bl > c) c = Bl;
            double mx = 0.0;
#pragma unroll
            for (int k = 0; k < kMS - kH; k++)
              if (k < nh) {
                const double ts =
                    __dmul_rn(tb.t(rh[k]), __dadd_rn(a1[k], tb.dd(rh[k] * p.ds + r2)));
                if (ts > mx) mx = ts;
              }
            const double t0 = __dmul_rn(tb.t(r0), __dadd_rn(s0p, tb.dd(r0 * p.ds + r2)));
            const double t1 = __dmul_rn(tb.t(r1), __dadd_rn(s1p, tb.dd(r1 * p.ds + r2)));
            const double t2 = __dmul_rn(tb.t(r2), __dadd_rn(__dadd_rn(Q[2][d2], tb.dd(r2 * p.ds + r0)),
                                                                    tb.dd(r2 * p.ds + r1)));
            if (t0 > mx) mx = t0;
            if (t1 > mx) mx = t1;
            if (t2 > mx) mx = t2;
            double Tg = __dmul_rn(mx, c);
            if (p.model & SCHED_MODEL_POWER_CAP) {
              const double tcap = __ddiv_rn(Dl, p.capd);
              if (tcap > Tg) Tg = tcap;
            }
            PPt x;
            x.t = Tg;
            x.e = dp_eg(p, Tg, Dl);
            x.v = (uint32_t)(base + (uint32_t)((d0 * L + d1) * L + d2));
            x.pad = 0;
            // quick reject: a point inserted earlier (lt, le) dominates or equals x ->
            // so does the front (transitivity), front_insert would keep it unchanged
            if (x.t < bt || (x.t == bt && x.e < be)) {
              bt = x.t;
              be = x.e;
            }
            if (x.t >= lt && x.e >= le) continue;
            ok &= front_insert<kLF>(f, nf, x);
            lt = x.t;
            le = x.e;
          }
        }
      }
      continue;
    }
    for (uint32_t lv = lv0; lv < lv1; lv++) {
      int dl[kH], rl[kH];
      {
        uint32_t x = lv;
#pragma unroll
        for (int j = kH - 1; j >= 0; j--) {
          dl[j] = (int)(x % (uint32_t)L);
          x /= (uint32_t)L;
          rl[j] = mw[nh + j] * L + dl[j];
        }
      }
      double Ul = U, Bl = Bw, Dl = D;
#pragma unroll
      for (int j = 0; j < kH; j++) {
        Ul = __dadd_rn(Ul, tb.uu(rl[j]));
        Bl = __dadd_rn(Bl, tb.bb(rl[j]));
        Dl = __dadd_rn(Dl, tb.dyn(rl[j]));
      }
      if ((p.model & SCHED_MODEL_NO_INTERFERENCE) && (Ul > 1.0 || Bl > 1.0)) continue;
      double c = 1.0;
      if (Ul > c) c = Ul;
      if (Bl > c) c = Bl;
      double mx = 0.0;
#pragma unroll
      for (int k = 0; k < kMS - kH; k++)
        if (k < nh) {
          double a = sg[k];
          const int rd = rh[k] * p.ds;
#pragma unroll
          for (int j = 0; j < kH; j++) a = __dadd_rn(a, tb.dd(rd + rl[j]));
          const double ts = __dmul_rn(tb.t(rh[k]), a);
          if (ts > mx) mx = ts;
        }
#pragma unroll
      for (int j = 0; j < kH; j++) {
        double a = Q[j][dl[j]];
#pragma unroll
        for (int j2 = 0; j2 < kH; j2++)
          if (j2 != j) a = __dadd_rn(a, tb.dd(rl[j] * p.ds + rl[j2]));
        const double ts = __dmul_rn(tb.t(rl[j]), a);
        if (ts > mx) mx = ts;
      }
      double Tg = __dmul_rn(mx, c);
      if (p.model & SCHED_MODEL_POWER_CAP) {
        const double tcap = __ddiv_rn(Dl, p.capd);
        if (tcap > Tg) Tg = tcap;
      }
      PPt x;
      x.t = Tg;
      x.e = dp_eg(p, Tg, Dl);
      x.v = (uint32_t)(base + lv);
      x.pad = 0;
      ok &= front_insert<kLF>(f, nf, x);
    }
  }
}

// the fp32-table path out of line: only for tables too large for the fp64
// shared-memory copies; keeps the hot kernel's code (instruction cache) small
__device__ __noinline__ void pf_split_a32(const Acc32 &tb, const DevParams &p, uint32_t B, int s, uint64_t v0,
                                          uint64_t v1, int lane, PPt *f, int &nf, bool &ok, double *scr) {
  pf_split(tb, p, B, s, v0, v1, lane, f, nf, ok, scr);
}

// small groups and PER_GPU: one from-scratch fp64 evaluation per level
// vector (out of line: small code in the hot kernel)
__device__ __noinline__ void pf_plain(const Tables &tb, const DevParams &p, uint32_t B, uint64_t v0, uint64_t v1,
                                      int lane, PPt *f, int &nf, bool &ok) {
  int lev[kMaxN];
  for (uint64_t v = v0 + lane; v < v1; v += 32) {
    decode_vec(p, B, (uint32_t)v, lev);
    PPt x;
    if (!group64(tb, p, B, lev, x.t, x.e)) continue;
    x.v = (uint32_t)v;
    x.pad = 0;
    ok &= front_insert<kLF>(f, nf, x);
  }
}

// phase 1a: work item = (group, 2^kItemLog2 level vectors); one warp per item
__global__ void __launch_bounds__(256, SCHED_PF_MINB) k_pf_items(const DpParams dp) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, dp.p);
  const Tables tb = tables_at(sm, dp.p);
  const int lane = threadIdx.x & 31;
  const bool use64 = dp.p.scope == SCHED_PER_CLIENT && acc64_bytes(dp.p) <= kAcc64Max;
  Acc64 a64{};
  if (use64) {
    const int R = dp.p.n * dp.p.L;
    double *b = (double *)(sm + ((dp.p.blob_bytes + 15) & ~15u));
    double *rows = b + (size_t)R * dp.p.ds;
    for (int i = threadIdx.x; i < R * dp.p.ds; i += blockDim.x) b[i] = (double)tb.d[i];
    for (int r = threadIdx.x; r < R; r += blockDim.x) {
      rows[r] = (double)tb.traw[r];
      rows[R + r] = (double)tb.u[r];
      rows[2 * R + r] = (double)tb.bw[r];
      rows[3 * R + r] = __dmul_rn(__dsub_rn((double)tb.praw[r], dp.p.ps), (double)tb.traw[r]);
    }
    a64 = Acc64{b, rows, rows + R, rows + 2 * R, rows + 3 * R};
    __syncthreads();
  }
  const Acc32 a32{tb, dp.p.ps};
  double *scr = (double *)(sm + ((dp.p.blob_bytes + 15) & ~15u) + (use64 ? acc64_bytes(dp.p) : 0)) +
                (size_t)(threadIdx.x >> 5) * kScr;  // this warp's corner-bound tables
  for (;;) {
    unsigned long long it = 0;
    if (lane == 0) it = atomicAdd(dp.ctr + kDpItem, 1ull);
    it = __shfl_sync(0xffffffffu, it, 0);
    if (it >= (unsigned long long)dp.nfull) break;
    int lo = 0, hi = dp.ns - 1;  // subset of the item: ioff[s] <= it < ioff[s+1]
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (dp.ioff[mid] <= it) lo = mid;
      else hi = mid - 1;
    }
    const uint32_t B = dp.smask[lo];
    const int s = __popc(B);
    uint64_t nv = dp.p.scope == SCHED_PER_GPU ? (uint64_t)dp.p.L : 1ull;
    if (dp.p.scope != SCHED_PER_GPU)
      for (int k = 0; k < s; k++) nv *= (uint64_t)dp.p.L;
    const uint64_t v0 = (it - dp.ioff[lo]) << kItemLog2;
    const uint64_t v1 = v0 + (1ull << kItemLog2) < nv ? v0 + (1ull << kItemLog2) : nv;
    PPt f[kLF];
    int nf = 0;
    bool ok = true;
    if (dp.p.scope == SCHED_PER_CLIENT && s > kH && s <= kMS && dp.p.L <= 4) {
      if (use64) pf_split(a64, dp.p, B, s, v0, v1, lane, f, nf, ok, scr);
      else pf_split_a32(a32, dp.p, B, s, v0, v1, lane, f, nf, ok, scr);
    } else {
      pf_plain(tb, dp.p, B, v0, v1, lane, f, nf, ok);
    }
    if (!ok) atomicExch(dp.ctr + kDpErr, 1ull);
    // warp merge: every lane keeps its points not dominated by another lane's
    // (ties: the lower (lane, slot) wins), survivors compacted by ballot
    PPt *out = dp.items + it * kOF;
    int nout = 0;
    for (int r = 0; r < kLF; r++) {  // round r: slot r of every lane
      const bool has = r < nf;
      if (!__any_sync(0xffffffffu, has)) break;
      PPt x = has ? f[r] : PPt{0, 0, 0, 0};
      bool keep = has;
      for (int o = 0; o < 32; o++) {  // compare with every point of lane o
        const int no = __shfl_sync(0xffffffffu, nf, o);
        for (int q = 0; q < no; q++) {
          PPt y;
          y.t = __shfl_sync(0xffffffffu, f[min(q, kLF - 1)].t, o);
          y.e = __shfl_sync(0xffffffffu, f[min(q, kLF - 1)].e, o);
          if (keep && (dom(y.t, y.e, x.t, x.e) ||
                       (y.t == x.t && y.e == x.e && (o < lane || (o == lane && q < r)))))
            keep = false;
        }
      }
      const unsigned bal = __ballot_sync(0xffffffffu, keep);
      const int pos = nout + __popc(bal & ((1u << lane) - 1));
      if (keep) {
        if (pos < kOF) out[pos] = x;
        else atomicExch(dp.ctr + kDpErr, 1ull);
      }
      nout += __popc(bal);
    }
    if (lane == 0) dp.icnt[it] = min(nout, kOF);
  }
}

// phase 1b: PF(B) = front of the group's item fronts; one warp per group
__global__ void __launch_bounds__(256) k_pf_merge(const DpParams dp) {
  __shared__ PPt fs[8][kOF + 1];
  __shared__ int fn[8];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  PPt *f = fs[warp];
  for (int sb = blockIdx.x * 8 + warp; sb < dp.ns; sb += gridDim.x * 8) {
    if (lane == 0) fn[warp] = 0;
    __syncwarp();
    const unsigned long long i0 = dp.ioff[sb], i1 = dp.ioff[sb + 1];
    for (unsigned long long it = i0; it < i1; it++) {
      const int c = dp.icnt[it];
      for (int q0 = 0; q0 < c; q0 += 32) {  // a batch of up to 32 candidates, one per lane
        const int q = q0 + lane;
        PPt x = q < c ? dp.items[it * kOF + q] : PPt{0, 0, 0, 0};
        bool keep = q < c;
        const int n0 = fn[warp];
        for (int j = 0; j < n0 && keep; j++)
          if (f[j].t <= x.t && f[j].e <= x.e) keep = false;
        unsigned bal = __ballot_sync(0xffffffffu, keep);
        while (bal) {  // insert survivors in lane order
          const int l = __ffs(bal) - 1;
          bal &= bal - 1;
          PPt y;
          y.t = __shfl_sync(0xffffffffu, x.t, l);
          y.e = __shfl_sync(0xffffffffu, x.e, l);
          y.v = __shfl_sync(0xffffffffu, x.v, l);
          y.pad = 0;
          if (lane == 0) {
            int n = fn[warp];
            bool in = true;
            for (int j = 0; j < n; j++)
              if (f[j].t <= y.t && f[j].e <= y.e) in = false;
            if (in) {
              int w = 0;
              for (int j = 0; j < n; j++)
                if (!(y.t <= f[j].t && y.e <= f[j].e)) f[w++] = f[j];
              if (w < kOF) f[w++] = y;
              else atomicExch(dp.ctr + kDpErr, 1ull);
              fn[warp] = w;
            }
          }
          __syncwarp();
        }
      }
    }
    __syncwarp();
    const int n = fn[warp];
    for (int j = lane; j < n; j += 32) dp.pf[(size_t)sb * kOF + j] = f[j];
    if (lane == 0) dp.pfcnt[sb] = n;
    __syncwarp();
  }
}

// phase 2: states S (containing workflow 0) with |S| = m; warp per (S, k)
__global__ void __launch_bounds__(256) k_dp_level(const DpParams dp, int m, int nstates,
                                                  const uint32_t *states) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int G = dp.p.g, C = dp.p.c;
  const int wid = blockIdx.x * 8 + warp;
  if (wid >= nstates * G) return;
  const uint32_t S = states[wid / G];
  const int k = wid % G + 1;  // groups in S
  const uint32_t full = dp.n >= 32 ? 0xffffffffu : (1u << dp.n) - 1;
  const uint32_t outside = full & ~S;
  const int fmin = outside ? __ffs(outside) - 1 : dp.n;  // smallest workflow not in S
  const uint32_t below = fmin >= 32 ? 0xffffffffu : (1u << fmin) - 1;  // B must meet these
  DPt f[kFM];
  int nf = 0;
  bool ok = true;
  // one candidate last group B of S: B meets `below`, |B| <= C, PF(B) non-empty
  auto visit = [&](uint32_t B) {
    if (!(B & below) || __popc(B) > C) return;
    const int sb = dp.sid[B];
    if (sb < 0) return;
    const int npf = dp.pfcnt[sb];
    if (!npf) return;
    const uint32_t R = S & ~B;
    if (R == 0) {
      if (k != 1) return;
      for (int q = 0; q < npf; q++) {
        const PPt b = dp.pf[(size_t)sb * kOF + q];
        DPt y{b.t, b.e, B, 0xff, (uint8_t)q, 0};
        ok &= front_insert<kFM>(f, nf, y);
      }
      return;
    }
    if (k == 1 || !(R & 1u)) return;
    const size_t src = ((size_t)(R >> 1) * (G + 1) + (k - 1));
    const int nr = dp.frcnt[src];
    for (int i = 0; i < nr; i++) {
      const DPt a = dp.fr[src * kFM + i];
      for (int q = 0; q < npf; q++) {
        const PPt b = dp.pf[(size_t)sb * kOF + q];
        DPt y{a.t > b.t ? a.t : b.t, __dadd_rn(a.e, b.e), B, (uint8_t)i, (uint8_t)q, 0};
        ok &= front_insert<kFM>(f, nf, y);
      }
    }
  };
  if (C <= 4 && C < m) {
    // capped groups: enumerate the <= C-subsets of S directly (O(m^C) instead
    // of all 2^m subsets), lanes split by the subset's lowest member
    int mem[32];
    int nm = 0;
    for (uint32_t mm = S; mm; mm &= mm - 1) mem[nm++] = __ffs(mm) - 1;
    for (int i1 = lane; i1 < nm; i1 += 32) {
      const uint32_t b1 = 1u << mem[i1];
      visit(b1);
      if (C < 2) continue;
      for (int i2 = i1 + 1; i2 < nm; i2++) {
        const uint32_t b2 = b1 | (1u << mem[i2]);
        visit(b2);
        if (C < 3) continue;
        for (int i3 = i2 + 1; i3 < nm; i3++) {
          const uint32_t b3 = b2 | (1u << mem[i3]);
          visit(b3);
          if (C < 4) continue;
          for (int i4 = i3 + 1; i4 < nm; i4++) visit(b3 | (1u << mem[i4]));
        }
      }
    }
  } else {
    const uint32_t nsub = 1u << m;
    for (uint32_t x = 1 + lane; x < nsub; x += 32) {
      uint32_t B = 0, xx = x;  // x-th subset of S (bit deposit)
      for (uint32_t mm = S; mm && xx; mm &= mm - 1, xx >>= 1)
        if (xx & 1u) B |= mm & (0u - mm);
      if (!(B & below) || __popc(B) > C) continue;
      const int sb = dp.sid[B];
      if (sb < 0) continue;
      const int npf = dp.pfcnt[sb];
      if (!npf) continue;
      const uint32_t R = S & ~B;
      if (R == 0) {
        if (k != 1) continue;
        for (int q = 0; q < npf; q++) {
          const PPt b = dp.pf[(size_t)sb * kOF + q];
          DPt y{b.t, b.e, B, 0xff, (uint8_t)q, 0};
          ok &= front_insert<kFM>(f, nf, y);
        }
        continue;
      }
      if (k == 1 || !(R & 1u)) continue;
      const size_t src = ((size_t)(R >> 1) * (G + 1) + (k - 1));
      const int nr = dp.frcnt[src];
      for (int i = 0; i < nr; i++) {
        const DPt a = dp.fr[src * kFM + i];
        for (int q = 0; q < npf; q++) {
          const PPt b = dp.pf[(size_t)sb * kOF + q];
          DPt y{a.t > b.t ? a.t : b.t, __dadd_rn(a.e, b.e), B, (uint8_t)i, (uint8_t)q, 0};
          ok &= front_insert<kFM>(f, nf, y);
        }
      }
    }
  }
  if (!ok) atomicExch(dp.ctr + kDpErr, 1ull);
  // warp merge (ties: lower (lane, slot) wins), write the state's front
  const size_t dst = (size_t)(S >> 1) * (G + 1) + k;
  int nout = 0;
  for (int r = 0; r < kFM; r++) {
    const bool has = r < nf;
    if (!__any_sync(0xffffffffu, has)) break;
    DPt x = has ? f[r] : DPt{0, 0, 0, 0, 0, 0};
    bool keep = has;
    for (int o = 0; o < 32; o++) {
      const int no = __shfl_sync(0xffffffffu, nf, o);
      for (int q = 0; q < no; q++) {
        const double yt = __shfl_sync(0xffffffffu, f[min(q, kFM - 1)].t, o);
        const double ye = __shfl_sync(0xffffffffu, f[min(q, kFM - 1)].e, o);
        if (keep && (dom(yt, ye, x.t, x.e) || (yt == x.t && ye == x.e && (o < lane || (o == lane && q < r)))))
          keep = false;
      }
    }
    const unsigned bal = __ballot_sync(0xffffffffu, keep);
    const int pos = nout + __popc(bal & ((1u << lane) - 1));
    if (keep) {
      if (pos < kFM) dp.fr[dst * kFM + pos] = x;
      else atomicExch(dp.ctr + kDpErr, 1ull);
    }
    nout += __popc(bal);
  }
  if (lane == 0) dp.frcnt[dst] = min(nout, kFM);
}

// phase 3: front of the whole set over k = 1..G (ordered by T, then E) with
// witness configurations (group masks in block order + level vectors)
struct DpOut {
  double t, e;
  uint32_t groups[kMaxG];
  uint32_t vecs[kMaxG];
  int k;
  int pad;
};

__global__ void k_dp_final(const DpParams dp, DpOut *out, int cap, int *nout, int *best) {
  // single thread: at most G * kFM candidates
  if (threadIdx.x || blockIdx.x) return;
  const int G = dp.p.g;
  const uint32_t full = dp.n >= 32 ? 0xffffffffu : (1u << dp.n) - 1;
  if (dp.p.model & SCHED_MODEL_COUNT_IDLE) {  // R26: E = (G P_s) T + sum_g D_g (group order), as the oracle
    for (int k = 1; k <= G; k++) {
      const size_t st = (size_t)(full >> 1) * (G + 1) + k;
      for (int i = 0; i < dp.frcnt[st]; i++) {
        DPt &x = dp.fr[st * kFM + i];
        x.e = __dadd_rn(__dmul_rn(dp.p.gps, x.t), x.e);
      }
    }
  }
  int n = 0;
  for (int k = 1; k <= G; k++) {
    const size_t st = (size_t)(full >> 1) * (G + 1) + k;
    for (int i = 0; i < dp.frcnt[st]; i++) {
      const DPt x = dp.fr[st * kFM + i];
      bool keep = true;
      for (int k2 = 1; k2 <= G && keep; k2++) {
        const size_t s2 = (size_t)(full >> 1) * (G + 1) + k2;
        for (int j = 0; j < dp.frcnt[s2]; j++) {
          const DPt y = dp.fr[s2 * kFM + j];
          if (dom(y.t, y.e, x.t, x.e) || (y.t == x.t && y.e == x.e && (k2 < k || (k2 == k && j < i)))) {
            keep = false;
            break;
          }
        }
      }
      if (!keep) continue;
      if (n < cap) {
        DpOut &o = out[n];
        o.t = x.t;
        o.e = x.e;
        // trace back through the states
        uint32_t S = full;
        int kk = k, pi = i, g = k - 1;
        while (g >= 0) {
          const DPt y = dp.fr[((size_t)(S >> 1) * (G + 1) + kk) * kFM + pi];
          o.groups[g] = y.B;
          o.vecs[g] = dp.pf[(size_t)dp.sid[y.B] * kOF + y.q].v;
          S &= ~y.B;
          kk--;
          g--;
          if (y.i == 0xff) break;
          pi = y.i;
        }
        o.k = k;
      }
      n++;
    }
  }
  // order by T ascending (then E): insertion sort on the output
  const int m = n < cap ? n : cap;
  for (int a = 1; a < m; a++) {
    DpOut x = out[a];
    int b = a - 1;
    while (b >= 0 && (out[b].t > x.t || (out[b].t == x.t && out[b].e > x.e))) {
      out[b + 1] = out[b];
      b--;
    }
    out[b + 1] = x;
  }
  *nout = n;
  // best point per weight: max F = X^a Y^b (fp64 canonical), first in T order on ties
  for (int w = 0; w < dp.p.nw; w++) {
    int bi = -1;
    double bf = 0.0;
    for (int a = 0; a < m; a++) {
      const double F = objective64(dp.p, out[a].t, out[a].e, dp.p.wa[w], dp.p.wb[w]);
      if (bi < 0 || F > bf) {
        bi = a;
        bf = F;
      }
    }
    best[w] = bi;
  }
}

// ------------------------------------------------------------------ host side
namespace {
struct DpLayout {
  size_t ctr, blob, smask, ioff, sid, items, icnt, pf, pfcnt, fr, frcnt, states, out, nout, total;
};

DpLayout dp_layout(const DevParams &p, int n, int ns, uint64_t nitems, size_t nstates) {
  DpLayout L;
  size_t o = 0;
  auto take = [&](size_t b) {
    o = (o + 255) / 256 * 256;
    const size_t r = o;
    o += b;
    return r;
  };
  L.ctr = take(8 * kDpN);
  L.blob = take(p.blob_bytes);
  L.smask = take(4 * (size_t)ns);
  L.ioff = take(8 * ((size_t)ns + 1));
  L.sid = take(4 * ((size_t)1 << n));
  L.items = take(sizeof(PPt) * kOF * (size_t)nitems);
  L.icnt = take(4 * (size_t)nitems);
  L.pf = take(sizeof(PPt) * kOF * (size_t)ns);
  L.pfcnt = take(4 * (size_t)ns);
  L.fr = take(sizeof(DPt) * kFM * ((size_t)1 << (n - 1)) * (p.g + 1));
  L.frcnt = take(4 * ((size_t)1 << (n - 1)) * (p.g + 1));
  L.states = take(4 * nstates);
  L.out = take(sizeof(DpOut) * (size_t)kFM * p.g);
  L.nout = take(8 + 4 * kMaxW);
  L.total = (o + 255) / 256 * 256;
  return L;
}

// the feasible groups (|B| <= C, memory) and the phase-1 work items
void dp_groups(const Profile &P, const Query &q, std::vector<uint32_t> *smask, std::vector<unsigned long long> *ioff,
               std::vector<int> *sid) {
  const int n = q.n;
  sid->assign((size_t)1 << n, -1);
  smask->clear();
  ioff->assign(1, 0ull);
  for (uint32_t B = 1; B < (1u << n); B++) {
    const int s = __builtin_popcount(B);
    if (s > q.c) continue;
    long long M = 0;
    for (int i = 0; i < n; i++)
      if (B >> i & 1u) M += P.mem[i];
    if (M > (long long)P.mem_cap) continue;
    unsigned long long nv = 1;
    if (q.scope == SCHED_PER_GPU) nv = (unsigned long long)q.L;
    else
      for (int k = 0; k < s; k++) nv *= (unsigned long long)q.L;
    (*sid)[B] = (int)smask->size();
    smask->push_back(B);
    ioff->push_back(ioff->back() + ((nv + (1ull << kItemLog2) - 1) >> kItemLog2));
  }
}
}  // namespace

int dp_front_workspace(const Profile &P, const Query &q, const DevParams &dp, size_t *bytes) {
  if (q.n < 2 || q.n > 20 || q.g > kMaxG || (q.model & SCHED_MODEL_TIME_SLICE))
    return SCHED_E_INVALID;
  if (q.scope == SCHED_PER_CLIENT) {
    double lg = 0.0;  // L^C must fit the 32-bit vector id
    for (int k = 0; k < q.c; k++) lg += std::log2((double)q.L);
    if (lg > 32.0) return SCHED_E_TOO_LARGE;
  }
  std::vector<uint32_t> smask;
  std::vector<unsigned long long> ioff;
  std::vector<int> sid;
  dp_groups(P, q, &smask, &ioff, &sid);
  const size_t nst = (size_t)1 << (q.n - 1);
  *bytes = dp_layout(dp, q.n, (int)smask.size(), ioff.back(), nst).total;
  return SCHED_OK;
}

#define CKD(x)                                  \
  do {                                          \
    cudaError_t e_ = (x);                       \
    if (e_ != cudaSuccess) return SCHED_E_CUDA; \
  } while (0)

int dp_front_run(const Profile &P, const Query &q, DevParams p, const std::vector<unsigned char> &blob, void *d_ws,
                 size_t ws_bytes, void *stream, std::vector<DpPoint> *front, int *best_pos, float *ms,
                 int *launches) {
  size_t need = 0;
  int st = dp_front_workspace(P, q, p, &need);
  if (st) return st;
  if (ws_bytes < need || ((uintptr_t)d_ws & 255)) return SCHED_E_WORKSPACE;
  std::vector<uint32_t> smask;
  std::vector<unsigned long long> ioff;
  std::vector<int> sid;
  dp_groups(P, q, &smask, &ioff, &sid);
  const int n = q.n, ns = (int)smask.size(), G = q.g;
  // states containing workflow 0, by popcount
  std::vector<std::vector<uint32_t>> lv(n + 1);
  for (uint32_t S = 1; S < (1u << n); S += 2) lv[__builtin_popcount(S)].push_back(S);
  const size_t nst = (size_t)1 << (n - 1);
  const DpLayout L = dp_layout(p, n, ns, ioff.back(), nst);
  unsigned char *ws = (unsigned char *)d_ws;
  cudaStream_t s = (cudaStream_t)stream;
  DpParams dp;
  p.blob = ws + L.blob;
  dp.p = p;
  dp.n = n;
  dp.ns = ns;
  dp.nfull = (int)ioff.back();
  dp.smask = (const uint32_t *)(ws + L.smask);
  dp.ioff = (const unsigned long long *)(ws + L.ioff);
  dp.sid = (const int *)(ws + L.sid);
  dp.items = (PPt *)(ws + L.items);
  dp.icnt = (int *)(ws + L.icnt);
  dp.pf = (PPt *)(ws + L.pf);
  dp.pfcnt = (int *)(ws + L.pfcnt);
  dp.fr = (DPt *)(ws + L.fr);
  dp.frcnt = (int *)(ws + L.frcnt);
  dp.ctr = (unsigned long long *)(ws + L.ctr);
  CKD(cudaMemsetAsync(ws + L.ctr, 0, 8 * kDpN, s));
  CKD(cudaMemsetAsync(ws + L.frcnt, 0, 4 * nst * (G + 1), s));
  CKD(cudaMemcpyAsync(ws + L.blob, blob.data(), blob.size(), cudaMemcpyHostToDevice, s));
  CKD(cudaMemcpyAsync(ws + L.smask, smask.data(), 4 * smask.size(), cudaMemcpyHostToDevice, s));
  CKD(cudaMemcpyAsync(ws + L.ioff, ioff.data(), 8 * ioff.size(), cudaMemcpyHostToDevice, s));
  CKD(cudaMemcpyAsync(ws + L.sid, sid.data(), 4 * sid.size(), cudaMemcpyHostToDevice, s));
  int dev = 0, nsm = 0;
  CKD(cudaGetDevice(&dev));
  CKD(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  const size_t smem = ((p.blob_bytes + 15) & ~15u) +
                      (p.scope == SCHED_PER_CLIENT && acc64_bytes(p) <= kAcc64Max ? acc64_bytes(p) : 0) +
                      sizeof(double) * kScr * (256 / 32);
  CKD(cudaFuncSetAttribute(k_pf_items, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  // per-level state lists (uploaded once, consecutive), before the timed region
  std::vector<uint32_t> all;
  std::vector<size_t> at(n + 1, 0);
  for (int m = 1; m <= n; m++) {
    at[m] = all.size();
    all.insert(all.end(), lv[m].begin(), lv[m].end());
  }
  CKD(cudaMemcpyAsync(ws + L.states, all.data(), 4 * all.size(), cudaMemcpyHostToDevice, s));
  // every kernel of the DP loaded before the timed region too (lazy module
  // loading loads a function at its first launch, inside the events otherwise)
  cudaFuncAttributes fa;
  CKD(cudaFuncGetAttributes(&fa, k_pf_merge));
  CKD(cudaFuncGetAttributes(&fa, k_dp_level));
  CKD(cudaFuncGetAttributes(&fa, k_dp_final));
  // the timed region (ms) holds the kernels only: uploads above, pageable or
  // not, and the attribute call complete before e0 is recorded
  CKD(cudaStreamSynchronize(s));
  EventGuard<2> ev;  // destroyed on every return path
  if (!ev.create()) return SCHED_E_CUDA;
  cudaEvent_t e0 = ev[0], e1 = ev[1];
  CKD(cudaEventRecord(e0, s));
  int nl = 0;
  if (dp.nfull > 0) {
    k_pf_items<<<nsm * 4, 256, smem, s>>>(dp);
    CKD(cudaGetLastError());
    nl++;
    k_pf_merge<<<std::max(1, std::min(nsm * 8, (ns + 7) / 8)), 256, 0, s>>>(dp);
    CKD(cudaGetLastError());
    nl++;
  }
  for (int m = 1; m <= n; m++) {
    const int nsts = (int)lv[m].size();
    if (!nsts) continue;
    const int warps = nsts * G;
    k_dp_level<<<(warps + 7) / 8, 256, 0, s>>>(dp, m, nsts, (const uint32_t *)(ws + L.states) + at[m]);
    CKD(cudaGetLastError());
    nl++;
  }
  const int cap = kFM * G;
  k_dp_final<<<1, 32, 0, s>>>(dp, (DpOut *)(ws + L.out), cap, (int *)(ws + L.nout), (int *)(ws + L.nout) + 2);
  CKD(cudaGetLastError());
  nl++;
  CKD(cudaEventRecord(e1, s));
  unsigned long long ctr[kDpN];
  int hdr[2 + kMaxW];
  CKD(cudaMemcpyAsync(ctr, ws + L.ctr, sizeof ctr, cudaMemcpyDeviceToHost, s));
  CKD(cudaMemcpyAsync(hdr, ws + L.nout, sizeof hdr, cudaMemcpyDeviceToHost, s));
  CKD(cudaStreamSynchronize(s));
  const int nout = hdr[0];
  for (int w = 0; w < q.nw; w++) best_pos[w] = hdr[2 + w];
  std::vector<DpOut> outv((size_t)std::min(nout, cap));
  if (!outv.empty()) {
    CKD(cudaMemcpyAsync(outv.data(), ws + L.out, sizeof(DpOut) * outv.size(), cudaMemcpyDeviceToHost, s));
    CKD(cudaStreamSynchronize(s));
  }
  CKD(cudaEventElapsedTime(ms, e0, e1));
  *launches = nl;
  if (ctr[kDpErr]) return SCHED_E_CAPACITY;
  if (nout > cap) return SCHED_E_CAPACITY;
  front->clear();
  for (const DpOut &o : outv) {
    DpPoint d;
    std::memset(&d, 0, sizeof d);
    d.t = o.t;
    d.e = o.e;
    d.k = o.k;
    for (int g = 0; g < o.k; g++) {
      const uint32_t B = o.groups[g];
      std::vector<int> digits(n, 0);
      uint32_t x = o.vecs[g];
      if (q.scope == SCHED_PER_GPU) {
        for (int i = 0; i < n; i++)
          if (B >> i & 1u) digits[i] = (int)x;
      } else {
        for (int i = n - 1; i >= 0; i--)
          if (B >> i & 1u) {
            digits[i] = (int)(x % (uint32_t)q.L);
            x /= (uint32_t)q.L;
          }
      }
      for (int i = 0; i < n; i++)
        if (B >> i & 1u) {
          d.group_of[i] = (int8_t)g;
          d.level_of[i] = (int8_t)digits[i];
        }
    }
    front->push_back(d);
  }
  return SCHED_OK;
}

}  // namespace sched
