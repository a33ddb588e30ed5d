// device_common.cuh -- device helpers shared by the search kernels:
// staged tables, DP unrank / successor, fp32 group scoring, the fp64
// canonical refine, the fp32 screens and the best / Pareto bookkeeping.
//
// PAPER.md = /root/reference/PAPER.md; R<n> = DESIGN.md readings.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "sched_internal.hpp"

namespace sched {

typedef unsigned long long u64;

struct Tables {
  const float *th, *u, *bw, *dh, *traw, *praw, *d;
  const int *mem;
  const u64 *W;
  const uint16_t *trans;
};

__device__ __forceinline__ Tables tables_at(const unsigned char *base, const DevParams &p) {
  Tables t;
  t.th = (const float *)(base + p.off_th);
  t.u = (const float *)(base + p.off_u);
  t.bw = (const float *)(base + p.off_bw);
  t.dh = (const float *)(base + p.off_dh);
  t.traw = (const float *)(base + p.off_traw);
  t.praw = (const float *)(base + p.off_praw);
  t.d = (const float *)(base + p.off_d);
  t.mem = (const int *)(base + p.off_mem);
  t.W = (const u64 *)(base + p.off_W);
  t.trans = (const uint16_t *)(base + p.off_trans);
  return t;
}

// Stage the table blob global -> shared memory once per CTA with the bulk
// copy engine (cp.async.bulk, 1-D TMA) completing on an mbarrier.
__device__ __forceinline__ void stage_blob(unsigned char *sm, const DevParams &p) {
  __shared__ __align__(8) unsigned long long mbar;
  const uint32_t bytes = p.blob_bytes;  // multiple of 16
  const uint32_t bar = (uint32_t)__cvta_generic_to_shared(&mbar);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
                 : "memory");
    const uint32_t dst = (uint32_t)__cvta_generic_to_shared(sm);
    const uint32_t kMax = 65536;  // split into <= 64 KiB bulk copies
    for (uint32_t o = 0; o < bytes; o += kMax) {
      const uint32_t nb = bytes - o < kMax ? bytes - o : kMax;
      asm volatile(
          "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
              dst + o),
          "l"(p.blob + o), "r"(nb), "r"(bar)
          : "memory");
    }
  }
  // every thread waits for phase 0 to complete
  asm volatile(
      "{\n .reg .pred P;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n"
      " @!P bra WAIT_%=;\n}" ::"r"(bar)
      : "memory");
}

// --------------------------------------------------------------- staircase
// Sound Pareto screen.  Verified (fp64) points p
// are keyed by their EXACT canonical makespan T_p (buckets of the fp64 bits
// of T, monotone) and carry val_p = up(E_p/E_seq * (1+gamma)) >= the fp32
// error band of any E.  A configuration with exact T and fp32 Ehat is
// dominated by p if T >= T_p and Ehat > val_p (then E > E_p exactly):
//   pm[j] = min val over points in buckets < j        (T > T_p for sure)
//   bp[j] = min (val << 32 | slot) over points in bucket j; the point's
//           exact T is read back from the candidate buffer slot.
// Equal-T ties (configurations sharing a bottleneck group) are therefore
// screened exactly.  All updates are monotone minima (race-free merges).
//   pe[j] = min EXACT fp64 E (bits) over points in buckets < j: a configuration
//           with exact (T, E), T in bucket j, is dominated if E >= pe[j]
//           (exact ties in E, e.g. the constant-energy plateaus of the power
//           cap model R28, are screened exactly).
struct Stair {
  unsigned int *pm;
  unsigned long long *bp;
  unsigned long long *pe;
};

// the CTA staircase in shared memory at `base` (kStairSmem bytes)
__device__ __forceinline__ Stair stair_at(unsigned char *base) {
  return Stair{(unsigned int *)(base + 16 * kBuckets), (unsigned long long *)base,
               (unsigned long long *)(base + 8 * kBuckets)};
}

__device__ __forceinline__ int bucket_of(double T, const DevParams &p) {
  const int b = (int)((unsigned long long)__double_as_longlong(T) >> p.bucket_shift) - (int)p.bucket_base;
  return b < 0 ? 0 : (b >= kBuckets ? kBuckets - 1 : b);
}

__device__ __forceinline__ void stair_init(Stair s) {
  for (int i = threadIdx.x; i < kBuckets; i += blockDim.x) {
    s.pm[i] = 0x7f800000u;
    s.bp[i] = ~0ull;
    s.pe[i] = ~0ull;
  }
}

// Warp-cooperative merge of the global staircase into a CTA staircase.
__device__ __forceinline__ void stair_merge(Stair s, const DevParams &p) {
  const int lane = threadIdx.x & 31;
  constexpr int K = kBuckets / 32;
  const int j0 = lane * K;
  unsigned int tot = 0x7f800000u;
  for (int k = 0; k < K; k++) {
    tot = min(tot, __ldcg(p.stv + j0 + k));
    const unsigned long long x = __ldcg(p.stp + j0 + k);
    if (x < s.bp[j0 + k]) atomicMin(s.bp + j0 + k, x);
  }
  unsigned int pre = tot;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned int x = __shfl_up_sync(0xffffffffu, pre, o);
    if (lane >= o) pre = min(pre, x);
  }
  unsigned int run = __shfl_up_sync(0xffffffffu, pre, 1);
  if (lane == 0) run = 0x7f800000u;
  for (int k = 0; k < K; k++) {
    if (run < s.pm[j0 + k]) atomicMin(s.pm + j0 + k, run);
    run = min(run, __ldcg(p.stv + j0 + k));
  }
  // exact-E prefix minima
  unsigned long long te = ~0ull;
  for (int k = 0; k < K; k++) te = min(te, __ldcg(p.ste + j0 + k));
  unsigned long long pre_e = te;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long x = __shfl_up_sync(0xffffffffu, pre_e, o);
    if (lane >= o) pre_e = min(pre_e, x);
  }
  unsigned long long run_e = __shfl_up_sync(0xffffffffu, pre_e, 1);
  if (lane == 0) run_e = ~0ull;
  for (int k = 0; k < K; k++) {
    if (run_e < s.pe[j0 + k]) atomicMin(s.pe + j0 + k, run_e);
    run_e = min(run_e, __ldcg(p.ste + j0 + k));
  }
  __threadfence_block();
  __syncwarp();
}

// T: exact canonical fp64 makespan (or a lower bound of it that is itself an
// exact canonical makespan); eh: fp32 normalised energy (or a lower bound).
__device__ __forceinline__ bool stair_dominated(const Stair &s, const DevParams &p, double T, float eh) {
  const int j = bucket_of(T, p);
  const unsigned int eb = __float_as_uint(eh);
  if (eb > s.pm[j]) return true;
  const unsigned long long pr = s.bp[j];
  if (eb > (unsigned int)(pr >> 32)) {
    const CandRec *c = (const CandRec *)p.cand + (unsigned int)pr;
    return T >= __ldcg(&c->t);
  }
  return false;
}

// Exact domination of a configuration with exact canonical (T, E) by a
// verified point: one in a strictly lower T bucket with E_p <= E, or the
// bucket's recorded point.  Sound (only verified points), used after the
// fp64 re-score, before a candidate is emitted.
__device__ __forceinline__ bool stair_dominated_exact(const Stair &s, const DevParams &p, double T, double E) {
  const int j = bucket_of(T, p);
  if ((unsigned long long)__double_as_longlong(E) >= s.pe[j]) return true;
  const unsigned long long pr = s.bp[j];
  if ((unsigned int)pr != 0xffffffffu) {
    const CandRec *c = (const CandRec *)p.cand + (unsigned int)pr;
    const double ct = __ldcg(&c->t), ce = __ldcg(&c->e);
    return ct <= T && ce <= E && (ct < T || ce < E);
  }
  return false;
}

// ---------------------------------------------------------- fp64 refine
// Canonical score in fp64: explicit
// round-to-nearest intrinsics, no contraction, same order as the oracle.
// members[g] = bitmask of group g; lam[i] = level digit of workflow i.
__device__ __forceinline__ void refine64(const Tables &tb, const DevParams &p, const uint32_t *members,
                                         int k, const int *lam, double *Tout, double *Eout) {
  const double ps = p.ps;
  double T = 0.0, E = 0.0, Dall = 0.0;
  for (int g = 0; g < k; g++) {
    const uint32_t m = members[g];
    double U = 0.0, B = 0.0;
    for (uint32_t mm = m; mm; mm &= mm - 1) {
      const int i = __ffs(mm) - 1, r = i * p.L + lam[i];
      U = __dadd_rn(U, (double)tb.u[r]);
      B = __dadd_rn(B, (double)tb.bw[r]);
    }
    double c = 1.0;
    if (U > c) c = U;
    if (B > c) c = B;
    double Tg = 0.0;
    if (p.model & SCHED_MODEL_TIME_SLICE) {  // R30: slices one after another at the solo profile
      for (uint32_t mm = m; mm; mm &= mm - 1) {
        const int r = (__ffs(mm) - 1) * p.L + lam[__ffs(mm) - 1];
        double tau = (double)tb.traw[r];
        if (p.model & SCHED_MODEL_POWER_CAP) {
          const double tc = __ddiv_rn(__dmul_rn(__dsub_rn((double)tb.praw[r], ps), tau), p.capd);
          if (tc > tau) tau = tc;
        }
        Tg = __dadd_rn(Tg, tau);
      }
    }
    for (uint32_t mm = (p.model & SCHED_MODEL_TIME_SLICE) ? 0u : m; mm; mm &= mm - 1) {
      const int i = __ffs(mm) - 1, ri = i * p.L + lam[i];
      double sigma = 1.0;
      for (uint32_t m2 = m & ~(1u << i); m2; m2 &= m2 - 1) {
        const int j = __ffs(m2) - 1, rj = j * p.L + lam[j];
        sigma = __dadd_rn(sigma, (double)tb.d[ri * p.ds + rj]);
      }
      const double tau = __dmul_rn(__dmul_rn((double)tb.traw[ri], sigma), c);
      if (tau > Tg) Tg = tau;
    }
    double D = 0.0;
    for (uint32_t mm = m; mm; mm &= mm - 1) {
      const int i = __ffs(mm) - 1, r = i * p.L + lam[i];
      D = __dadd_rn(D, __dmul_rn(__dsub_rn((double)tb.praw[r], ps), (double)tb.traw[r]));
    }
    if ((p.model & (SCHED_MODEL_POWER_CAP | SCHED_MODEL_TIME_SLICE)) == SCHED_MODEL_POWER_CAP) {  // R28
      const double tc = __ddiv_rn(D, p.capd);
      if (tc > Tg) Tg = tc;
    }
    const double Eg = __dadd_rn(__dmul_rn(ps, Tg), D);
    if (Tg > T) T = Tg;
    E = __dadd_rn(E, Eg);
    Dall = __dadd_rn(Dall, D);
  }
  if (p.model & SCHED_MODEL_COUNT_IDLE) E = __dadd_rn(__dmul_rn(p.gps, T), Dall);  // R26
  *Tout = T;
  *Eout = E;
}

// R27 (NO_INTERFERENCE): every group's combined SM and BW utilisation, summed
// in fp64 in ascending member order exactly as the oracle, is <= 1.
__device__ __forceinline__ bool no_interference64(const Tables &tb, const DevParams &p, const uint32_t *members,
                                                  int k, const int *lam) {
  for (int g = 0; g < k; g++) {
    double U = 0.0, B = 0.0;
    for (uint32_t mm = members[g]; mm; mm &= mm - 1) {
      const int i = __ffs(mm) - 1, r = i * p.L + lam[i];
      U = __dadd_rn(U, (double)tb.u[r]);
      B = __dadd_rn(B, (double)tb.bw[r]);
    }
    if (U > 1.0 || B > 1.0) return false;
  }
  return true;
}

__device__ __forceinline__ double objective64(const DevParams &p, double T, double E, int a, int b) {
  const double X = __ddiv_rn(p.tseq, T), Y = __ddiv_rn(p.eseq, E);
  double F = 1.0;
  for (int i = 0; i < a; i++) F = __dmul_rn(F, X);
  for (int i = 0; i < b; i++) F = __dmul_rn(F, Y);
  return F;
}

__device__ __forceinline__ bool better(double f1, u64 i1, double f2, u64 i2) {
  return f1 > f2 || (f1 == f2 && i1 < i2);
}

__device__ __forceinline__ void best_init(BestRec &b) {
  b.f = -1.0;
  b.idx = ~0ull;
  b.t = b.e = 0.0;
  b.t32 = b.e32 = 0.f;
  b.valid = 0;
  b.pad = 0;
}

// warp-reduce a BestRec (all lanes get the winner)
__device__ __forceinline__ void warp_best(BestRec &b) {
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    BestRec x;
    x.f = __shfl_xor_sync(0xffffffffu, b.f, o);
    x.idx = __shfl_xor_sync(0xffffffffu, b.idx, o);
    x.t = __shfl_xor_sync(0xffffffffu, b.t, o);
    x.e = __shfl_xor_sync(0xffffffffu, b.e, o);
    x.t32 = __shfl_xor_sync(0xffffffffu, b.t32, o);
    x.e32 = __shfl_xor_sync(0xffffffffu, b.e32, o);
    x.valid = __shfl_xor_sync(0xffffffffu, b.valid, o);
    x.pad = 0;
    if (x.valid && (!b.valid || better(x.f, x.idx, b.f, b.idx))) b = x;
  }
}

// Record a refined (fp64-exact) feasible configuration as a Pareto candidate
// and tighten the staircases (sound: only verified points enter).
__device__ __forceinline__ void emit_candidate(const DevParams &p, Stair s, u64 idx, double T, double E,
                                               float t32, float e32) {
  const unsigned long long slot = atomicAdd(p.ctr + kCtrCand, 1ull);
  const double g1 = 1.0 + (double)p.gamma;
  const float val = __double2float_ru(__dmul_ru(__ddiv_ru(E, p.eseq), g1));
  const unsigned int vb = __float_as_uint(val);
  const int jb = bucket_of(T, p);
  bool improved = false;
  if (vb < __ldcg(p.stv + jb)) {
    atomicMin(p.stv + jb, vb);
    improved = true;
  }
  unsigned long long pr = ((unsigned long long)vb << 32) | 0xffffffffull;  // val-only entry
  if (slot < p.cand_cap) {
    CandRec *c = (CandRec *)p.cand + slot;
    c->idx = idx;
    c->t = T;
    c->e = E;
    c->t32 = t32;
    c->e32 = e32;
    __threadfence();  // the record is visible before its slot is published
    pr = ((unsigned long long)vb << 32) | slot;
    if (pr < __ldcg(p.stp + jb)) {
      atomicMin(p.stp + jb, pr);
      improved = true;
    }
    atomicMin(s.bp + jb, pr);
    const unsigned long long eb = (unsigned long long)__double_as_longlong(E);
    if (eb < __ldcg(p.ste + jb)) {
      atomicMin(p.ste + jb, eb);
      improved = true;
    }
    const int hie = jb + 64 < kBuckets ? jb + 64 : kBuckets;
    for (int i = jb + 1; i < hie; i++) atomicMin(s.pe + i, eb);
  } else {
    atomicExch(p.ctr + kCtrOverflow, 1ull);
  }
  if (improved) {  // publish in the insertion log (seq = version)
    const unsigned long long seq = atomicAdd(p.ctr + kCtrStairVer, 1ull);
    LogEnt *L = (LogEnt *)p.stlog + (seq % kLog);
    L->pr = pr;
    L->jb = (unsigned int)jb;
    __threadfence();
    atomicExch(&L->tag, (unsigned int)(seq + 1));
  }
  const int hi = jb + 64 < kBuckets ? jb + 64 : kBuckets;
  for (int i = jb + 1; i < hi; i++) atomicMin(s.pm + i, vb);
}

// Bring this warp's view of the CTA staircase up to date with the global
// insertion log (entries pos .. version-1); falls back to a full merge when
// the ring buffer has wrapped.  Idempotent (monotone minima).  All lanes call.
__device__ __forceinline__ void stair_sync(Stair s, const DevParams &p, u64 &pos, u64 ver) {
  ver = __shfl_sync(0xffffffffu, ver, 0);  // one view of the version for the whole warp
  if (ver == pos) return;
  if (ver - pos > (u64)kLog) {
    stair_merge(s, p);
    pos = ver;
    return;
  }
  const int lane = threadIdx.x & 31;
  for (u64 q = pos; q < ver; q++) {
    // lane 0 reads the entry (acquire on its tag) and broadcasts it: every
    // lane must take the same branch (the ballots below need the full warp)
    unsigned int tag = 0, jb = 0;
    unsigned long long pr = 0;
    if (lane == 0) {
      const LogEnt *L = (const LogEnt *)p.stlog + (q % kLog);
      asm volatile("ld.acquire.gpu.u32 %0, [%1];" : "=r"(tag) : "l"(&L->tag) : "memory");
      pr = __ldcg(&L->pr);
      jb = __ldcg(&L->jb);
    }
    tag = __shfl_sync(0xffffffffu, tag, 0);
    if (tag != (unsigned int)(q + 1)) {  // not yet visible: stop here
      pos = q;
      return;
    }
    pr = __shfl_sync(0xffffffffu, pr, 0);
    jb = __shfl_sync(0xffffffffu, jb, 0);
    const unsigned int vb = (unsigned int)(pr >> 32);
    if (lane == 0 && (unsigned int)pr != 0xffffffffu && pr < s.bp[jb]) atomicMin(s.bp + jb, pr);
    for (int i0 = (int)jb + 1; i0 < kBuckets; i0 += 32) {  // pm is non-increasing: stop at the first pm <= val
      const int i = i0 + lane;
      const bool need = i < kBuckets && s.pm[i] > vb;
      if (need) atomicMin(s.pm + i, vb);
      if (__ballot_sync(0xffffffffu, need) != 0xffffffffu) break;
    }
    if ((unsigned int)pr != 0xffffffffu) {  // exact E of the recorded point
      unsigned long long eb = 0;
      if (lane == 0) eb = (unsigned long long)__double_as_longlong(__ldcg(&((const CandRec *)p.cand + (unsigned int)pr)->e));
      eb = __shfl_sync(0xffffffffu, eb, 0);
      for (int i0 = (int)jb + 1; i0 < kBuckets; i0 += 32) {  // pe is non-increasing as well
        const int i = i0 + lane;
        const bool need = i < kBuckets && s.pe[i] > eb;
        if (need) atomicMin(s.pe + i, eb);
        if (__ballot_sync(0xffffffffu, need) != 0xffffffffu) break;
      }
    }
  }
  pos = ver;
  __syncwarp();
}

// fp32 tuple + exact canonical fp64 (T_g, E_g) of group `m` with every member
// at level mu (canonical order of DESIGN.md section 2, as in refine64).
// Returns false if the group is infeasible under NO_INTERFERENCE (R27).
__device__ __forceinline__ bool group_eval(const Tables &tb, const DevParams &p, uint32_t m, int mu,
                                           float &t32, float &e32, double &t64, double &e64) {
  const int L = p.L;
  float U = 0.f, B = 0.f, D = 0.f;
  double U64 = 0.0, B64 = 0.0, D64 = 0.0;
  for (uint32_t mm = m; mm; mm &= mm - 1) {
    const int r = (__ffs(mm) - 1) * L + mu;
    U += tb.u[r];
    B += tb.bw[r];
    D += tb.dh[r];
    U64 = __dadd_rn(U64, (double)tb.u[r]);
    B64 = __dadd_rn(B64, (double)tb.bw[r]);
  }
  if ((p.model & SCHED_MODEL_NO_INTERFERENCE) && (U64 > 1.0 || B64 > 1.0)) return false;
  const float cg = fmaxf(fmaxf(1.f, U), B);
  double c = 1.0;
  if (U64 > c) c = U64;
  if (B64 > c) c = B64;
  float Tg = 0.f;
  double Tg64 = 0.0;
  if (p.model & SCHED_MODEL_TIME_SLICE) {  // R30: the slices one after another (per-slice cap)
    for (uint32_t mm = m; mm; mm &= mm - 1) {
      const int r = (__ffs(mm) - 1) * L + mu;
      double tau = (double)tb.traw[r];
      if (p.model & SCHED_MODEL_POWER_CAP) {
        Tg += fmaxf(tb.th[r], tb.dh[r] * p.kcap);
        const double tc = __ddiv_rn(__dmul_rn(__dsub_rn((double)tb.praw[r], p.ps), tau), p.capd);
        if (tc > tau) tau = tc;
      } else {
        Tg += tb.th[r];
      }
      Tg64 = __dadd_rn(Tg64, tau);
    }
  }
  for (uint32_t mm = (p.model & SCHED_MODEL_TIME_SLICE) ? 0u : m; mm; mm &= mm - 1) {
    const int i = __ffs(mm) - 1, ri = i * L + mu;
    float s = 1.f;
    double s64 = 1.0;
    for (uint32_t m2 = m & ~(1u << i); m2; m2 &= m2 - 1) {
      const float dv = tb.d[ri * p.ds + (__ffs(m2) - 1) * L + mu];
      s += dv;
      s64 = __dadd_rn(s64, (double)dv);
    }
    Tg = fmaxf(Tg, tb.th[ri] * s * cg);
    const double tau = __dmul_rn(__dmul_rn((double)tb.traw[ri], s64), c);
    if (tau > Tg64) Tg64 = tau;
  }
  for (uint32_t mm = m; mm; mm &= mm - 1) {
    const int r = (__ffs(mm) - 1) * L + mu;
    D64 = __dadd_rn(D64, __dmul_rn(__dsub_rn((double)tb.praw[r], p.ps), (double)tb.traw[r]));
  }
  if ((p.model & (SCHED_MODEL_POWER_CAP | SCHED_MODEL_TIME_SLICE)) == SCHED_MODEL_POWER_CAP) {
    // R28: throttled to P_cap, dynamic energy conserved
    Tg = fmaxf(Tg, D * p.kcap);
    const double tc = __ddiv_rn(D64, p.capd);
    if (tc > Tg64) Tg64 = tc;
  }
  t32 = Tg;
  t64 = Tg64;
  if (p.model & SCHED_MODEL_COUNT_IDLE) {
    // R26: E = G P_s T + sum_g D_g -- the record carries D_g only; the tile
    // kernel adds kidle * T (fp32) / gps * T (fp64) per configuration
    e32 = D;
    e64 = D64;
  } else {
    e32 = p.phat * Tg + D;
    e64 = __dadd_rn(__dmul_rn(p.ps, Tg64), D64);
  }
  return true;
}

// a configuration's fp32 E-hat from its T-hat and the sum of its group
// records' e32 (COUNT_IDLE: the records hold D-hat, R26: E = kidle T + D;
// monotone in both arguments, so min-reduced corners stay exact bounds)
__device__ __forceinline__ float e_total(const DevParams &p, float T, float esum) {
  return (p.model & SCHED_MODEL_COUNT_IDLE) ? fmaf(p.kidle, T, esum) : esum;
}

// ------------------------------------------------------------ DP walk (RGS state)
struct LaneCfg {
  int8_t a[kMaxN];
  uint16_t st[kMaxN];   // st[i] = DP state after placing element i
  uint32_t mask[kMaxG];
  int8_t sz[kMaxG];
  int k;
  u64 v, Pn;            // level residue in [0, Pn), Pn = L^(#digits)
  bool feasible;
};

__device__ __forceinline__ void cfg_feasibility(const Tables &tb, const DevParams &p, LaneCfg &c) {
  bool ok = true;
  for (int g = 0; g < c.k; g++) {
    long long M = 0;
    for (uint32_t mm = c.mask[g]; mm; mm &= mm - 1) M += tb.mem[__ffs(mm) - 1];
    ok &= M <= (long long)p.mem_cap;
  }
  c.feasible = ok;
}

__device__ __forceinline__ int col_for(const DevParams &p, int j, int b, const int8_t *sz) {
  if (j < b) {
    if (p.capped) return sz[j] >= p.c ? -1 : sz[j];
    return 1;
  }
  return b >= p.g ? -1 : 0;
}

__device__ __forceinline__ void place(LaneCfg &c, int i, int j) {
  c.a[i] = (int8_t)j;
  if (j == c.k) {
    c.sz[c.k] = 0;
    c.mask[c.k] = 0;
    c.k++;
  }
  c.sz[j]++;
  c.mask[j] |= 1u << i;
}

// index -> (RGS, residue) through the DP count table (R4 index order)
static __device__ bool dev_unrank(const Tables &tb, const DevParams &p, u64 idx, LaneCfg &c) {
  u64 r = idx;
  int s = p.root;
  c.k = 0;
  place(c, 0, 0);
  c.st[0] = (uint16_t)s;
  for (int i = 1; i < p.n; i++) {
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
    if (chosen < 0) return false;
    place(c, i, chosen);
    c.st[i] = (uint16_t)s;
  }
  c.Pn = tb.W[c.st[p.n - 1]];
  c.v = r;
  cfg_feasibility(tb, p, c);
  return true;
}

// next RGS in lexicographic order (valid + completable), digits reset by caller
static __device__ bool dev_successor(const Tables &tb, const DevParams &p, LaneCfg &c) {
  for (int i = p.n - 1; i >= 1; i--) {
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
      for (int m = i + 1; m < p.n; m++) {  // greedy lexicographically-smallest completion
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

__device__ __forceinline__ bool dev_advance(const Tables &tb, const DevParams &p, LaneCfg &c, u64 m) {
  c.v += m;
  while (c.v >= c.Pn) {
    c.v -= c.Pn;
    if (!dev_successor(tb, p, c)) return false;
    c.Pn = tb.W[c.st[p.n - 1]];
    cfg_feasibility(tb, p, c);
  }
  return true;
}

}  // namespace sched
