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
// bucket of a positive normalised makespan (monotone non-decreasing in v)
__device__ __forceinline__ int bucket_of(float v, uint32_t base) {
  const int b = (int)(__float_as_uint(v) >> kBucketShift) - (int)base;
  return b < 0 ? 0 : (b >= kBuckets ? kBuckets - 1 : b);
}

// Per-warp exclusive prefix-min of the global raw staircase:
// pm[i] = min_{j<i} raw[j].  All 32 lanes must call.
__device__ __forceinline__ void refresh_stair(float *pm, const unsigned int *raw) {
  const int lane = threadIdx.x & 31;
  constexpr int K = kBuckets / 32;
  float v[K];
#pragma unroll
  for (int k = 0; k < K; k++) v[k] = __uint_as_float(__ldcg(raw + lane * K + k));
  float run = __int_as_float(0x7f800000);
  float ex[K];
#pragma unroll
  for (int k = 0; k < K; k++) {
    ex[k] = run;
    run = fminf(run, v[k]);
  }
  // exclusive scan of lane totals
  float pre = run;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    float x = __shfl_up_sync(0xffffffffu, pre, o);
    if (lane >= o) pre = fminf(pre, x);
  }
  float excl = __shfl_up_sync(0xffffffffu, pre, 1);
  if (lane == 0) excl = __int_as_float(0x7f800000);
#pragma unroll
  for (int k = 0; k < K; k++) pm[lane * K + k] = fminf(excl, ex[k]);
  __syncwarp();
}

// ---------------------------------------------------------- fp64 refine
// Canonical score in fp64: explicit
// round-to-nearest intrinsics, no contraction, same order as the oracle.
// members[g] = bitmask of group g; lam[i] = level digit of workflow i.
__device__ __forceinline__ void refine64(const Tables &tb, const DevParams &p, const uint32_t *members,
                                         int k, const int *lam, double *Tout, double *Eout) {
  const double ps = p.ps;
  double T = 0.0, E = 0.0;
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
    for (uint32_t mm = m; mm; mm &= mm - 1) {
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
    const double Eg = __dadd_rn(__dmul_rn(ps, Tg), D);
    if (Tg > T) T = Tg;
    E = __dadd_rn(E, Eg);
  }
  *Tout = T;
  *Eout = E;
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
__device__ __forceinline__ void emit_candidate(const DevParams &p, float *pm, u64 idx, double T, double E,
                                               float t32, float e32) {
  const unsigned long long slot = atomicAdd(p.ctr + kCtrCand, 1ull);
  if (slot < p.cand_cap) {
    CandRec *c = (CandRec *)p.cand + slot;
    c->idx = idx;
    c->t = T;
    c->e = E;
    c->t32 = t32;
    c->e32 = e32;
  } else {
    atomicExch(p.ctr + kCtrOverflow, 1ull);
  }
  const double g1 = 1.0 + (double)p.gamma;
  const float key = __double2float_ru(__dmul_ru(__ddiv_ru(T, p.tseq), g1));
  const float val = __double2float_ru(__dmul_ru(__ddiv_ru(E, p.eseq), g1));
  const int jb = bucket_of(key, p.bucket_base);
  atomicMin(p.stair + jb, __float_as_uint(val));
  for (int i = jb + 1; i < kBuckets; i++) atomicMin((unsigned int *)pm + i, __float_as_uint(val));
}

}  // namespace sched
