// search_tile.cuh -- PER_GPU tile kernel (c3 / c4 fast path).
//
// In PER_GPU scope a configuration is (partition, one level per group) and
// the score decomposes over groups:
//   T = max_g T_g(mu_g),  E = sum_g E_g(mu_g),  feasibility per partition.
// A warp walks consecutive partitions of its index unit.  Per partition the
// lanes evaluate the k x L group tuples once (fp32 T_g/T_seq, E_g/E_seq and
// the exact fp64 canonical T_g) into per-warp shared memory; the L^k level
// vectors are then scored per configuration from registers:
//   tile = the L^2 level pairs of the last two groups (register-resident),
//   prefix = max/sum over groups 0..k-3 (per-lane odometer, compile-time k).
// Every configuration's (T, E) and product-metric proxies T^a E^b are
// computed; per tile the proxies are min-reduced and compared with the
// running threshold (fp32 margin delta_w), and the tile's exact corner
// (min fp64 T, min fp32 E) is screened against the Pareto staircase.  A tile
// that is not cleared re-checks its configurations one by one and re-scores
// candidates in fp64 (refine64), exactly like the generic kernel.
#pragma once
#include "device_common.cuh"
#include "tile_registry.hpp"

namespace sched {

// ---- compile-time product-metric sets: q_s = (T/T_seq)^a (E/E_seq)^b ----
struct WS_P {  // Pareto only
  static constexpr bool RT = false;
  static constexpr bool DUMP = false;
  static constexpr int N = 0;
  __host__ __device__ static constexpr int A(int s) { return 0; }
  __host__ __device__ static constexpr int B(int s) { return 0; }
  __device__ static __forceinline__ void q(float, float, float *) {}
};
struct WS_11 {
  static constexpr bool RT = false;
  static constexpr bool DUMP = false;
  static constexpr int N = 1;
  __host__ __device__ static constexpr int A(int s) { return 1; }
  __host__ __device__ static constexpr int B(int s) { return 1; }
  __device__ static __forceinline__ void q(float T, float E, float *o) { o[0] = E * T; }
};
struct WS_10 {
  static constexpr bool RT = false;
  static constexpr bool DUMP = false;
  static constexpr int N = 1;
  __host__ __device__ static constexpr int A(int s) { return 1; }
  __host__ __device__ static constexpr int B(int s) { return 0; }
  __device__ static __forceinline__ void q(float T, float, float *o) { o[0] = T; }
};
struct WS_01 {
  static constexpr bool RT = false;
  static constexpr bool DUMP = false;
  static constexpr int N = 1;
  __host__ __device__ static constexpr int A(int s) { return 0; }
  __host__ __device__ static constexpr int B(int s) { return 1; }
  __device__ static __forceinline__ void q(float, float E, float *o) { o[0] = E; }
};
struct WS_11_21 {  // c4: [T x E], [T x T x E]
  static constexpr bool RT = false;
  static constexpr bool DUMP = false;
  static constexpr int N = 2;
  __host__ __device__ static constexpr int A(int s) { return (s == 0 ? 1 : 2); }
  __host__ __device__ static constexpr int B(int s) { return (s == 0 ? 1 : 1); }
  __device__ static __forceinline__ void q(float T, float E, float *o) {
    o[0] = E * T;
    o[1] = o[0] * T;
  }
};
struct WS_C1 {  // (1,0) (0,1) (1,1) (2,1)
  static constexpr bool RT = false;
  static constexpr bool DUMP = false;
  static constexpr int N = 4;
  __host__ __device__ static constexpr int A(int s) { return (s == 0 ? 1 : (s == 1 ? 0 : (s == 2 ? 1 : 2))); }
  __host__ __device__ static constexpr int B(int s) { return (s == 0 ? 0 : (s == 1 ? 1 : (s == 2 ? 1 : 1))); }
  __device__ static __forceinline__ void q(float T, float E, float *o) {
    o[0] = T;
    o[1] = E;
    o[2] = E * T;
    o[3] = o[2] * T;
  }
};
struct WS_SWEEP {  // c5 sweep (1,0) (3,1) (2,1) (1,1) (1,2) (1,3) (0,1)
  static constexpr bool RT = false;
  static constexpr bool DUMP = false;
  static constexpr int N = 7;
  __host__ __device__ static constexpr int A(int s) { return (s == 0 ? 1 : (s == 1 ? 3 : (s == 2 ? 2 : (s == 3 ? 1 : (s == 4 ? 1 : (s == 5 ? 1 : 0)))))); }
  __host__ __device__ static constexpr int B(int s) { return (s == 0 ? 0 : (s == 1 ? 1 : (s == 2 ? 1 : (s == 3 ? 1 : (s == 4 ? 2 : (s == 5 ? 3 : 1)))))); }
  __device__ static __forceinline__ void q(float T, float E, float *o) {
    o[0] = T;
    o[3] = E * T;
    o[2] = o[3] * T;
    o[1] = o[2] * T;
    const float ee = E * E;
    o[4] = ee * T;
    o[5] = (ee * E) * T;
    o[6] = E;
  }
};

// Any W <= 8 product metrics with the exponents read at run time
// (p.wa / p.wb, "different product metrics"): the per-tile
// corner screen evaluates q_w = T^a E^b by repeated multiplication; the
// lane's running thresholds live in its shared-memory row (thr_sm), not in
// registers, so the tile loop's register footprint is that of WS_11_21.
template <int NW, bool B0>
struct WS_RTT {
  static constexpr int N = NW;         // weight slots (the query's p.nw <= NW are used)
  static constexpr bool RT = true;
  static constexpr bool MAYB0 = B0;    // the set may hold b = 0 weights (vote-guarded tile loop)
  static constexpr bool DUMP = false;
  __host__ __device__ static constexpr int A(int) { return 0; }
  __host__ __device__ static constexpr int B(int) { return 0; }
  __device__ static __forceinline__ void q(float, float, float *) {}
};
struct WS_RT : WS_RTT<kMaxW, true> {};
// every b >= 1 (host-checked): the plain tile loop, like the compiled sets
// without b = 0 weights; up to 4 weights with 4 threshold registers
struct WS_RTN : WS_RTT<kMaxW, false> {};
struct WS_RT4N : WS_RTT<4, false> {};

// WS_11 that also writes every configuration's fp32 (T-hat, E-hat), as the
// tile loop computes them, to p.dump (sched_debug_scores32: the hot loop's
// fp32 scores checked against the oracle configuration by configuration)
struct WS_11_DUMP : WS_11 {
  static constexpr bool DUMP = true;
};

template <class WS>
__device__ __forceinline__ void dump_score(const DevParams &p, u64 idx, float T, float E) {
  if constexpr (WS::DUMP) {
    if (idx >= p.dump_lo && idx - p.dump_lo < p.dump_n) ((float2 *)p.dump)[idx - p.dump_lo] = make_float2(T, E);
  }
}

// three-input fp32 max (one FMNMX3, the ALU slot of a two-input max;
// max is exact, so the value is that of fmaxf(fmaxf(a, b), c))
__device__ __forceinline__ float fmax3f(float a, float b, float c) {
  float d;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
  return d;
}

// q_s = (T/T_seq)^a (E/E_seq)^b for query weight s, run-time exponents
__device__ __forceinline__ float rt_q(const DevParams &p, int s, float T, float E) {
  float q = 1.f;
  for (int i = 0; i < p.wa[s]; i++) q *= T;
  for (int i = 0; i < p.wb[s]; i++) q *= E;
  return q;
}


struct WarpPart {
  LaneCfg cfg;
  u64 base;
  u64 ncfg, nfeas;   // configurations scored / feasible (lane 0 counts; shared memory, not registers)
  u64 sver;          // staircase insertion-log position this warp has applied
  float gt[kTileMaxG * 4], ge[kTileMaxG * 4];
  double g64[kTileMaxG * 4];
  double ge64[kTileMaxG * 4];  // exact canonical fp64 E_g per (group, level)
  float2 lp[64];  // loop-prefix (max T, sum E) over groups 0..k-6, one entry per digit string
};

// The lane's running thresholds live in its shared-memory row (thr_sm, the
// master copy, also used by the out-of-line slow paths); the tile screen
// reads their products with 1 + delta from registers: one register per
// weight (the c5 sweep's 7 weights: 7, not 14).
template <class WS>
struct Thr {
  float vm[WS::N > 0 ? WS::N : 1];  // thr_sm[s] * (1 + delta of the weight in slot s)
};

// quick Pareto screen from fp32 values: tlb = certified lower bound of the
// exact makespan T (unnormalised, float, rounded down), eh = fp32 E/E_seq.
// Buckets of a float coincide with buckets of the same value as a double.
__device__ __forceinline__ bool stair_dominated_f(const Stair &s, const DevParams &p, float tlb, float eh) {
  // bits64(x) >> s == (bits32(x) >> (s - 29)) + (896 << (52 - s)) for a float x, s >= 29
  const int b = (int)((__float_as_uint(tlb) >> (p.bucket_shift - 29)) + (896u << (52 - p.bucket_shift))) -
                (int)p.bucket_base;
  const int j = b < 0 ? 0 : (b >= kBuckets ? kBuckets - 1 : b);
  const unsigned int eb = __float_as_uint(eh);
  if (eb > s.pm[j]) return true;
  const unsigned long long pr = s.bp[j];
  if (eb > (unsigned int)(pr >> 32)) {
    const CandRec *c = (const CandRec *)p.cand + (unsigned int)pr;
    return (double)tlb >= __ldcg(&c->t);
  }
  return false;
}

// the CTA staircase's pm / bp arrays as shared-window addresses: the tile
// loop's screen loads them with ld.shared (a generic pointer costs a
// generic LD per tile)
struct StairSm {
  uint32_t pm, bp;
};

__device__ __forceinline__ StairSm stair_sm(const Stair &s) {
  return StairSm{(uint32_t)__cvta_generic_to_shared(s.pm), (uint32_t)__cvta_generic_to_shared(s.bp)};
}

// stair_dominated_f with the bucket from the host-made float-bits constants
// (p.bkt_sh32, p.bkt_off32) and shared-window loads
__device__ __forceinline__ bool stair_dominated_fs(const StairSm &s, const DevParams &p, float tlb, float eh) {
  const int b = (int)((__float_as_uint(tlb) >> p.bkt_sh32) + p.bkt_off32);
  const uint32_t j = (uint32_t)(b < 0 ? 0 : (b >= kBuckets ? kBuckets - 1 : b));
  const unsigned int eb = __float_as_uint(eh);
  unsigned int pm;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(pm) : "r"(s.pm + 4u * j));
  if (eb > pm) return true;
  unsigned long long pr;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(pr) : "r"(s.bp + 8u * j));
  if (eb > (unsigned int)(pr >> 32)) {
    const CandRec *c = (const CandRec *)p.cand + (unsigned int)pr;
    return (double)tlb >= __ldcg(&c->t);
  }
  return false;
}

// pm of the bucket of a float lower bound tlb (the staircase's prefix minimum
// over strictly lower buckets): pm is non-increasing in the bucket, so every
// T >= tlb has pm[bucket(T)] <= this value
__device__ __forceinline__ unsigned int stair_pm_at(const StairSm &s, const DevParams &p, float tlb) {
  const int b = (int)((__float_as_uint(tlb) >> p.bkt_sh32) + p.bkt_off32);
  const uint32_t j = (uint32_t)(b < 0 ? 0 : (b >= kBuckets ? kBuckets - 1 : b));
  unsigned int pm;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(pm) : "r"(s.pm + 4u * j));
  return pm;
}

// bit s set: weight s has b = 0 (F = X^a depends on T alone) and the lane's
// best for it has T <= T64 and a lower index than idx: configurations with
// makespan >= T64 and index >= idx have F <= that best's F (rounding is
// monotone) and a higher index, so none of them can replace it
template <class WS>
__device__ __forceinline__ unsigned b0_beaten(const DevParams &p, const BestRec *lb, unsigned mask, double T64,
                                              u64 idx) {
  unsigned out = 0;
  if constexpr (WS::RT) {
    for (int s = 0; s < p.nw; s++)
      if ((mask >> s & 1u) && p.wb[s] == 0 && lb[s].valid && T64 >= lb[s].t && idx > lb[s].idx) out |= 1u << s;
  } else {
#pragma unroll
    for (int s = 0; s < WS::N; s++)
      if (WS::B(s) == 0 && (mask >> s & 1u) && lb[s].valid && T64 >= lb[s].t && idx > lb[s].idx)
        out |= 1u << s;
  }
  return out;
}

// does the (compile-time) weight set contain a b = 0 weight? (run-time sets: maybe)
template <class WS>
__host__ __device__ constexpr bool ws_has_b0() {
  if constexpr (WS::RT) {
    return WS::MAYB0;
  } else {
    for (int s = 0; s < WS::N; s++)
      if (WS::B(s) == 0) return true;
    return false;
  }
}

// mask of the weights with b = 0
template <class WS>
__device__ __forceinline__ unsigned b0_mask(const DevParams &p) {
  unsigned m = 0;
  if constexpr (WS::RT) {
    for (int s = 0; s < p.nw; s++)
      if (p.wb[s] == 0) m |= 1u << s;
  } else {
#pragma unroll
    for (int s = 0; s < WS::N; s++)
      if (WS::B(s) == 0) m |= 1u << s;
  }
  return m;
}

// any weight with b = 0 among mask
template <class WS>
__device__ __forceinline__ bool b0_any(const DevParams &p, unsigned mask) {
  if constexpr (WS::RT) {
    for (int s = 0; s < p.nw; s++)
      if ((mask >> s & 1u) && p.wb[s] == 0) return true;
    return false;
  } else {
    bool any = false;
#pragma unroll
    for (int s = 0; s < WS::N; s++) any |= WS::B(s) == 0 && (mask >> s & 1u);
    return any;
  }
}

// One configuration of the current partition (level digits dig[0..k-1],
// exact T64, fp32 T/E): per-weight screen against the lane's thresholds
// (thr: shared-memory copy), Pareto screen, fp64 refine, record.  Out of
// line (slow path).  Returns 1 if it issued a refine.
template <class WS>
__device__ __noinline__ int check_config(const Tables &tb, const DevParams &p, const Stair &stair,
                                         const WarpPart &wp, float *thr, BestRec *lb, u64 idx,
                                         const int *dig, float T, float E, double T64) {
  unsigned need = 0;
  if constexpr (WS::RT) {
    for (int s = 0; s < p.nw; s++) {
      const float q = rt_q(p, s, T, E);
      if (q <= fminf(thr[s], q) * p.mul[s]) need |= 1u << s;
      thr[s] = fminf(thr[s], q);
    }
  } else if constexpr (WS::N > 0) {
    float q[WS::N];
    WS::q(T, E, q);
#pragma unroll
    for (int s = 0; s < WS::N; s++) {
      if (q[s] <= fminf(thr[s], q[s]) * p.mul[p.ws_perm[s]]) need |= 1u << s;
      thr[s] = fminf(thr[s], q[s]);
    }
  }
  // weights with b = 0 (F = X^a, X = T_seq / T): exact early reject against
  // the lane's best (b0_beaten) -- stops the tie flood of (1,0), where every
  // configuration sharing the optimum's bottleneck group ties it
  need &= ~b0_beaten<WS>(p, lb, need, T64, idx);
  const bool par = p.want_pareto && !stair_dominated(stair, p, T64, E);
  if (!need && !par) return 0;
  // fp64 canonical re-score from the exact group tuples: T = max_g T_g (exact),
  // E = ((0 + E_0) + E_1) + ... in block order (the canonical order)
  const double T64r = T64;
  double E64 = 0.0;
  for (int b = 0; b < wp.cfg.k; b++) E64 = __dadd_rn(E64, wp.ge64[b * 4 + dig[b]]);
  if (p.model & SCHED_MODEL_COUNT_IDLE) E64 = __dadd_rn(__dmul_rn(p.gps, T64r), E64);  // R26 (records: D_g)
  if constexpr (WS::N > 0) {
#pragma unroll
    for (int s = 0; s < WS::N; s++) {
      if (need >> s & 1u) {
        const double F = WS::RT ? objective64(p, T64r, E64, p.wa[s], p.wb[s])
                                : objective64(p, T64r, E64, WS::A(s), WS::B(s));
        BestRec &b = lb[s];
        if (!b.valid || better(F, idx, b.f, b.idx)) {
          b.f = F;
          b.idx = idx;
          b.t = T64r;
          b.e = E64;
          b.t32 = T;
          b.e32 = E;
          b.valid = 1;
        }
      }
    }
  }
  if (par && !stair_dominated(stair, p, T64r, __double2float_rd(__ddiv_rd(E64, p.eseq))) &&
      !stair_dominated_exact(stair, p, T64r, E64))
    emit_candidate(p, stair, idx, T64r, E64, T, E);
  return 1;
}

// Per-configuration path for v in [v0, v1) of the current partition with
// stride `step` (lanes interleave with step 32, a single lane uses 1).
// thr is the lane's shared-memory threshold copy (updated here).
template <class WS>
__device__ __noinline__ int edge_configs(const Tables &tb, const DevParams &p, const Stair &stair,
                                         const WarpPart &wp, float *thr, BestRec *lb, uint32_t v0, uint32_t v1,
                                         int step) {
  const int k = wp.cfg.k;
  int nref = 0;
  for (uint32_t v = v0; v < v1; v += step) {
    int dig[kTileMaxG];
    float T = 0.f, E = 0.f;
    double T64 = 0.0;
    for (int b = 0; b < k; b++) {
      dig[b] = (int)(v >> (2 * (k - 1 - b))) & 3;
      T = fmaxf(T, wp.gt[b * 4 + dig[b]]);
      E += wp.ge[b * 4 + dig[b]];
      T64 = fmax(T64, wp.g64[b * 4 + dig[b]]);
    }
    E = e_total(p, T, E);
    dump_score<WS>(p, wp.base + v, T, E);
    if constexpr (WS::RT) {
      for (int s = 0; s < p.nw; s++) thr[s] = fminf(thr[s], rt_q(p, s, T, E));
    } else if constexpr (WS::N > 0) {
      float q[WS::N];
      WS::q(T, E, q);
#pragma unroll
      for (int s = 0; s < WS::N; s++) thr[s] = fminf(thr[s], q[s]);
    }
    nref += check_config<WS>(tb, p, stair, wp, thr, lb, wp.base + v, dig, T, E, T64);
  }
  return nref;
}

// Slow path of one 64-configuration tile (v = vt .. vt+63, k >= 5), with
// hierarchical exact Pareto corners (per a, then per (a, b)) before the
// per-configuration checks.
template <class WS>
__device__ __noinline__ int tile_slow(const Tables &tb, const DevParams &p, const Stair &stair,
                                      const WarpPart &wp, float *thr, BestRec *lb, uint32_t vt, float Tp,
                                      float Ep, bool arg_hit) {
  const int k = wp.cfg.k;
  int dig[kTileMaxG];
  double Tp64 = 0.0;
  for (int b = 0; b < k - 3; b++) {
    dig[b] = (int)(vt >> (2 * (k - 1 - b))) & 3;
    Tp64 = fmax(Tp64, wp.g64[b * 4 + dig[b]]);
  }
  const int ga = (k - 3) * 4, gb = (k - 2) * 4, gc = (k - 1) * 4;
  const double minC64 = fmin(fmin(wp.g64[gc], wp.g64[gc + 1]), fmin(wp.g64[gc + 2], wp.g64[gc + 3]));
  const double minB64 = fmin(fmin(wp.g64[gb], wp.g64[gb + 1]), fmin(wp.g64[gb + 2], wp.g64[gb + 3]));
  const float minCe = fminf(fminf(wp.ge[gc], wp.ge[gc + 1]), fminf(wp.ge[gc + 2], wp.ge[gc + 3]));
  const float minBe = fminf(fminf(wp.ge[gb], wp.ge[gb + 1]), fminf(wp.ge[gb + 2], wp.ge[gb + 3]));
  int nref = 0;
  const bool prune = !arg_hit && !(p.model & SCHED_MODEL_COUNT_IDLE);  // idle: corner E needs T (not tracked here)
  for (int a = 0; a < 4; a++) {
    const float T1 = fmaxf(Tp, wp.gt[ga + a]), E1 = Ep + wp.ge[ga + a];
    const double A64 = fmax(Tp64, wp.g64[ga + a]);
    if (prune && stair_dominated(stair, p, fmax(fmax(A64, minB64), minC64), (E1 + minBe) + minCe)) continue;
    for (int b = 0; b < 4; b++) {
      const float T2 = fmaxf(T1, wp.gt[gb + b]), E2 = E1 + wp.ge[gb + b];
      const double B64 = fmax(A64, wp.g64[gb + b]);
      if (prune && stair_dominated(stair, p, fmax(B64, minC64), E2 + minCe)) continue;
      for (int c = 0; c < 4; c++) {
        const float T = fmaxf(T2, wp.gt[gc + c]), E = e_total(p, T, E2 + wp.ge[gc + c]);
        const double T64 = fmax(B64, wp.g64[gc + c]);
        dig[k - 3] = a;
        dig[k - 2] = b;
        dig[k - 1] = c;
        nref += check_config<WS>(tb, p, stair, wp, thr, lb, wp.base + vt + a * 16 + b * 4 + c, dig, T, E, T64);
      }
    }
  }
  return nref;
}

// exact min fp64 makespan over a tile (its corner), k >= 5
static __device__ __noinline__ double tile_corner64(const WarpPart &wp, uint32_t vt) {
  const int k = wp.cfg.k;
  const int ga = (k - 3) * 4, gb = (k - 2) * 4, gc = (k - 1) * 4;
  double t = fmax(fmax(fmin(fmin(wp.g64[gb], wp.g64[gb + 1]), fmin(wp.g64[gb + 2], wp.g64[gb + 3])),
                       fmin(fmin(wp.g64[gc], wp.g64[gc + 1]), fmin(wp.g64[gc + 2], wp.g64[gc + 3]))),
                  fmin(fmin(wp.g64[ga], wp.g64[ga + 1]), fmin(wp.g64[ga + 2], wp.g64[ga + 3])));
  for (int b = 0; b < k - 3; b++) t = fmax(t, wp.g64[b * 4 + ((int)(vt >> (2 * (k - 1 - b))) & 3)]);
  return t;
}

// after the lane's shared-memory thresholds changed: refresh the register
// products (WS_RT screens from shared memory directly)
template <class WS>
__device__ __forceinline__ void thr_from_sm(const DevParams &p, Thr<WS> &thr, const float *thr_sm) {
  if constexpr (!WS::RT) {
#pragma unroll
    for (int s = 0; s < WS::N; s++) thr.vm[s] = thr_sm[s] * p.mul[p.ws_perm[s]];
  } else {  // log2 thresholds of the pre-screen (rt_screen), +inf while unset
#pragma unroll
    for (int s = 0; s < WS::N; s++)
      if (s < p.nw) thr.vm[s] = __log2f(thr_sm[s] * p.mul[s]) + p.lmargin[s];
  }
}

// run-time-weight corner screen: bit s set iff q_s(mT, mE) <= thr_s (1 + delta_s).
// A log-domain pre-screen (2 MUFU per tile, 2 FMA-pipe ops + 1 compare per
// weight, exponents from the constant bank) is passed by every weight that
// the exact test passes (lmargin, host_core.cpp); only those run the exact
// repeated-multiplication test.  Operands outside 2^+-32 skip the pre-screen.
template <class WS>
__device__ __forceinline__ unsigned rt_screen(const DevParams &p, const Thr<WS> &thr, const float *thr_sm, float mT,
                                              float mE) {
  const float lt = __log2f(mT), le = __log2f(mE);
  const bool inr = fabsf(lt) < 32.f && fabsf(le) < 32.f;
  unsigned pre = 0;
#pragma unroll
  for (int s = 0; s < WS::N; s++)
    if (s < p.nw && (!inr || fmaf(p.fa[s], lt, p.fb[s] * le) <= thr.vm[s])) pre |= 1u << s;
  unsigned hit = 0;
  if (pre) {
    for (int s = 0; s < p.nw; s++)
      if ((pre >> s & 1u) && rt_q(p, s, mT, mE) <= thr_sm[s] * p.mul[s]) hit |= 1u << s;
  }
  return hit;
}

// L = 2 or 3 searched levels, per configuration: configurations v of
// [v0, v1) with stride `step`, decoded into base-L level digits and scored
// from the partition's group records (T = max, E = block-order sum), screened
// (run-time weights: log-domain pre-screen; Pareto: fp32 staircase, then the
// exact fp64 makespan), survivors through check_config.  Used for partitions
// of fewer than 3 groups and for tiles straddling the unit's range.
template <int L, class WS>
__device__ __noinline__ int small_l_edge(const Tables &tb, const DevParams &p, const Stair &stair,
                                         const WarpPart &wp, float *thr_sm, BestRec *lb, uint32_t v0,
                                         uint32_t v1, uint32_t step) {
  const int k = wp.cfg.k;
  int nref = 0;
  for (uint32_t v = v0; v < v1; v += step) {
    int dig[kTileMaxG];
    uint32_t x = v;
    for (int b = k - 1; b >= 0; b--) {
      dig[b] = (int)(x % (uint32_t)L);
      x /= (uint32_t)L;
    }
    float T = 0.f, E = 0.f;
    double T64 = 0.0;
    for (int b = 0; b < k; b++) {
      T = fmaxf(T, wp.gt[b * 4 + dig[b]]);
      E += wp.ge[b * 4 + dig[b]];
      T64 = fmax(T64, wp.g64[b * 4 + dig[b]]);
    }
    E = e_total(p, T, E);
    nref += check_config<WS>(tb, p, stair, wp, thr_sm, lb, wp.base + v, dig, T, E, T64);
  }
  return nref;
}

// L = 2 or 3 searched levels: tiles of the last two groups (L^2
// configurations, their 2 x L records in registers); every lane takes a
// contiguous range of the other groups' digit strings ("outer" strings,
// odometer in base L), per string folds the outer groups into (T_p, E_p),
// scores the tile's configurations (T = max, E = add, min-reduced to the
// tile's exact lower corner like the L = 4 tile), screens the corner once and
// re-checks a tile that is not cleared configuration by configuration.
template <int L, class WS>
__device__ __forceinline__ int small_l_configs(const Tables &tb, const DevParams &p, const Stair &stair,
                                               const WarpPart &wp, Thr<WS> &thr, float *thr_sm, BestRec *lb,
                                               uint32_t v0, uint32_t v1, int lane) {
  const int k = wp.cfg.k;
  if (k < 3) {
    const int r = small_l_edge<L, WS>(tb, *p.gp, stair, wp, thr_sm, lb, v0 + lane, v1, 32);
    thr_from_sm<WS>(p, thr, thr_sm);
    return r;
  }
  constexpr uint32_t TL = (uint32_t)(L * L);
  const int nb = (k - 2) * 4, nc = (k - 1) * 4;
  float Bt[L], Be[L], Ct[L], Ce[L];
#pragma unroll
  for (int m = 0; m < L; m++) {
    Bt[m] = wp.gt[nb + m];
    Be[m] = wp.ge[nb + m];
    Ct[m] = wp.gt[nc + m];
    Ce[m] = wp.ge[nc + m];
  }
  double minBC64 = 0.0;
  {
    double mb = wp.g64[nb], mc = wp.g64[nc];
#pragma unroll
    for (int m = 1; m < L; m++) {
      mb = fmin(mb, wp.g64[nb + m]);
      mc = fmin(mc, wp.g64[nc + m]);
    }
    minBC64 = fmax(mb, mc);
  }
  // outer strings meeting [v0, v1), split into 32 contiguous lane ranges
  const uint32_t o_lo = v0 / TL, o_hi = (v1 + TL - 1) / TL;
  const uint32_t q = (o_hi - o_lo + 31) / 32;
  uint32_t o = o_lo + min((uint32_t)lane * q, o_hi - o_lo);
  const uint32_t oe = o_lo + min((uint32_t)(lane + 1) * q, o_hi - o_lo);
  int dig[kTileMaxG];
  {
    uint32_t x = o;
    for (int b = k - 3; b >= 0; b--) {
      dig[b] = (int)(x % (uint32_t)L);
      x /= (uint32_t)L;
    }
  }
  int nref = 0;
  for (; o < oe; o++) {
    float Tp = 0.f, Ep = 0.f;
    for (int b = 0; b < k - 2; b++) {
      Tp = fmaxf(Tp, wp.gt[b * 4 + dig[b]]);
      Ep += wp.ge[b * 4 + dig[b]];
    }
    const uint32_t vt = o * TL;
    if (vt < v0 || vt + TL > v1) {  // a tile straddling the unit's range
      nref += small_l_edge<L, WS>(tb, *p.gp, stair, wp, thr_sm, lb, vt > v0 ? vt : v0, vt + TL < v1 ? vt + TL : v1, 1);
      thr_from_sm<WS>(p, thr, thr_sm);
    } else {
      float mT = __int_as_float(0x7f800000), mE = mT;
#pragma unroll
      for (int b = 0; b < L; b++) {
        const float T1 = fmaxf(Tp, Bt[b]), E1 = Ep + Be[b];
#pragma unroll
        for (int c = 0; c < L; c++) {
          mT = fminf(mT, fmaxf(T1, Ct[c]));
          mE = fminf(mE, E1 + Ce[c]);
        }
      }
      mE = e_total(p, mT, mE);  // the exact corner's E (COUNT_IDLE: kidle T + D)
      unsigned hitm = 0;
      if constexpr (WS::RT) {
        hitm = rt_screen<WS>(p, thr, thr_sm, mT, mE);
      } else if constexpr (WS::N > 0) {
        float mq[WS::N];
        WS::q(mT, mE, mq);
#pragma unroll
        for (int s2 = 0; s2 < WS::N; s2++)
          if (mq[s2] <= thr.vm[s2]) hitm |= 1u << s2;
      }
      bool par = p.want_pareto && !stair_dominated_f(stair, p, __fmul_rd(mT, p.tlb_scale_f), mE);
      if (par && !hitm) {  // the tile's exact corner makespan
        double c = minBC64;
        for (int b = 0; b < k - 2; b++) c = fmax(c, wp.g64[b * 4 + dig[b]]);
        par = !stair_dominated(stair, p, c, mE);
      }
      if (hitm || par) {
        nref += small_l_edge<L, WS>(tb, *p.gp, stair, wp, thr_sm, lb, vt, vt + TL, 1);
        thr_from_sm<WS>(p, thr, thr_sm);
      }
    }
    for (int b = k - 3; b >= 0; b--) {  // next outer string
      if (++dig[b] < L) break;
      dig[b] = 0;
    }
  }
  return nref;
}

// All level vectors v in [v0, v1) of the current partition (L = 4).
// k >= 5: lane = (h, digit of group k-5, digit of group k-4); the warp loop
// runs over j = digit strings of groups 0..k-6, two per step (h selects);
// each lane scores the 64-configuration tile of groups k-3..k-1 in registers.
template <int L, class WS>
__device__ __forceinline__ int partition_configs(const Tables &tb, const DevParams &p, const Stair &stair,
                                                 const StairSm &ss, WarpPart &wp, Thr<WS> &thr, float *thr_sm,
                                                 BestRec *lb, uint32_t v0, uint32_t v1, int lane) {
  if constexpr (L != 4) return small_l_configs<L, WS>(tb, p, stair, wp, thr, thr_sm, lb, v0, v1, lane);
  const int k = wp.cfg.k;
  if (k < 5) {
    const int r = edge_configs<WS>(tb, *p.gp, stair, wp, thr_sm, lb, v0 + lane, v1, 32);
    thr_from_sm<WS>(p, thr, thr_sm);
    return r;
  }
  const int nloop = 1 << (2 * (k - 5));
  for (int j = lane; j < nloop; j += 32) {  // loop-prefix table
    float T = 0.f, E = 0.f;
    for (int b = 0; b < k - 5; b++) {
      const int d = (j >> (2 * (k - 6 - b))) & 3;
      T = fmaxf(T, wp.gt[b * 4 + d]);
      E += wp.ge[b * 4 + d];
    }
    wp.lp[j] = make_float2(T, E);
  }
  __syncwarp();
  const int l4 = lane & 15;
  const int ga = (k - 3) * 4, gb = (k - 2) * 4, gc = (k - 1) * 4;
  const float Tl = fmaxf(wp.gt[(k - 5) * 4 + (l4 >> 2)], wp.gt[(k - 4) * 4 + (l4 & 3)]);
  const float El = wp.ge[(k - 5) * 4 + (l4 >> 2)] + wp.ge[(k - 4) * 4 + (l4 & 3)];
  float At[4], Ae[4], Bt[4], Be[4], Ct[4], Ce[4];
#pragma unroll
  for (int m = 0; m < 4; m++) {
    At[m] = wp.gt[ga + m];
    Ae[m] = wp.ge[ga + m];
    Bt[m] = wp.gt[gb + m];
    Be[m] = wp.ge[gb + m];
    Ct[m] = wp.gt[gc + m];
    Ce[m] = wp.ge[gc + m];
  }
  // weights with b = 0 that no configuration of this partition can improve
  // for this lane: the partition's exact min makespan (max over groups of the
  // group's min over levels of the exact fp64 T_g) is >= the T of the lane's
  // best and every index is higher (b0_beaten) -- then the tie flood of such
  // weights (every configuration sharing the optimum's bottleneck group ties
  // it) never reaches the per-tile exact corner
  unsigned b0skip = 0;
  {
    const unsigned b0m = (p.b0mode & 1) ? b0_mask<WS>(p) : 0u;
    if (b0m) {
      double pc = 0.0;
      for (int b = 0; b < k; b++)
        pc = fmax(pc, fmin(fmin(wp.g64[b * 4], wp.g64[b * 4 + 1]), fmin(wp.g64[b * 4 + 2], wp.g64[b * 4 + 3])));
      b0skip = b0_beaten<WS>(p, lb, b0m, pc, wp.base + v0);
    }
  }
  const float minTin = WS::N > 0 ? 0.f
                                 : fmaxf(fmaxf(fminf(fminf(At[0], At[1]), fminf(At[2], At[3])),
                                               fminf(fminf(Bt[0], Bt[1]), fminf(Bt[2], Bt[3]))),
                                         fminf(fminf(Ct[0], Ct[1]), fminf(Ct[2], Ct[3])));
  int nref = 0;
  if constexpr (!ws_has_b0<WS>()) {
    // sets without b = 0 weights (the c4 bench set): the plain loop; its rare
    // paths are divergent calls (measured faster here than vote-guarded ones:
    // c4 slice 639 vs 700 ms).  Tile t (v = 64t .. 64t+63) belongs to lane
    // t mod 32 (t = 32 step + lane: loop string j = t >> 4, lane digits
    // t & 15 = l4).  The (at most two) tiles cut by the unit's range are
    // checked per configuration first; the loop then runs over the lane's
    // full tiles without bounds checks.
    const uint32_t tb0 = v0 >> 6, tb1 = (v1 - 1) >> 6;
    bool edge = false;
    if ((v0 & 63u) && (tb0 & 31u) == (uint32_t)lane) {
      nref += edge_configs<WS>(tb, *p.gp, stair, wp, thr_sm, lb, v0, min(v1, (tb0 + 1) << 6), 1);
      edge = true;
    }
    if ((v1 & 63u) && (tb1 & 31u) == (uint32_t)lane && !(tb1 == tb0 && (v0 & 63u))) {
      nref += edge_configs<WS>(tb, *p.gp, stair, wp, thr_sm, lb, max(v0, tb1 << 6), v1, 1);
      edge = true;
    }
    if (edge) thr_from_sm<WS>(p, thr, thr_sm);
    const uint32_t te = v1 >> 6;
    const uint32_t tf = (v0 + 63u) >> 6;
#ifndef SCHED_TILE_NO_PMP
    // a partition-wide staircase bound: every tile corner's T is at least
    // the partition's fp32 min makespan (max over groups of the group's min
    // over levels), so pm of that bucket bounds pm of every tile's bucket
    // from above: E above it is dominated without the per-tile bucket lookup
    unsigned int pmp = 0xffffffffu;
    if (WS::N > 0 && p.want_pareto) {  // (Pareto-only sets measured slower with it: 350 -> 358 ms)
      float tmin = 0.f;
      for (int b = 0; b < k; b++)
        tmin = fmaxf(tmin, fminf(fminf(wp.gt[b * 4], wp.gt[b * 4 + 1]), fminf(wp.gt[b * 4 + 2], wp.gt[b * 4 + 3])));
      pmp = stair_pm_at(ss, p, __fmul_rd(tmin, p.tlb_scale_f));
    }
#endif
    for (uint32_t t = tf + (((uint32_t)lane - tf) & 31u); t < te; t += 32) {
      const float2 lp = wp.lp[t >> 4];
      const float Tp = fmaxf(lp.x, Tl), Ep = lp.y + El;
      unsigned hitm = 0;
      float cE, cT;
      bool fdom = false;  // WS::RT: corner discarded by the fp32 staircase screen
      if constexpr (WS::N > 0) {
        // every configuration's (T, E), min-reduced over the tile: the tile's
        // exact lower corner.  q_w = T^a E^b is monotone in T and E, so the
        // corner's proxies bound every configuration's from below (a tile
        // whose corner misses every threshold holds no candidate); a tile that
        // is not cleared is re-checked configuration by configuration.
        float mT = __int_as_float(0x7f800000), mE = mT;
  #pragma unroll
        for (int a = 0; a < 4; a++) {
          const float T1 = fmaxf(Tp, At[a]), E1 = Ep + Ae[a];
  #pragma unroll
          for (int b = 0; b < 4; b++) {
            const float E2 = E1 + Be[b];
  #pragma unroll
            for (int c = 0; c < 4; c++) {
              const float T = fmax3f(T1, Bt[b], Ct[c]);  // one ALU slot per configuration
              const float E = E2 + Ce[c];
              mT = fminf(mT, T);
              mE = fminf(mE, E);
              dump_score<WS>(p, wp.base + (t << 6) + (uint32_t)(a * 16 + b * 4 + c), T, e_total(p, T, E));
            }
          }
        }
        // the exact corner's E: COUNT_IDLE adds kidle T as one FFMA; without
        // it kidle0 = 0 and fma(0, T, E) == E exactly (T finite: feasible partition)
        mE = fmaf(p.kidle0, mT, mE);
#if !defined(SCHED_TILE_NO_PMP) && !defined(SCHED_TILE_NO_PMSKIP)
        // every weight has b >= 1 here: a corner the partition-wide bound
        // clears is dominated with margin by a verified configuration, so
        // no configuration of the tile reaches or ties a weight's optimum
        // (section 5) either -- the whole tile is done with one compare
        if constexpr (!WS::RT) {
          if (__float_as_uint(mE) > pmp) continue;
        }
#endif
        if constexpr (WS::RT) {
          // run-time weights (every b >= 1 here): the fp32 staircase screen
          // first.  A corner it discards is dominated by a verified
          // configuration p with T_p <= T and E > E_p (1 + 4u) (the val_p
          // margin, section 5), so every configuration c of the tile has
          // F_w(c) < F_w(p) strictly, in fp64 too, for every weight with
          // b >= 1: the tile holds no optimum and no tie of one, and the
          // weight screen (log-domain pre-screen + exact test) is skipped.
#ifndef SCHED_TILE_NO_PMP
          fdom = p.want_pareto &&
                 (__float_as_uint(mE) > pmp || stair_dominated_fs(ss, p, __fmul_rd(mT, p.tlb_scale_f), mE));
#else
          fdom = p.want_pareto && stair_dominated_fs(ss, p, __fmul_rd(mT, p.tlb_scale_f), mE);
#endif
          if (!fdom) hitm = rt_screen<WS>(p, thr, thr_sm, mT, mE);
        } else {
          float mq[WS::N];
          WS::q(mT, mE, mq);
  #pragma unroll
          for (int s = 0; s < WS::N; s++)
            if (mq[s] <= thr.vm[s]) hitm |= 1u << s;
        }
        cE = mE;
        cT = mT;
      } else {  // Pareto only: per-configuration E, min-reduced
        cT = fmaxf(Tp, minTin);
        cE = __int_as_float(0x7f800000);
  #pragma unroll
        for (int a = 0; a < 4; a++) {
          const float E1 = Ep + Ae[a];
  #pragma unroll
          for (int b = 0; b < 4; b++) {
            const float E2 = E1 + Be[b];
  #pragma unroll
            for (int c = 0; c < 4; c++) cE = fminf(cE, E2 + Ce[c]);
          }
        }
        cE = fmaf(p.kidle0, cT, cE);
      }
      const bool hit = hitm != 0;
      bool par = false;
#ifndef SCHED_TILE_NO_PMP
      if (p.want_pareto && !(WS::RT ? fdom : ((WS::N > 0 && __float_as_uint(cE) > pmp) ||
                                              stair_dominated_fs(ss, p, __fmul_rd(cT, p.tlb_scale_f), cE))))
#else
      if (p.want_pareto && !(WS::RT ? fdom : stair_dominated_fs(ss, p, __fmul_rd(cT, p.tlb_scale_f), cE)))
#endif
        par = !stair_dominated(stair, p, tile_corner64(wp, t << 6), cE);
      if (hit || par) {
        nref += tile_slow<WS>(tb, *p.gp, stair, wp, thr_sm, lb, t << 6, Tp, Ep, hit);
        thr_from_sm<WS>(p, thr, thr_sm);
      }
    }
  } else {
    // Every rare path of the tile loop (unit-boundary tiles, exact corners,
    // slow re-checks) is entered warp-uniformly (a vote), so the common
    // iteration carries no convergence-barrier bookkeeping; lanes without work
    // in a rare path skip it inside.  Tiles as in the plain loop (tile t of
    // lane t mod 32); the steps run warp-uniformly over the full tiles.
    const uint32_t tb0 = v0 >> 6, tb1 = (v1 - 1) >> 6;
    const bool e0 = (v0 & 63u) && (tb0 & 31u) == (uint32_t)lane;
    const bool e1 = (v1 & 63u) && (tb1 & 31u) == (uint32_t)lane && !(tb1 == tb0 && (v0 & 63u));
    if (__any_sync(0xffffffffu, e0 || e1)) {  // partial tiles at a unit boundary
      if (e0) nref += edge_configs<WS>(tb, *p.gp, stair, wp, thr_sm, lb, v0, min(v1, (tb0 + 1) << 6), 1);
      if (e1) nref += edge_configs<WS>(tb, *p.gp, stair, wp, thr_sm, lb, max(v0, tb1 << 6), v1, 1);
      thr_from_sm<WS>(p, thr, thr_sm);
    }
    const uint32_t te = v1 >> 6;
    const uint32_t tf = (v0 + 63u) >> 6;
    unsigned int pmp = 0xffffffffu;  // the partition-wide staircase bound (see the plain loop;
    if (WS::N > 0 && !WS::RT && p.want_pareto) {  // run-time sets here measured slower: 858 -> 869 ms)
      float tmin = 0.f;
      for (int b = 0; b < k; b++)
        tmin = fmaxf(tmin, fminf(fminf(wp.gt[b * 4], wp.gt[b * 4 + 1]), fminf(wp.gt[b * 4 + 2], wp.gt[b * 4 + 3])));
      pmp = stair_pm_at(ss, p, __fmul_rd(tmin, p.tlb_scale_f));
    }
    for (uint32_t st = tf >> 5; (st << 5) < te; st++) {
      const uint32_t t = (st << 5) + (uint32_t)lane;
      const bool full = t >= tf && t < te;
      const float2 lp = wp.lp[full ? t >> 4 : 0u];
      const float Tp = fmaxf(lp.x, Tl), Ep = lp.y + El;
      unsigned hitm = 0;
      float cE, cT;
      if constexpr (WS::N > 0) {
        // every configuration's (T, E), min-reduced over the tile: the tile's
        // exact lower corner.  q_w = T^a E^b is monotone in T and E, so the
        // corner's proxies bound every configuration's from below (a tile
        // whose corner misses every threshold holds no candidate); a tile that
        // is not cleared is re-checked configuration by configuration.
        float mT = __int_as_float(0x7f800000), mE = mT;
  #pragma unroll
        for (int a = 0; a < 4; a++) {
          const float T1 = fmaxf(Tp, At[a]), E1 = Ep + Ae[a];
  #pragma unroll
          for (int b = 0; b < 4; b++) {
            const float E2 = E1 + Be[b];
  #pragma unroll
            for (int c = 0; c < 4; c++) {
              const float T = fmax3f(T1, Bt[b], Ct[c]), E = E2 + Ce[c];
              mT = fminf(mT, T);
              mE = fminf(mE, E);
            }
          }
        }
        mE = fmaf(p.kidle0, mT, mE);  // the exact corner's E (COUNT_IDLE: kidle T + D; else + 0)
        if constexpr (WS::RT) {
          hitm = rt_screen<WS>(p, thr, thr_sm, mT, mE);
        } else {
          float mq[WS::N];
          WS::q(mT, mE, mq);
  #pragma unroll
          for (int s = 0; s < WS::N; s++)
            if (mq[s] <= thr.vm[s]) hitm |= 1u << s;
        }
        cE = mE;
        cT = mT;
      } else {  // Pareto only: per-configuration E, min-reduced
        cT = fmaxf(Tp, minTin);
        cE = __int_as_float(0x7f800000);
  #pragma unroll
        for (int a = 0; a < 4; a++) {
          const float E1 = Ep + Ae[a];
  #pragma unroll
          for (int b = 0; b < 4; b++) {
            const float E2 = E1 + Be[b];
  #pragma unroll
            for (int c = 0; c < 4; c++) cE = fminf(cE, E2 + Ce[c]);
          }
        }
        cE = fmaf(p.kidle0, cT, cE);
      }
      hitm = full ? (hitm & ~b0skip) : 0u;
      // exact tile corner (fp64 min makespan) where a screen needs it: b = 0
      // weights (no configuration of the tile beats the lane's best) and the
      // Pareto screen when the fp32 staircase test cannot decide
      const bool b0c = (p.b0mode & 2) && hitm && b0_any<WS>(p, hitm);
      const bool fpar = full && p.want_pareto && !((WS::N > 0 && !WS::RT && __float_as_uint(cE) > pmp) ||
                                                    stair_dominated_fs(ss, p, __fmul_rd(cT, p.tlb_scale_f), cE));
      bool par = false;
      if (__any_sync(0xffffffffu, b0c || fpar)) {
        if (b0c || fpar) {
          const double c64 = tile_corner64(wp, t << 6);
          if (b0c) hitm &= ~b0_beaten<WS>(p, lb, hitm, c64, wp.base + (t << 6));
          if (fpar) par = !stair_dominated(stair, p, c64, cE);
        }
      }
      const bool hit = hitm != 0;
      const bool slow = hit || par;
      if (__any_sync(0xffffffffu, slow)) {
        if (slow) nref += tile_slow<WS>(tb, *p.gp, stair, wp, thr_sm, lb, t << 6, Tp, Ep, hit);
        thr_from_sm<WS>(p, thr, thr_sm);
      }
    }
  }
  __syncwarp();
  return nref;
}

template <int L, class WS>
__global__ void __launch_bounds__(kTileThreads, kTileMinBlocks) k_tile(const DevParams p) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned char *after = sm + ((p.blob_bytes + 15) & ~15u);
  Stair stair = stair_at(after);
  const StairSm ss = stair_sm(stair);
  WarpPart *wps = (WarpPart *)(after + kStairSmem);
  WarpPart &wp = wps[warp];
  BestRec *red = (BestRec *)(wps + kTileWarps);
  float *thr_sm = (float *)(red + kTileWarps * kMaxW) + threadIdx.x * (kMaxW + 1);  // odd row stride: no bank conflicts
  const GroupRec *gtab = (const GroupRec *)p.gtab;
  stair_init(stair);
  __syncthreads();

  Thr<WS> thr;
  BestRec lb[WS::N > 0 ? WS::N : 1];
#pragma unroll
  for (int s = 0; s < (WS::N > 0 ? WS::N : 1); s++) {
    thr_sm[s] = __int_as_float(0x7f800000);
    thr.vm[s] = __int_as_float(0x7f800000);
    best_init(lb[s]);
  }
  const int nws = WS::RT ? p.nw : WS::N;  // weights searched
  if (lane == 0) {
    wp.ncfg = 0;
    wp.nfeas = 0;
    wp.sver = 0;
  }
  __syncwarp();
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
    for (int w = 0; w < WS::N; w++) {
      if (w >= nws) break;
      thr_sm[w] = fminf(thr_sm[w], __uint_as_float(__ldcg(p.thr + p.ws_perm[w])));
    }
    thr_from_sm<WS>(p, thr, thr_sm);
    if (p.want_pareto) {
      u64 sv = wp.sver;
      stair_sync(stair, p, sv, __ldcg(p.ctr + kCtrStairVer));
      __syncwarp();
      if (lane == 0) wp.sver = sv;
    }
    if (lane == 0) {
      dev_unrank(tb, p, s, wp.cfg);
      wp.base = s - wp.cfg.v;
    }
    __syncwarp();
    u64 ver_pref = p.want_pareto ? __ldcg(p.ctr + kCtrStairVer) : 0;  // stair_sync broadcasts lane 0's
    for (;;) {
      if (p.want_pareto) {  // staircase refresh per partition (version prefetched one partition ahead)
        u64 sv = wp.sver;
        stair_sync(stair, p, sv, ver_pref);
        ver_pref = __ldcg(p.ctr + kCtrStairVer);  // consumed next partition: load latency off the path
        __syncwarp();
        if (lane == 0) wp.sver = sv;
      }
      const u64 base = wp.base;
      const uint32_t Pn = (uint32_t)wp.cfg.Pn;
      const int k = wp.cfg.k;
      const uint32_t v0 = s > base ? (uint32_t)(s - base) : 0u;
      const uint32_t v1 = e - base < (u64)Pn ? (uint32_t)(e - base) : Pn;
      // group tuples of the partition: table lookups (lane = (group, level))
      bool infeas = false;
      if (lane < k * L) {
        const int b = lane / L, mu = lane % L;
        const GroupRec r = gtab[(size_t)wp.cfg.mask[b] * L + mu];
        wp.gt[b * 4 + mu] = r.t32;
        wp.ge[b * 4 + mu] = r.e32;
        wp.g64[b * 4 + mu] = r.t64;
        wp.ge64[b * 4 + mu] = r.e64;
        infeas = r.t32 == __int_as_float(0x7f800000);
      }
      const bool feas = __ballot_sync(0xffffffffu, infeas) == 0u;
      if (lane == 0) {
        wp.ncfg += v1 - v0;
        if (feas) wp.nfeas += v1 - v0;
      }
      __syncwarp();
      if (feas) nref += partition_configs<L, WS>(tb, p, stair, ss, wp, thr, thr_sm, lb, v0, v1, lane);
      __syncwarp();
      if (base + Pn >= e) break;
      if (lane == 0) {
        wp.base = base + Pn;
        dev_successor(tb, p, wp.cfg);
        wp.cfg.Pn = tb.W[wp.cfg.st[p.n - 1]];
        wp.cfg.v = 0;
      }
      __syncwarp();
    }
#pragma unroll
    for (int w = 0; w < WS::N; w++) {
      if (w >= nws) break;
      float t = thr_sm[w];
#pragma unroll
      for (int o = 16; o; o >>= 1) t = fminf(t, __shfl_xor_sync(0xffffffffu, t, o));
      thr_sm[w] = t;
      if (lane == 0 && t < __uint_as_float(__ldcg(p.thr + p.ws_perm[w])))
        atomicMin(p.thr + p.ws_perm[w], __float_as_uint(t));
    }
  }
  // ---- reductions ----
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
  for (int w = 0; w < WS::N; w++) {
    if (w >= nws) break;
    warp_best(lb[w]);
    if (lane == 0) red[warp * kMaxW + w] = lb[w];
  }
  __syncthreads();
  if ((int)threadIdx.x < nws) {
    const int w = threadIdx.x;
    BestRec b = red[w];
    for (int k = 1; k < kTileWarps; k++) {
      const BestRec x = red[k * kMaxW + w];
      if (x.valid && (!b.valid || better(x.f, x.idx, b.f, b.idx))) b = x;
    }
    ((BestRec *)p.slots)[(size_t)blockIdx.x * p.nw + p.ws_perm[w]] = b;
  }
}

// ---- per-TU instantiation: tile_<ws>.cu defines TILE_WS and includes this ----
template <int L, class WS>
const void *tile_fn();

#define SCHED_TILE_INSTANTIATE(L, WS)          \
  template <>                                  \
  const void *tile_fn<L, WS>() {               \
    return (const void *)k_tile<L, WS>;        \
  }

}  // namespace sched
