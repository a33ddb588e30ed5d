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
  static constexpr int N = 0;
  __host__ __device__ static constexpr int A(int s) { return 0; }
  __host__ __device__ static constexpr int B(int s) { return 0; }
  __device__ static __forceinline__ void q(float, float, float *) {}
};
struct WS_11 {
  static constexpr int N = 1;
  __host__ __device__ static constexpr int A(int s) { return 1; }
  __host__ __device__ static constexpr int B(int s) { return 1; }
  __device__ static __forceinline__ void q(float T, float E, float *o) { o[0] = E * T; }
};
struct WS_10 {
  static constexpr int N = 1;
  __host__ __device__ static constexpr int A(int s) { return 1; }
  __host__ __device__ static constexpr int B(int s) { return 0; }
  __device__ static __forceinline__ void q(float T, float, float *o) { o[0] = T; }
};
struct WS_01 {
  static constexpr int N = 1;
  __host__ __device__ static constexpr int A(int s) { return 0; }
  __host__ __device__ static constexpr int B(int s) { return 1; }
  __device__ static __forceinline__ void q(float, float E, float *o) { o[0] = E; }
};
struct WS_11_21 {  // c4: [T x E], [T x T x E]
  static constexpr int N = 2;
  __host__ __device__ static constexpr int A(int s) { return (s == 0 ? 1 : 2); }
  __host__ __device__ static constexpr int B(int s) { return (s == 0 ? 1 : 1); }
  __device__ static __forceinline__ void q(float T, float E, float *o) {
    o[0] = E * T;
    o[1] = o[0] * T;
  }
};
struct WS_C1 {  // (1,0) (0,1) (1,1) (2,1)
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


struct WarpPart {
  LaneCfg cfg;
  u64 base;
  float gt[kTileMaxG * kTileMaxL], ge[kTileMaxG * kTileMaxL];
  double g64[kTileMaxG * kTileMaxL];
};

// fp32 + exact fp64 makespan of group `m` with every member at level mu
__device__ __forceinline__ void group_eval(const Tables &tb, const DevParams &p, uint32_t m, int mu,
                                           float &t32, float &e32, double &t64) {
  const int L = p.L;
  float U = 0.f, B = 0.f, D = 0.f;
  double U64 = 0.0, B64 = 0.0;
  for (uint32_t mm = m; mm; mm &= mm - 1) {
    const int r = (__ffs(mm) - 1) * L + mu;
    U += tb.u[r];
    B += tb.bw[r];
    D += tb.dh[r];
    U64 = __dadd_rn(U64, (double)tb.u[r]);
    B64 = __dadd_rn(B64, (double)tb.bw[r]);
  }
  const float cg = fmaxf(fmaxf(1.f, U), B);
  double c = 1.0;
  if (U64 > c) c = U64;
  if (B64 > c) c = B64;
  float Tg = 0.f;
  double Tg64 = 0.0;
  for (uint32_t mm = m; mm; mm &= mm - 1) {
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
  t32 = Tg;
  e32 = p.phat * Tg + D;
  t64 = Tg64;
}

template <class WS>
struct LaneAcc {
  float thr[WS::N > 0 ? WS::N : 1];
  BestRec lb[WS::N > 0 ? WS::N : 1];
  u64 nref;
};

// One configuration (digits dig[0..K-1], exact T64 and fp32 T/E): per-weight
// screen, Pareto screen, fp64 refine, record.  Slow path.
template <int L, class WS, int K>
__device__ __noinline__ void check_config(const Tables &tb, const DevParams &p, const Stair &stair,
                                             const WarpPart &wp, LaneAcc<WS> &acc, u64 idx,
                                             const int *dig, float T, float E, double T64) {
  unsigned need = 0;
  if constexpr (WS::N > 0) {
    float q[WS::N];
    WS::q(T, E, q);
#pragma unroll
    for (int s = 0; s < WS::N; s++) {
      acc.thr[s] = fminf(acc.thr[s], q[s]);
      if (q[s] <= acc.thr[s] * (1.f + p.delta[p.ws_perm[s]])) need |= 1u << s;
    }
  }
  const bool par = p.want_pareto && !stair_dominated(stair, p, T64, E);
  if (!need && !par) return;
  acc.nref++;
  int lam[kMaxN];
  for (int i = 0; i < p.n; i++) lam[i] = dig[wp.cfg.a[i]];
  double T64r, E64;
  refine64(tb, p, wp.cfg.mask, K, lam, &T64r, &E64);
  if constexpr (WS::N > 0) {
#pragma unroll
    for (int s = 0; s < WS::N; s++) {
      if (need >> s & 1u) {
        const double F = objective64(p, T64r, E64, WS::A(s), WS::B(s));
        BestRec &b = acc.lb[s];
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
  if (par && !stair_dominated(stair, p, T64r, __double2float_rd(__ddiv_rd(E64, p.eseq))))
    emit_candidate(p, stair, idx, T64r, E64, T, E);
}

// per-config path for v in [v0, v1) of the current partition, strided by lanes
template <int L, class WS, int K>
__device__ __forceinline__ void edge_configs(const Tables &tb, const DevParams &p, const Stair &stair,
                                             const WarpPart &wp, LaneAcc<WS> &acc, u64 v0, u64 v1, int lane) {
  for (u64 v = v0 + lane; v < v1; v += 32) {
    int dig[K];
    u64 x = v;
#pragma unroll
    for (int b = K - 1; b >= 0; b--) {
      dig[b] = (int)(x % L);
      x /= L;
    }
    float T = 0.f, E = 0.f;
    double T64 = 0.0;
#pragma unroll
    for (int b = 0; b < K; b++) {
      T = fmaxf(T, wp.gt[b * L + dig[b]]);
      E += wp.ge[b * L + dig[b]];
      T64 = fmax(T64, wp.g64[b * L + dig[b]]);
    }
    check_config<L, WS, K>(tb, p, stair, wp, acc, wp.base + v, dig, T, E, T64);
  }
}

// Full tiles [t0, t1) of this lane (tile t = level digits of groups 0..K-3).
template <int L, class WS, int K>
__device__ __forceinline__ void lane_tiles(const Tables &tb, const DevParams &p, const Stair &stair,
                                           const WarpPart &wp, LaneAcc<WS> &acc, u64 t0, u64 t1) {
  constexpr int KP = K - 2;  // prefix groups
  constexpr int L2 = L * L;
  float At[L], Ae[L], Bt[L], Be[L];
  double A64[L], B64[L];
#pragma unroll
  for (int m = 0; m < L; m++) {
    At[m] = wp.gt[(K - 2) * L + m];
    Ae[m] = wp.ge[(K - 2) * L + m];
    A64[m] = wp.g64[(K - 2) * L + m];
    Bt[m] = wp.gt[(K - 1) * L + m];
    Be[m] = wp.ge[(K - 1) * L + m];
    B64[m] = wp.g64[(K - 1) * L + m];
  }
  float minAe = Ae[0], minBe = Be[0];
  double minA64 = A64[0], minB64 = B64[0];
#pragma unroll
  for (int m = 1; m < L; m++) {
    minAe = fminf(minAe, Ae[m]);
    minBe = fminf(minBe, Be[m]);
    minA64 = fmin(minA64, A64[m]);
    minB64 = fmin(minB64, B64[m]);
  }
  // odometer over the prefix digits
  int dg[KP > 0 ? KP : 1];
  float PT[KP > 0 ? KP : 1], PE[KP > 0 ? KP : 1];
  double P64[KP > 0 ? KP : 1];
  {
    u64 x = t0;
#pragma unroll
    for (int j = KP - 1; j >= 0; j--) {
      dg[j] = (int)(x % L);
      x /= L;
    }
#pragma unroll
    for (int j = 0; j < KP; j++) {
      const float pt = j ? PT[j - 1] : 0.f, pe = j ? PE[j - 1] : 0.f;
      const double p64 = j ? P64[j - 1] : 0.0;
      PT[j] = fmaxf(pt, wp.gt[j * L + dg[j]]);
      PE[j] = pe + wp.ge[j * L + dg[j]];
      P64[j] = fmax(p64, wp.g64[j * L + dg[j]]);
    }
  }
  for (u64 t = t0; t < t1; t++) {
    const float Tp = KP ? PT[KP - 1] : 0.f, Ep = KP ? PE[KP - 1] : 0.f;
    const double Tp64 = KP ? P64[KP - 1] : 0.0;
    // ---- score the L^2 configurations of the tile ----
    bool hit = false;
    if constexpr (WS::N > 0) {
      float mq[WS::N];
#pragma unroll
      for (int s = 0; s < WS::N; s++) mq[s] = __int_as_float(0x7f800000);
#pragma unroll
      for (int mu = 0; mu < L; mu++) {
        const float T1 = fmaxf(Tp, At[mu]), E1 = Ep + Ae[mu];
#pragma unroll
        for (int nu = 0; nu < L; nu++) {
          const float T = fmaxf(T1, Bt[nu]), E = E1 + Be[nu];
          float q[WS::N];
          WS::q(T, E, q);
#pragma unroll
          for (int s = 0; s < WS::N; s++) mq[s] = fminf(mq[s], q[s]);
        }
      }
#pragma unroll
      for (int s = 0; s < WS::N; s++) {
        acc.thr[s] = fminf(acc.thr[s], mq[s]);
        hit |= mq[s] <= acc.thr[s] * (1.f + p.delta[p.ws_perm[s]]);
      }
    }
    float cE;
    if constexpr (WS::N == 0) {  // Pareto only: per-configuration E, min-reduced
      cE = __int_as_float(0x7f800000);
#pragma unroll
      for (int mu = 0; mu < L; mu++) {
        const float E1 = Ep + Ae[mu];
#pragma unroll
        for (int nu = 0; nu < L; nu++) cE = fminf(cE, E1 + Be[nu]);
      }
    } else {
      cE = (Ep + minAe) + minBe;  // = min over the tile of the fp32 E above
    }
    if (!hit && p.want_pareto) {
      const double cT64 = fmax(fmax(Tp64, minA64), minB64);  // exact min T64 over the tile
      hit = !stair_dominated(stair, p, cT64, cE);
    }
    if (hit) {  // slow path: configuration by configuration
      int dig[K];
#pragma unroll
      for (int j = 0; j < KP; j++) dig[j] = dg[j];
#pragma unroll
      for (int mu = 0; mu < L; mu++) {
#pragma unroll
        for (int nu = 0; nu < L; nu++) {
          dig[K - 2] = mu;
          dig[K - 1] = nu;
          const float T = fmaxf(fmaxf(Tp, At[mu]), Bt[nu]), E = (Ep + Ae[mu]) + Be[nu];
          const double T64 = fmax(fmax(Tp64, A64[mu]), B64[nu]);
          check_config<L, WS, K>(tb, p, stair, wp, acc, wp.base + t * L2 + mu * L + nu, dig, T, E, T64);
        }
      }
    }
    // ---- advance the odometer ----
    if constexpr (KP > 0) {
      int j = KP - 1;
      while (j >= 0 && ++dg[j] == L) {
        dg[j] = 0;
        j--;
      }
      if (j < 0) j = 0;
#pragma unroll
      for (int jj = 0; jj < KP; jj++) {
        if (jj >= j) {
          const float pt = jj ? PT[jj - 1] : 0.f, pe = jj ? PE[jj - 1] : 0.f;
          const double p64 = jj ? P64[jj - 1] : 0.0;
          PT[jj] = fmaxf(pt, wp.gt[jj * L + dg[jj]]);
          PE[jj] = pe + wp.ge[jj * L + dg[jj]];
          P64[jj] = fmax(p64, wp.g64[jj * L + dg[jj]]);
        }
      }
    }
  }
}

template <int L, class WS, int K>
__device__ __forceinline__ void partition_configs(const Tables &tb, const DevParams &p, const Stair &stair,
                                                  const WarpPart &wp, LaneAcc<WS> &acc, u64 v0, u64 v1,
                                                  int lane) {
  constexpr u64 L2 = (u64)L * L;
  if constexpr (K == 1) {
    edge_configs<L, WS, K>(tb, p, stair, wp, acc, v0, v1, lane);
  } else {
    const u64 ta = (v0 + L2 - 1) / L2, tb2 = v1 / L2;
    if (ta >= tb2) {
      edge_configs<L, WS, K>(tb, p, stair, wp, acc, v0, v1, lane);
      return;
    }
    edge_configs<L, WS, K>(tb, p, stair, wp, acc, v0, ta * L2, lane);
    edge_configs<L, WS, K>(tb, p, stair, wp, acc, tb2 * L2, v1, lane);
    const u64 nt = tb2 - ta, q = nt / 32, r = nt % 32;
    const u64 my0 = ta + lane * q + (lane < (int)r ? lane : r);
    const u64 my1 = my0 + q + (lane < (int)r ? 1 : 0);
    if (my0 < my1) lane_tiles<L, WS, K>(tb, p, stair, wp, acc, my0, my1);
  }
}


template <int L, class WS>
__global__ void __launch_bounds__(kTileThreads) k_tile(const DevParams p) {
  extern __shared__ __align__(16) unsigned char sm[];
  stage_blob(sm, p);
  const Tables tb = tables_at(sm, p);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  unsigned char *after = sm + ((p.blob_bytes + 15) & ~15u);
  Stair stair{(unsigned int *)(after + 8 * kBuckets), (unsigned long long *)after};
  WarpPart *wps = (WarpPart *)(after + 12 * kBuckets);
  WarpPart &wp = wps[warp];
  BestRec *red = (BestRec *)(wps + kTileWarps);
  stair_init(stair);
  __syncthreads();

  LaneAcc<WS> acc;
#pragma unroll
  for (int s = 0; s < (WS::N > 0 ? WS::N : 1); s++) {
    acc.thr[s] = __int_as_float(0x7f800000);
    best_init(acc.lb[s]);
  }
  acc.nref = 0;
  u64 ncfg = 0, nfeas = 0, stair_ver = 0;
  const int ul = p.unit_log2, cl = p.chunk_log2;

  for (;;) {
    u64 unit = 0;
    if (lane == 0) unit = atomicAdd(p.ctr + kCtrUnit, 1ull);
    unit = __shfl_sync(0xffffffffu, unit, 0);
    if (unit >= p.n_units) break;
    const u64 ch = p.first_chunk + (unit >> (cl - ul)) * (u64)p.shard_count;
    u64 s = (ch << cl) + ((unit & ((1ull << (cl - ul)) - 1)) << ul);
    u64 e = s + (1ull << ul);
    s = s > p.lo ? s : p.lo;
    e = e < p.hi ? e : p.hi;
    if (s >= e) continue;
#pragma unroll
    for (int w = 0; w < WS::N; w++) acc.thr[w] = fminf(acc.thr[w], __uint_as_float(__ldcg(p.thr + p.ws_perm[w])));
    if (p.want_pareto) {
      const u64 v = __ldcg(p.ctr + kCtrStairVer);
      if (v != stair_ver) {
        stair_ver = v;
        stair_merge(stair, p);
      }
    }
    if (lane == 0) {
      dev_unrank(tb, p, s, wp.cfg);
      wp.base = s - wp.cfg.v;
    }
    __syncwarp();
    for (;;) {
      const u64 base = wp.base, Pn = wp.cfg.Pn;
      const int k = wp.cfg.k;
      const u64 v0 = s > base ? s - base : 0, v1 = e - base < Pn ? e - base : Pn;
      const bool feas = wp.cfg.feasible;
      if (lane == 0) {
        ncfg += v1 - v0;
        if (feas) nfeas += v1 - v0;
      }
      if (feas) {
        if (lane < k * L) {
          const int b = lane / L, mu = lane % L;
          float t32, e32;
          double t64;
          group_eval(tb, p, wp.cfg.mask[b], mu, t32, e32, t64);
          wp.gt[b * L + mu] = t32;
          wp.ge[b * L + mu] = e32;
          wp.g64[b * L + mu] = t64;
        }
        __syncwarp();
        switch (k) {
          case 1: partition_configs<L, WS, 1>(tb, p, stair, wp, acc, v0, v1, lane); break;
          case 2: partition_configs<L, WS, 2>(tb, p, stair, wp, acc, v0, v1, lane); break;
          case 3: partition_configs<L, WS, 3>(tb, p, stair, wp, acc, v0, v1, lane); break;
          case 4: partition_configs<L, WS, 4>(tb, p, stair, wp, acc, v0, v1, lane); break;
          case 5: partition_configs<L, WS, 5>(tb, p, stair, wp, acc, v0, v1, lane); break;
          case 6: partition_configs<L, WS, 6>(tb, p, stair, wp, acc, v0, v1, lane); break;
          case 7: partition_configs<L, WS, 7>(tb, p, stair, wp, acc, v0, v1, lane); break;
          default: partition_configs<L, WS, 8>(tb, p, stair, wp, acc, v0, v1, lane); break;
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
    for (int w = 0; w < WS::N; w++) {
      float t = acc.thr[w];
#pragma unroll
      for (int o = 16; o; o >>= 1) t = fminf(t, __shfl_xor_sync(0xffffffffu, t, o));
      acc.thr[w] = t;
      if (lane == 0 && t < __uint_as_float(__ldcg(p.thr + p.ws_perm[w])))
        atomicMin(p.thr + p.ws_perm[w], __float_as_uint(t));
    }
  }
  // ---- reductions ----
  u64 nref = acc.nref;
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
    warp_best(acc.lb[w]);
    if (lane == 0) red[warp * kMaxW + w] = acc.lb[w];
  }
  __syncthreads();
  if (threadIdx.x < WS::N) {
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
