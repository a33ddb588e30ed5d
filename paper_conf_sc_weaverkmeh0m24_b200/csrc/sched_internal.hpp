// sched_internal.hpp -- types shared by the host core (host_core.cpp), the
// C ABI (capi.cpp) and the kernels (search.cu).  Not part of the public ABI.
//
// Citations: PAPER.md = /root/reference/PAPER.md; R<n> = DESIGN.md readings.
#pragma once

#include <cstddef>
#include <cstdint>
#include <vector>

#include "sched.h"

namespace sched {

constexpr int kMaxN = SCHED_MAX_WORKFLOWS;      // 32
constexpr int kMaxG = SCHED_MAX_GPUS;           // 16
constexpr int kMaxL = SCHED_MAX_SEARCH_LEVELS;  // 8
constexpr int kMaxW = SCHED_MAX_WEIGHTS;        // 8
constexpr int kBuckets = 2048;                  // Pareto staircase buckets (per CTA)
constexpr int kBucketShift = 45;                // of the fp64 bits of T: 128 buckets per binade (default)
constexpr int kBucketShiftMin = 33;             // finest re-bucketing: 2^19 buckets per binade (>= 29: fp32 screen)
constexpr uint16_t kNoState = 0xFFFF;
constexpr int kUnitLog2 = 11;
constexpr int kStairSmem = 20 * kBuckets;       // per-CTA staircase: bp, pe (u64) + pm (u32) per bucket
constexpr int kLog = 4096;                      // staircase insertion log (ring buffer entries)                   // generic kernel: 2048 configs per warp unit

// Validated host copy of sched_profile.
struct Profile {
  int n = 0, lp = 0;
  std::vector<int> pct;
  std::vector<float> t, p, u, bw, d;  // [n][lp], d: [n][lp][n][lp]
  std::vector<int> mem;
  int mem_cap = 0;
  float ps = 0.f;
  int l100 = -1;
  // > 0: sequential baselines fixed by the caller instead of computed from
  // this profile (the unsplit queue of a split search, R29)
  double tseq_base = 0.0, eseq_base = 0.0;
};

// Validated query (levels resolved to profile level indices).
struct Query {
  int n, g, c, L, scope, nw;
  int lev[kMaxL];           // profile level index of searched digit d
  int wa[kMaxW], wb[kMaxW];
  uint64_t lo, hi;          // resolved window (hi <= |Omega|)
  int rank, count, chunk_log2;
  int want_pareto;
  uint32_t cand_cap;
  uint32_t model;           // SCHED_MODEL_* bits
  float pcap;               // P_cap (W) for SCHED_MODEL_POWER_CAP
};

// DP count table (host + device): state = (elements placed, open groups,
// histogram of non-full group sizes); W[s] = #(RGS completions x level
// vectors) below s.  trans[s*tc + col]: col 0 = open a new group, col z =
// join a group of size z (capped) / col 1 = join any group (uncapped).
struct Space {
  int n = 0, g = 0, c = 0, L = 0, scope = 0;
  bool capped = false;
  int tc = 0;
  std::vector<uint64_t> W;
  std::vector<uint16_t> trans;
  int root = 0;
  uint64_t total = 0;
};

// Device-side parameter block (kernel argument, by value).
struct DevParams {
  // problem
  int n, g, c, L, scope, nw, capped, tc, R, ds;  // R = n*L rows, ds = d row stride
  int wa[kMaxW], wb[kMaxW];
  float delta[kMaxW];       // fp32 screen margin per weight
  float gamma;              // Pareto "surely dominated" margin
  int ws_perm[kMaxW];       // tile kernel: compile-time weight slot -> query weight index
  float mul[kMaxW];         // 1 + delta[w]
  float fa[kMaxW], fb[kMaxW];  // the exponents as floats (run-time-weight tile screen, log domain)
  float lmargin[kMaxW];     // its conservative margin in log2 units (host_core.cpp)
  double tlb_scale;         // T_seq / (1 + 2 eps_T) rounded down: T64 >= T32hat * tlb_scale
  float tlb_scale_f;        // the same, as a float rounded down
  float phat;               // P_s * T_seq / E_seq
  double ps, tseq, eseq;
  uint32_t model;           // SCHED_MODEL_* bits (R26-R28)
  double capd;              // P_cap - P_s (exact) for POWER_CAP
  float kcap;               // E_seq / ((P_cap - P_s) T_seq): normalised capped time = D-hat * kcap
  float kidle;              // g P_s T_seq / E_seq: COUNT_IDLE energy term per normalised T
  float kidle0;             // kidle under COUNT_IDLE, else 0 (tile loop: E + kidle0 T as one FFMA)
  double gps;               // g * P_s (exact) for COUNT_IDLE
  int mem_cap, want_pareto, root, nstates;
  int c2_seed_tiles;        // k_ctile2 seed pass: whole tiles sampled around each unit's position
  int abort_ovf;            // the fast kernels stop taking units once the candidate buffer overflowed
  int wb_pos;               // every weight has b >= 1 (corner screens: staircase domination implies no weight hit)
  uint32_t bucket_base;     // (bits64(T_lower) >> bucket_shift)
  int bucket_shift;         // kBucketShift, or finer after the seed pass (re-bucketing, search.cu)
  // the same buckets from the bits of a float T (stair_dominated_f):
  // bucket = (bits32(T) >> bkt_sh32) + bkt_off32 (mod 2^32); set_buckets() keeps them in step
  int bkt_sh32;
  uint32_t bkt_off32;
  // work split
  uint64_t lo, hi;          // window
  uint64_t first_chunk;     // first owned chunk id
  uint64_t n_owned;         // owned chunks intersecting [lo, hi)
  int shard_count, chunk_log2, unit_log2;
  int lane_strided;         // generic kernel: lanes interleave indices (1) or take contiguous runs (0)
  uint64_t n_units;
  uint64_t unit_stride;      // unit u covers global unit u * unit_stride (seed pass samples)
  // staged blob offsets (bytes from blob start) and size
  uint32_t off_th, off_u, off_bw, off_dh, off_traw, off_praw, off_mem, off_d, off_W, off_trans;
  uint32_t blob_bytes;
  // workspace pointers
  const unsigned char *blob;   // staged tables (device)
  unsigned long long *ctr;     // counters (see kCtr*)
  unsigned int *thr;           // [kMaxW] global fp32 proxy threshold bits (min)
  unsigned int *stv;           // [kBuckets] min val of verified points per bucket
  unsigned long long *stp;     // [kBuckets] min (val << 32 | candidate slot) per bucket
  unsigned long long *ste;     // [kBuckets] min exact E (fp64 bits) of the verified points per bucket
  unsigned char *stlog;        // [kLog] LogEnt: insertion log (seq = ctr[kCtrStairVer])
  unsigned char *slots;        // [grid][W] BestRec
  unsigned char *cand;         // [cand_cap] CandRec
  uint32_t cand_cap;
  unsigned char *out;          // finalize output area
  const unsigned char *gtab;   // [2^n][L] GroupRec: fp32/fp64 group tuples (nullptr: compute)
  int gtab_ok;                 // workspace holds a group table for this query
  int b0mode;                  // tile kernel, weights with b = 0: bit 0 partition-level, bit 1 tile-level
                               // early reject (default 3; SCHED_B0 overrides, measurement only)
  unsigned char *dump;         // sched_debug_scores32: float2 (T-hat, E-hat) per configuration of
  uint64_t dump_lo, dump_n;    // [dump_lo, dump_lo + dump_n) (nullptr: no dump)
  double *c2t64;               // k_ctile2: per-warp exact fp64 T_g table (global, [grid][warps][tab])
  const DevParams *gp;         // this block's copy in the workspace (global memory): handed to the
                               // out-of-line slow paths, so no thread copies the kernel parameters
                               // to its stack (local memory)
};
// bucket_shift / bucket_base and their float-bits form (bits64(x) >> s ==
// (bits32(x) >> (s - 29)) + (896 << (52 - s)) for a float x, s >= 29)
inline void set_buckets(DevParams &dp, int shift, uint32_t base) {
  dp.bucket_shift = shift;
  dp.bucket_base = base;
  dp.bkt_sh32 = shift - 29;
  dp.bkt_off32 = (896u << (52 - shift)) - base;
}


enum {
  kCtrUnit = 0,      // next work unit
  kCtrCand = 1,      // candidates appended
  kCtrConfigs = 2,   // configs scored
  kCtrFeasible = 3,  // feasible configs
  kCtrRefined = 4,   // fp64 refines
  kCtrOverflow = 5,  // candidate overflow flag
  kCtrSurv = 6,      // finalize: Pareto survivors
  kCtrFront = 7,     // finalize: front size
  kCtrStairVer = 8,  // staircase version (bumped per insertion)
  kCtrPass = 9,      // search passes run
  kCtrN = 16
};

struct BestRec {      // 48 B
  double f, t, e;
  unsigned long long idx;
  float t32, e32;     // normalised fp32 T/T_seq, E/E_seq of the hot loop
  int valid, pad;
};

struct GroupRec {     // 24 B: one (group mask, level) tuple; t32 = +inf marks memory-infeasible
  float t32, e32;     // normalised fp32 T_g / T_seq, E_g / E_seq of the hot loop
  double t64;         // exact canonical fp64 T_g
  double e64;         // exact canonical fp64 E_g = P_s T_g + D_g
};

struct LogEnt {       // 16 B staircase insertion: bucket, (val << 32 | slot or 0xffffffff), tag = seq + 1
  unsigned long long pr;
  unsigned int jb, tag;
};

struct CandRec {      // 32 B
  unsigned long long idx;
  double t, e;
  float t32, e32;
};

// ---- host core (host_core.cpp) ----
int validate_profile(const sched_profile *in, Profile *out);
int resolve_query(const Profile *P, const sched_query *q, Query *out, uint64_t *total);
int resolve_query_shape(const sched_query *q, int n_profile_levels, Query *out);
int build_space(const Query &q, Space *sp);
int host_unrank(const Space &sp, uint64_t idx, int8_t *a, int8_t *digits, int *k);
int host_rank(const Space &sp, const int8_t *a, const int8_t *digits, uint64_t *idx);
void host_constants(const Profile &P, const Query &q, double *tseq, double *eseq);
int host_score(const Profile &P, const Query &q, const int8_t *a, int k, const int8_t *digits,
               double *T, double *E);
double host_objective(double tseq, double eseq, double T, double E, int a, int b);
// scheduling-configuration split (R29): admissible
// split vectors in rank order, and the expanded client profile of one
int split_vectors(int n, const int32_t *tasks, const int32_t *max_split, std::vector<std::vector<int>> *out);
int expand_split(const Profile &P, int n, const int32_t *tasks, const std::vector<int> &split, Profile *out);
// staged table blob + DevParams (work split, bounds) for one query
int build_stage(const Profile &P, const Query &q, const Space &sp, std::vector<unsigned char> *blob,
                DevParams *dp);
int merge_picks(int n_ranks, int nw, const sched_pick *rank_best, const sched_pick *rank_pareto,
                const uint64_t *rank_np, sched_pick *best, sched_pick *pareto, uint64_t cap,
                uint64_t *np);

// ---- subset-DP front (dp_front.cu) ----
struct DpPoint {           // a front point with one witness configuration
  double t, e;             // exact canonical fp64 T, E
  int k;                   // groups
  int8_t group_of[kMaxN];  // RGS (block order)
  int8_t level_of[kMaxN];  // searched-level digit per workflow
};
int dp_front_workspace(const Profile &P, const Query &q, const DevParams &dp, size_t *bytes);
int dp_front_run(const Profile &P, const Query &q, DevParams p, const std::vector<unsigned char> &blob, void *d_ws,
                 size_t ws_bytes, void *stream, std::vector<DpPoint> *front, int *best_pos, float *ms,
                 int *launches);

// ---- device launchers (search.cu) ----
struct LaunchInfo {
  int path, grid, launches, passes;
  float search_ms;
  float main_ms;   // the final full pass's search kernel launch
  uint64_t d2h_bytes;
};
size_t workspace_bytes(const DevParams &dp, int max_grid);
int stage_tables(const DevParams &dp, const std::vector<unsigned char> &blob, void *d_ws, void *host_pinned,
                 void *stream);
int launch_unrank(DevParams dp, void *d_ws, size_t ws_bytes, void *stream, const uint64_t *d_idx, uint64_t n,
                  uint64_t advance, int8_t *gout, int8_t *lout);
int launch_search(DevParams dp, void *d_ws, size_t ws_bytes, void *stream, LaunchInfo *info,
                  std::vector<BestRec> *best, std::vector<CandRec> *pareto, uint64_t *ctr_out);

}  // namespace sched
