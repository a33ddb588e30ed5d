/*
 * sched.h -- C ABI of the B200 exhaustive co-scheduling configuration search.
 *
 * The hot path of the granularity- and interference-aware MPS scheduler of
 * Weaver et al., "Granularity- and Interference-Aware GPU Sharing with MPS"
 * (SC'24 workshops).  PAPER.md below is /root/reference/PAPER.md; R<n> are
 * the readings of the paper listed in DESIGN.md ("Readings of the paper").
 *
 * Problem statement (Sec. IV-B): "we select groups of queued
 * workflows to co-schedule on available GPUs based on (1) predicted
 * interference and (2) evaluation metric priority (i.e., optimize throughput
 * or energy)".  The library scores EVERY configuration -- a set partition of
 * the queued workflows 0..n-1 into k <= g MPS client groups (one group per
 * GPU, <= max_clients members) times an MPS active-thread
 * level per client (PER_CLIENT) or per GPU (PER_GPU) (granularity, PAPER.md
 * L75) -- for throughput X = T_seq/T and energy efficiency Y = E_seq/E
 * relative to sequential scheduling, and returns the best
 * configuration for each product metric X^a * Y^b and
 * the exact throughput/energy Pareto set.  The score is DESIGN.md
 * "Canonical score" (memory clause and SM/BW predicate of PAPER.md L87).
 *
 * Conventions
 *  - Every function returns an int status: SCHED_OK (0) or a negative
 *    SCHED_E_* code; sched_strerror() names it.  No C++ exception crosses
 *    the ABI.  Output arguments are written only on SCHED_OK unless stated.
 *  - Every input pointer is owned by the caller and may be freed as soon
 *    as the call returns (sched_create copies the profile).
 *  - A handle owns only host memory (and a small pinned staging buffer).
 *    ALL device memory is caller-provided (d_workspace), and so is the
 *    CUDA stream (cudaStream_t passed as void*; NULL = legacy default).
 *  - A handle is not thread-safe; distinct handles are independent.
 *  - Indices are uint64; the space must have |Omega| <= 2^63.
 *  - Index order (R4): restricted-growth strings (RGS) of the partition in
 *    lexicographic order; within a partition the level digits read as a
 *    base-L number, most significant digit = client 0 (PER_CLIENT) or
 *    group 0 (PER_GPU).  Ties between equal fp64 scores go to the lowest
 *    index (BASELINE.json north_star).
 */
#ifndef SCHED_H_
#define SCHED_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  SCHED_OK = 0,
  SCHED_E_INVALID = -1,     /* bad argument / profile / query */
  SCHED_E_TOO_LARGE = -2,   /* |Omega| > 2^63, or tables exceed device limits */
  SCHED_E_CUDA = -3,        /* a CUDA runtime call failed */
  SCHED_E_CAPACITY = -4,    /* output/candidate capacity too small; *n_pareto = required */
  SCHED_E_INFEASIBLE = -5,  /* no feasible configuration in the searched range
                               (outputs ARE written, with valid = 0) */
  SCHED_E_WORKSPACE = -6,   /* workspace too small or misaligned (256 B) */
  SCHED_E_NODEVICE = -7     /* no CUDA device: there is no CPU fallback */
};

enum { SCHED_PER_CLIENT = 0, SCHED_PER_GPU = 1 };

/* Scoring-model variants (sched_query.model_flags; readings
 * R26-R28, R30 in DESIGN.md).  0 = the canonical model.
 *  COUNT_IDLE       every one of the g GPUs draws the static power P_s for
 *                   the whole makespan: E = g*P_s*T + sum_g D_g, and the
 *                   sequential baseline E_seq = g*P_s*T_seq + sum_i dyn_i (R8 variant).
 *  NO_INTERFERENCE  the PAPER.md L87 interference predicate as a hard rule
 *                   (criterion 2, L90): a group whose combined SM or combined
 *                   memory-BW utilisation exceeds 100 % is infeasible.
 *  POWER_CAP        software power capping at power_cap_w (PAPER.md L162:
 *                   300 W on A100X): a group is throttled until its average
 *                   power is <= P_cap with its dynamic energy conserved,
 *                   T_g' = max(T_g, D_g / (P_cap - P_s)); solo tasks of the
 *                   sequential baseline likewise.
 *  TIME_SLICE       time slicing instead of MPS (the
 *                   default CUDA sharing, processes take turns on the whole
 *                   GPU; reading R30): no concurrent execution, so no
 *                   contention stretch and no co-run slowdown; the clients
 *                   of a group run one after another at their solo profile,
 *                   T_g = sum_i tau_i (members ascending), tau_i = t_i, or
 *                   under POWER_CAP tau_i = max(t_i, dyn_i/(P_cap - P_s))
 *                   (each slice throttled on its own, as the sequential
 *                   baseline); E_g = P_s*T_g + D_g.  Cannot be combined with
 *                   NO_INTERFERENCE (a concurrency rule): SCHED_E_INVALID.
 *                   Scored through the group table (tile / suffix / pair
 *                   kernels) or the generic kernel; the PER_CLIENT tile
 *                   kernel declines it and sched_front_dp rejects it. */
enum {
  SCHED_MODEL_COUNT_IDLE = 1,
  SCHED_MODEL_NO_INTERFERENCE = 2,
  SCHED_MODEL_POWER_CAP = 4,
  SCHED_MODEL_TIME_SLICE = 8
};

#define SCHED_MAX_WORKFLOWS 32
#define SCHED_MAX_GPUS 16
#define SCHED_MAX_PROFILE_LEVELS 32
#define SCHED_MAX_SEARCH_LEVELS 8
#define SCHED_MAX_WEIGHTS 8
#define SCHED_MAX_EXPONENT 8
#define SCHED_MAX_CLIENTS 48    /* MPS client limit */

/* Offline solo + co-run profile (SM, memory, memory-bandwidth
 * utilisation and average power per workflow task; Table II).
 * Row-major; [N][L] means element (i, l) at i*L + l. */
typedef struct {
  int32_t n_workflows;          /* N_max >= 1: queue order = index order */
  int32_t n_levels;             /* L_p >= 1: profile grid of MPS active-thread % */
  const int32_t *level_pct;     /* [L_p] strictly ascending in (0,100]; must contain 100 */
  const float *solo_time_s;     /* [N][L_p] > 0: solo wall time of the workflow at that level */
  const float *solo_power_w;    /* [N][L_p] >= static_power_w: average GPU power */
  const float *sm_util;         /* [N][L_p] >= 0: average SM utilisation, fraction of the GPU */
  const float *bw_util;         /* [N][L_p] >= 0: average memory-BW utilisation, fraction */
  const int32_t *max_mem_mib;   /* [N] >= 0: maximum memory of the task */
  const float *corun_slowdown;  /* [N][L_p][N][L_p] >= 0: additive slowdown of i at level l
                                   caused by co-runner j at level m; diagonal i == j ignored */
  int32_t mem_capacity_mib;     /* device memory capacity (e.g. 81920 for A100X 80 GB) */
  float static_power_w;         /* P_s > 0: static GPU power charged per busy second (R8, R9) */
} sched_profile;

/* One search request (queue, available GPUs, metric priority). */
typedef struct {
  int32_t n;                    /* search workflows [0, n), 1 <= n <= N_max */
  int32_t g;                    /* available GPUs, 1..SCHED_MAX_GPUS */
  int32_t max_clients;          /* C: MPS clients per GPU, 1..48; C >= n means uncapped */
  uint32_t level_mask;          /* bit l selects profile level l for the search (L = popcount,
                                   1..SCHED_MAX_SEARCH_LEVELS); digit d = d-th set bit */
  int32_t level_scope;          /* SCHED_PER_CLIENT | SCHED_PER_GPU */
  int32_t n_weights;            /* W, 0..SCHED_MAX_WEIGHTS */
  const int32_t *weights;       /* [W][2] integer exponents (a,b) of F = X^a * Y^b,
                                   0 <= a,b <= 8, a+b >= 1 */
  uint64_t index_lo, index_hi;  /* searched window [lo, hi); hi = UINT64_MAX means |Omega| */
  int32_t shard_rank;           /* this rank's share: chunks c with c % shard_count == rank */
  int32_t shard_count;          /* >= 1 (multi-GPU split, one process per GPU) */
  int32_t chunk_log2;           /* chunk = 2^chunk_log2 consecutive indices, 12..40 (0 = default 24) */
  int32_t want_pareto;          /* nonzero: also compute the (T, E) Pareto set */
  uint32_t candidate_cap;       /* device Pareto-candidate buffer records; 0 = 1<<20 */
  uint32_t model_flags;         /* SCHED_MODEL_* bits; 0 = canonical model */
  float power_cap_w;            /* P_cap > P_s for SCHED_MODEL_POWER_CAP (else ignored) */
} sched_query;

/* One configuration and its scores.  score64/x64/y64/makespan_s/energy_j are
 * the fp64 canonical values (bitwise those of the CPU oracle); score32/x32/
 * y32 are the fp32 hot-loop values of the same configuration. */
typedef struct {
  uint64_t index;
  double score64, x64, y64;     /* F = X^a Y^b, X = T_seq/T, Y = E_seq/E */
  double makespan_s, energy_j;  /* T, E of the configuration */
  float score32, x32, y32;
  int32_t valid;                /* 0: no feasible configuration found (pick is empty) */
} sched_pick;

typedef struct {
  uint64_t n_configs;           /* configurations scored by this call (range x shard) */
  uint64_t n_feasible;          /* of which memory-feasible */
  uint64_t n_refined;           /* fp64 re-scores issued by the fp32 screen */
  uint64_t n_candidates;        /* Pareto candidates emitted to the device buffer */
  double t_seq_s, e_seq_j;      /* sequential baselines */
  float search_ms;              /* device time of the search kernel(s) (CUDA events) */
  float total_ms;               /* device time of the whole call on the stream */
  int32_t kernel_path;          /* 0 generic, 1 PER_GPU tile, 2 L=1 pair, 3 L=1 suffix, 4 subset-DP front,
                                   5 PER_CLIENT tile */
  int32_t grid_ctas;            /* persistent CTAs launched by the search kernel */
  int32_t kernel_launches;      /* kernels this call launched (init, search pass(es), finalize) */
  int32_t passes;               /* search passes (2 = re-run after candidate overflow) */
  uint64_t h2d_bytes;           /* host->device bytes this call copied (staged tables) */
  uint64_t d2h_bytes;           /* device->host bytes this call copied (counters, picks) */
  float main_ms;                /* device time of the final full search pass's kernel launch alone
                                   (CUDA events; search_ms also holds the seed pass, group table,
                                   re-runs); sched_front_dp: its kernels */
} sched_stats;

/* One point of the exact front computed by sched_front_dp, with one witness
 * configuration (no index: the literal per-client spaces exceed 2^64). */
typedef struct {
  double makespan_s, energy_j;  /* exact canonical fp64 T, E (bitwise the oracle's) */
  double x64, y64;              /* X = T_seq/T, Y = E_seq/E */
  double score64;               /* best[w]: F_w = X^a Y^b; front points: X */
  int32_t n_groups;
  int8_t group_of[SCHED_MAX_WORKFLOWS];  /* witness: RGS (block order) */
  int8_t level_of[SCHED_MAX_WORKFLOWS];  /* witness: searched-level digit of each workflow */
  int32_t valid;
} sched_dp_point;

typedef struct sched_handle sched_handle;

/* Copy + validate the profile, precompute host-side derived tables.
 * Errors: SCHED_E_INVALID (null/invalid field, p < P_s, level grid without 100). */
int sched_create(const sched_profile *profile, sched_handle **out);
int sched_destroy(sched_handle *h);

/* Exact |Omega| of the query's full space (ignores index window and shard).
 * Host only (no device needed).  SCHED_E_TOO_LARGE if > 2^63. */
int sched_count(const sched_query *q, uint64_t *count);

/* Bytes of device workspace sched_search needs for this query. */
int sched_workspace_size(const sched_handle *h, const sched_query *q, size_t *bytes);

/* Upload the query's staged tables (profile rows at the searched levels,
 * DP count table) into d_workspace on `stream`.  Optional: sched_search
 * stages itself when the workspace does not already hold this query. */
int sched_stage(sched_handle *h, const sched_query *q, void *d_workspace, size_t ws_bytes,
                void *cuda_stream);

/* Exhaustive search of [index_lo, index_hi) restricted to this shard.
 * best[W]: best configuration per weight (max F; ties -> lowest index).
 * pareto[pareto_cap]: Pareto set of distinct (T,E) ordered by X descending,
 * one (lowest) index per point; *n_pareto = its size (if > pareto_cap the
 * call returns SCHED_E_CAPACITY and *n_pareto is the required size).
 * Synchronous w.r.t. its host outputs (synchronises `stream`).
 * stats may be NULL.  Errors: INVALID, TOO_LARGE, WORKSPACE, CUDA, CAPACITY,
 * INFEASIBLE (outputs written with valid = 0), NODEVICE. */
int sched_search(sched_handle *h, const sched_query *q, void *d_workspace, size_t ws_bytes,
                 void *cuda_stream, sched_pick *best, sched_pick *pareto, uint64_t pareto_cap,
                 uint64_t *n_pareto, sched_stats *stats);

/* Merge per-rank results of sharded searches (exact, deterministic,
 * independent of the rank count): rank_best is [n_ranks][n_weights];
 * rank_pareto is the concatenation of each rank's Pareto list, rank r
 * contributing rank_npareto[r] picks.  Host only.  Invalid picks are skipped. */
int sched_merge(int32_t n_ranks, int32_t n_weights, const sched_pick *rank_best,
                const sched_pick *rank_pareto, const uint64_t *rank_npareto,
                sched_pick *best, sched_pick *pareto, uint64_t pareto_cap, uint64_t *n_pareto);

/* index -> configuration: group_of[i] in 0..k-1 (RGS, group 0 holds
 * workflow 0) and level_of[i] = searched-level digit (0..L-1) of workflow i
 * (PER_GPU: the digit of its group).  Host only. */
int sched_unrank(const sched_query *q, uint64_t index, int8_t *group_of, int8_t *level_of);

/* configuration -> index (inverse of sched_unrank).  group_of must be an
 * RGS; PER_GPU requires equal level_of within a group.  Host only. */
int sched_rank(const sched_query *q, const int8_t *group_of, const int8_t *level_of,
               uint64_t *index);

/* Device unrank (SURVEY 8(a) H3/H4, 4.2 "device unrank == host unrank"):
 * for t in [0, n): configuration of index d_index[t] + advance, computed on
 * the device by the search kernels' own routines -- unrank of d_index[t]
 * through the DP count table staged in shared memory, then `advance` steps of
 * the successor walk (level digits, then the next RGS) -- written as
 * d_group_of[t*q->n + i] / d_level_of[t*q->n + i] (layout of sched_unrank).
 * Indices (after advance) >= |Omega| give d_group_of[t*q->n] = -1.
 * d_index, d_group_of, d_level_of are DEVICE pointers owned by the caller;
 * ws is the query's search workspace (sched_workspace_size); asynchronous on
 * `stream` (no host sync).  SCHED_E_INVALID on a bad query or null pointer. */
int sched_unrank_device(sched_handle *h, const sched_query *q, const uint64_t *d_index, uint64_t n,
                        uint64_t advance, int8_t *d_group_of, int8_t *d_level_of, void *ws,
                        size_t ws_bytes, void *stream);

/* Debug / verification entry (tests/test_gpu_scores32.py): runs the PER_GPU
 * tile kernel (the bench's path; query must be PER_GPU with 4 searched
 * levels, G <= 8) over the query's window [index_lo, index_hi) (at most 2^26
 * configurations) with the weight (1,1) and no Pareto set, and writes every
 * configuration's fp32 hot-loop score as the kernel computes it:
 * d_scores[2 (i - index_lo)] = T / T_seq and [2 (i - index_lo) + 1] =
 * E / E_seq (fp32, normalised by the sequential baselines).
 * Configurations of memory-infeasible partitions are not written (pre-fill).
 * d_scores is a DEVICE pointer owned by the caller; synchronous.
 * SCHED_E_INVALID if the query does not run on the tile kernel. */
int sched_debug_scores32(sched_handle *h, const sched_query *q, void *ws, size_t ws_bytes, void *stream,
                         float *d_scores);

/* fp64 canonical score of one configuration on the host, weight w (0..W-1;
 * with W == 0 score64 = X).  out->valid = 0 if memory-infeasible.  Host only. */
int sched_score(const sched_handle *h, const sched_query *q, uint64_t index, int32_t w,
                sched_pick *out);

/* Exact Pareto front and per-weight optimum of the WHOLE space of the query
 * by a subset dynamic program on the device (dp_front.cu):
 * for every feasible group the Pareto front of its (T_g, E_g) over its level
 * vectors, then the block-order DP over workflow subsets.  Reaches spaces
 * that cannot be enumerated, e.g. the literal per-client c4 (16 workflows,
 * 8 GPUs, 4 levels per client: 4.05e19 configurations).  Requires
 * 2 <= n <= 20, L^max_clients <= 2^32 (PER_CLIENT), no SCHED_MODEL_TIME_SLICE
 * (SCHED_MODEL_COUNT_IDLE: the DP adds up the dynamic energies and applies
 * the idle term G P_s T to the whole-set front);
 * the index window and shard fields must be the defaults (whole space, one
 * shard).  front[front_cap] is ordered by X descending (T ascending), one
 * witness configuration per distinct (T, E); best[W] is the max F_w over the
 * front (ties: the first in that order; not necessarily the lowest index).
 * Errors: INVALID, TOO_LARGE, WORKSPACE, CUDA, CAPACITY (an internal front
 * overflowed, or *n_front > front_cap), INFEASIBLE (empty front), NODEVICE. */
int sched_dp_workspace_size(const sched_handle *h, const sched_query *q, size_t *bytes);
int sched_front_dp(sched_handle *h, const sched_query *q, void *d_workspace, size_t ws_bytes,
                   void *cuda_stream, sched_dp_point *best, sched_dp_point *front, uint64_t front_cap,
                   uint64_t *n_front, sched_stats *stats);

/* The paper's rule-based co-scheduling heuristic (reading
 * R25 in DESIGN.md), for measuring its optimality gap against the exhaustive
 * search: (1) workflows in ascending solo SM utilisation (at 100 %), (2) a
 * GPU's combined SM utilisation kept <= 100 %, (3) combined max memory <=
 * capacity, (4) at most 2 clients per GPU if priority = throughput (0), at
 * most max_clients if priority = energy (1).  Each workflow goes to the
 * first open GPU satisfying (2)-(4), else a new GPU, else the open GPU with
 * the lowest utilisation satisfying (3)-(4).  All clients run at the
 * highest searched level.  Writes the configuration (canonical RGS,
 * group_of/level_of as sched_unrank), its index in the query's space, and
 * its fp64 score for weight w (out->valid = 0 if infeasible).  Host only.
 * SCHED_E_INFEASIBLE if the rules cannot place every workflow. */
int sched_heuristic(const sched_handle *h, const sched_query *q, int32_t priority, int32_t w,
                    int8_t *group_of, int8_t *level_of, uint64_t *index, sched_pick *out);

/* Scheduling-configuration search ("scheduling
 * configuration ... the number of sequential tasks in each workflow as well as
 * the number of concurrent workflows", L176 "split them into multiple parallel
 * workflows", Figs 4-5 "s-p" labels; reading R29 in DESIGN.md).
 * Workflow i of the query consists of tasks[i] >= 1 identical independent
 * tasks (its profile row is the whole workflow).  A split vector p runs it as
 * p_i concurrent MPS clients (p_i a divisor of tasks[i], p_i <= max_split[i]
 * if max_split != NULL) of tasks[i]/p_i tasks each.  Split vectors are ranked
 * lexicographically (divisors ascending, workflow 0 most significant).  For
 * every split the expanded queue (clients workflow-major; client time
 * fl32((t_i * s_i) / tasks[i]) at every level, the workflow's power, SM, BW
 * and memory; co-run slowdown between siblings = the profile's diagonal
 * block d[i,l][i,m]) is searched exhaustively on the device exactly as
 * sched_search does, against the SAME sequential baselines T_seq, E_seq of
 * the unsplit queue (q as given), so X and Y compare across splits.
 * best[W]: max F per weight over all splits (ties -> lowest split rank, then
 * lowest index in that split's space); pareto: the distinct (T, E) not
 * dominated by any configuration of any split, one witness each (lowest
 * (rank, index)), T ascending; *n_pareto as in sched_search (CAPACITY ->
 * required size).  The query must cover the whole space of one shard
 * (index window default, shard_count 1).  Every split must have <= 32
 * clients and |Omega| <= 2^63 (else SCHED_E_TOO_LARGE: bound max_split).
 * stats (may be NULL): sums over the splits; t_seq_s/e_seq_j = the unsplit
 * baselines.  Workspace: sched_split_workspace_size (the max over splits),
 * which also returns the number of split vectors. */
typedef struct {
  sched_pick pick;                     /* index in the expanded space of split `split_rank` */
  uint32_t split_rank;                 /* rank of the split vector */
  int32_t n_clients;                   /* sum of split[0..n) */
  int32_t split[SCHED_MAX_WORKFLOWS];  /* p_i: concurrent clients of workflow i */
} sched_split_pick;

int sched_split_workspace_size(const sched_handle *h, const sched_query *q, const int32_t *tasks,
                               const int32_t *max_split, size_t *bytes, uint32_t *n_splits);
int sched_search_splits(sched_handle *h, const sched_query *q, const int32_t *tasks,
                        const int32_t *max_split, void *d_workspace, size_t ws_bytes, void *cuda_stream,
                        sched_split_pick *best, sched_split_pick *pareto, uint64_t pareto_cap,
                        uint64_t *n_pareto, sched_stats *stats);

const char *sched_strerror(int status);

/* Library version string, e.g. "sched-b200 0.1 sm_100a". */
const char *sched_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SCHED_H_ */
