/*
 * oracle/enum.c -- O1: plain, slow, obviously-correct fp64 recursive enumerator.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load liboracle.so.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_sc_weaverkmeh0m24_b200/); neither side includes the other.
 *
 * Build: gcc -O2 -ffp-contract=off -fno-fast-math -shared -fPIC (x86-64 SSE2
 * doubles: every +, *, / below rounds exactly once, in the order written).
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md; readings R1..R24 are
 * listed in DESIGN.md, section "Readings of the paper"):
 *
 *  Space.  A configuration is a set partition of queued workflows 0..N-1 into
 *   k <= G unlabeled groups ("select groups of queued workflows to co-schedule
 *   on available GPUs") of size <= C (MPS clients, L35/L92),
 *   written as a restricted-growth string a[0..N-1] (a[0]=0,
 *   a[i] <= 1+max(a[0..i-1])), together with MPS active-thread levels
 *   (granularity): one per workflow (PER_CLIENT) or one per
 *   group (PER_GPU).  Index order (R4): RGS lexicographic, then the level
 *   digits in base L, most significant digit first (client 0 / group 0).
 *
 *  Score (R5-R11, canonical order):
 *   infeasible if some group has sum(max_mem) > M_cap
 *   U_g = sum u, B_g = sum bw (ascending), c_g = max(max(1,U_g),B_g) (L87)
 *   sigma_i = 1 + sum_{j in g, j != i, ascending} d[i][l_i][j][l_j]
 *   tau_i = (t_i * sigma_i) * c_g ;  T_g = max tau_i
 *   dyn_i = (p_i - P_s) * t_i ; D_g = sum dyn (ascending) ; E_g = P_s*T_g + D_g
 *   T = max_g T_g ; E = sum_g E_g (group order)
 *   X = T_seq / T ; Y = E_seq / E   (relative to sequential)
 *   F_w = ((1*X)*X...)*Y... (a factors X then b factors Y)
 *   T_seq: queue-order list schedule at 100% on G GPUs, lowest id on ties
 *   E_seq = sum_i p_i * t_i at 100%
 *
 *  Results: best index per weight (max F, ties -> lowest index) and the
 *  Pareto set of distinct (T,E) over feasible configurations, one (lowest)
 *  index per point.
 *
 *  Scoring-model variants (readings R26-R28, R30 in DESIGN.md),
 *  selected by or_query.model bits; 0 is the canonical model above:
 *   1 COUNT_IDLE: every one of the G GPUs draws P_s for the whole makespan
 *     (R8 variant).  With E_g = P_s*T_g + D_g this is
 *       E = (G*P_s)*T + D,  D = sum_g D_g (group order),
 *     and the sequential baseline likewise E_seq = (G*P_s)*T_seq + sum_i dyn_i.
 *   2 NO_INTERFERENCE: the PAPER.md L87 predicate as a hard rule ("two
 *     workflows are predicted to interfere if ... combined average SM
 *     utilization over 100%, combined average memory bandwidth utilization
 *     over 100%", criterion 2 "kept under 100%", L90): a group with
 *     U_g > 1 or B_g > 1 is infeasible.
 *   4 POWER_CAP: software power capping at P_cap (PAPER.md L162, 300 W on
 *     A100X): a group whose average power P_s + D_g/T_g exceeds P_cap is
 *     throttled until it does not, its dynamic energy conserved:
 *       T_g' = max(T_g, D_g / (P_cap - P_s)),  E_g = P_s*T_g' + D_g.
 *     A solo task in the sequential baseline likewise runs for
 *     t' = max(t, dyn / (P_cap - P_s)); its energy stays p*t when not capped,
 *     else P_s*t' + dyn.
 *   8 TIME_SLICE: time slicing instead of MPS (without
 *     MPS the clients of a GPU take turns on the whole device; reading R30):
 *     nothing runs concurrently, so there is no contention stretch c_g and
 *     no co-run slowdown; each member runs its own slice at its solo
 *     profile, one after another:
 *       T_g = sum_{i in g, ascending} tau_i,  tau_i = t_i,
 *     with POWER_CAP each slice is throttled on its own like a solo task of
 *     the sequential baseline: tau_i = max(t_i, dyn_i / (P_cap - P_s));
 *       E_g = P_s*T_g + D_g.
 *     (Not combined with NO_INTERFERENCE, a rule about concurrent clients.)
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
  int n, lp;               /* workflows in the profile, profile levels */
  const int *level_pct;    /* [lp] */
  const float *t, *p, *u, *bw;  /* [n][lp] */
  const int *mem;          /* [n] */
  const float *d;          /* [n][lp][n][lp] */
  int mem_cap;
  float ps;
} or_profile;

typedef struct {
  int n, g, c;             /* use workflows 0..n-1, G GPUs, C clients max */
  int L;                   /* searched levels */
  const int *lev;          /* [L] profile level index of each searched level */
  int scope;               /* 0 PER_CLIENT, 1 PER_GPU */
  int nw;
  const int *wa, *wb;      /* [nw] exponents */
  uint64_t lo, hi;         /* index window [lo, hi) */
  int want_pareto;
  unsigned model;          /* variant bits: 1 COUNT_IDLE, 2 NO_INTERFERENCE, 4 POWER_CAP, 8 TIME_SLICE */
  float power_cap;         /* P_cap (W) for POWER_CAP */
  double tseq_base, eseq_base;  /* > 0: sequential baselines given by the caller (the unsplit
                                   queue of a split search, R29); 0: computed below */
} or_query;

#define OR_COUNT_IDLE 1u
#define OR_NO_INTERFERENCE 2u
#define OR_POWER_CAP 4u
#define OR_TIME_SLICE 8u

typedef struct { uint64_t idx; double f, t, e; int found; } or_best;
typedef struct { uint64_t idx; double t, e; } or_point;

/* ------------------------------------------------------------------ counts */
/* count(r, b, hist): number of (RGS completions x level vectors) when r
 * elements remain, b groups are open, hist[s] = #groups of size s.  Plain
 * memoised recursion over the next element's choices. */
typedef unsigned __int128 u128;
#define KEYMAX 40
typedef struct { unsigned char key[KEYMAX]; int used; u128 val; } memo_ent;
static memo_ent *g_memo = 0;
static size_t g_memo_cap = 0;
static int g_n, g_g, g_c, g_L, g_scope;

static u128 ipow(u128 b, int e) { u128 r = 1; while (e-- > 0) r *= b; return r; }

static size_t hkey(const unsigned char *k) {
  size_t h = 1469598103934665603ull;
  for (int i = 0; i < KEYMAX; i++) { h ^= k[i]; h *= 1099511628211ull; }
  return h;
}

static u128 count_rec(int r, int b, int *hist) {
  if (r == 0) return g_scope == 0 ? ipow((u128)g_L, g_n) : ipow((u128)g_L, b);
  unsigned char key[KEYMAX];
  memset(key, 0, sizeof key);
  key[0] = (unsigned char)r; key[1] = (unsigned char)b;
  for (int s = 1; s <= g_c && s + 1 < KEYMAX; s++) key[s + 1] = (unsigned char)hist[s];
  size_t h = hkey(key) & (g_memo_cap - 1);
  while (g_memo[h].used) {
    if (!memcmp(g_memo[h].key, key, KEYMAX)) return g_memo[h].val;
    h = (h + 1) & (g_memo_cap - 1);
  }
  u128 tot = 0;
  for (int s = 1; s < g_c; s++) {           /* join one of hist[s] groups of size s */
    if (!hist[s]) continue;
    hist[s]--; hist[s + 1]++;
    tot += (u128)(hist[s] + 1) * count_rec(r - 1, b, hist);
    hist[s + 1]--; hist[s]++;
  }
  if (b < g_g) {                             /* open a new group */
    hist[1]++;
    tot += count_rec(r - 1, b + 1, hist);
    hist[1]--;
  }
  h = hkey(key) & (g_memo_cap - 1);
  while (g_memo[h].used) h = (h + 1) & (g_memo_cap - 1);
  memcpy(g_memo[h].key, key, KEYMAX); g_memo[h].used = 1; g_memo[h].val = tot;
  return tot;
}

static void count_setup(const or_query *q) {
  g_n = q->n; g_g = q->g; g_c = q->c < q->n ? q->c : q->n; g_L = q->L; g_scope = q->scope;
  if (!g_memo) { g_memo_cap = 1u << 18; g_memo = calloc(g_memo_cap, sizeof(memo_ent)); }
  else memset(g_memo, 0, g_memo_cap * sizeof(memo_ent));
}

/* subtree count given group sizes sz[0..b-1] after placing elements 0..i-1 */
static u128 subtree(int i, int b, const int *sz) {
  int hist[KEYMAX + 2];
  memset(hist, 0, sizeof hist);
  for (int j = 0; j < b; j++) hist[sz[j]]++;
  return count_rec(g_n - i, b, hist);
}

/* |Omega| as two u64 halves (lo, hi) so callers can detect > 2^64 */
void oracle_count(const or_query *q, uint64_t *lo, uint64_t *hi) {
  count_setup(q);
  int sz[64] = {0};
  sz[0] = 1;
  u128 v = q->n >= 1 ? subtree(1, 1, sz) : 0;
  *lo = (uint64_t)v; *hi = (uint64_t)(v >> 64);
}

/* -------------------------------------------------------------- constants */
void oracle_constants(const or_profile *P, const or_query *q, int l100,
                      double *tseq, double *eseq) {
  const double ps = (double)P->ps;
  const double capd = (double)q->power_cap - ps;   /* exact: two floats */
  double fin[64];
  for (int g = 0; g < q->g; g++) fin[g] = 0.0;
  for (int i = 0; i < q->n; i++) {          /* queue order, min finish, lowest id */
    double t = (double)P->t[i * P->lp + l100];
    if (q->model & OR_POWER_CAP) {
      double tc = (((double)P->p[i * P->lp + l100] - ps) * t) / capd;
      if (tc > t) t = tc;
    }
    int best = 0;
    for (int g = 1; g < q->g; g++) if (fin[g] < fin[best]) best = g;
    fin[best] = fin[best] + t;
  }
  double T = 0.0;
  for (int g = 0; g < q->g; g++) if (fin[g] > T) T = fin[g];
  double E = 0.0;
  if (q->model & OR_COUNT_IDLE) {
    double D = 0.0;
    for (int i = 0; i < q->n; i++)
      D = D + ((double)P->p[i * P->lp + l100] - ps) * (double)P->t[i * P->lp + l100];
    E = ((double)q->g * ps) * T + D;
  } else {
    for (int i = 0; i < q->n; i++) {
      double t = (double)P->t[i * P->lp + l100], p = (double)P->p[i * P->lp + l100];
      double e = p * t;
      if (q->model & OR_POWER_CAP) {
        double dyn = (p - ps) * t, tc = dyn / capd;
        if (tc > t) e = ps * tc + dyn;
      }
      E = E + e;
    }
  }
  if (q->tseq_base > 0.0) T = q->tseq_base;   /* R29: baselines of the unsplit queue */
  if (q->eseq_base > 0.0) E = q->eseq_base;
  *tseq = T; *eseq = E;
}

/* ------------------------------------------------------------------ score */
/* a[i]: group of workflow i; k groups; pl[i]: PROFILE level index of i;
 * q: G and the model variant bits.  returns 1 if feasible (T,E filled), 0
 * otherwise. */
int oracle_score_config(const or_profile *P, const or_query *q, int n, const int *a, int k,
                        const int *pl, double *Tout, double *Eout) {
  const int lp = P->lp;
  for (int g = 0; g < k; g++) {
    long long M = 0;
    for (int i = 0; i < n; i++) if (a[i] == g) M += P->mem[i];
    if (M > (long long)P->mem_cap) return 0;
  }
  const double ps = (double)P->ps;
  const double capd = (double)q->power_cap - ps;
  double T = 0.0, E = 0.0, Dall = 0.0;
  for (int g = 0; g < k; g++) {
    double U = 0.0, B = 0.0;
    for (int i = 0; i < n; i++) if (a[i] == g) {
      U = U + (double)P->u[i * lp + pl[i]];
      B = B + (double)P->bw[i * lp + pl[i]];
    }
    if ((q->model & OR_NO_INTERFERENCE) && (U > 1.0 || B > 1.0)) return 0;
    double c = 1.0;
    if (U > c) c = U;
    if (B > c) c = B;
    double Tg = 0.0;
    if (q->model & OR_TIME_SLICE) {          /* R30: the slices one after another */
      for (int i = 0; i < n; i++) if (a[i] == g) {
        double tau = (double)P->t[i * lp + pl[i]];
        if (q->model & OR_POWER_CAP) {
          double tc = (((double)P->p[i * lp + pl[i]] - ps) * (double)P->t[i * lp + pl[i]]) / capd;
          if (tc > tau) tau = tc;
        }
        Tg = Tg + tau;
      }
    } else {
      for (int i = 0; i < n; i++) if (a[i] == g) {
        double sigma = 1.0;
        for (int j = 0; j < n; j++) if (a[j] == g && j != i)
          sigma = sigma + (double)P->d[((size_t)(i * lp + pl[i]) * P->n + j) * lp + pl[j]];
        double tau = ((double)P->t[i * lp + pl[i]] * sigma) * c;
        if (tau > Tg) Tg = tau;
      }
    }
    double D = 0.0;
    for (int i = 0; i < n; i++) if (a[i] == g) {
      double dyn = ((double)P->p[i * lp + pl[i]] - ps) * (double)P->t[i * lp + pl[i]];
      D = D + dyn;
    }
    if ((q->model & OR_POWER_CAP) && !(q->model & OR_TIME_SLICE)) {
      double tc = D / capd;
      if (tc > Tg) Tg = tc;
    }
    double Eg = ps * Tg + D;
    if (Tg > T) T = Tg;
    E = E + Eg;
    Dall = Dall + D;
  }
  if (q->model & OR_COUNT_IDLE) E = ((double)q->g * ps) * T + Dall;
  *Tout = T; *Eout = E;
  return 1;
}

static double objective(double tseq, double eseq, double T, double E, int a, int b) {
  double X = tseq / T, Y = eseq / E, F = 1.0;
  for (int i = 0; i < a; i++) F = F * X;
  for (int i = 0; i < b; i++) F = F * Y;
  return F;
}

/* ------------------------------------------------------------ enumeration */
typedef struct {
  const or_profile *P; const or_query *q;
  double tseq, eseq;
  int a[64], sz[64];
  or_best *best;
  or_point *par; int par_n, par_cap, par_overflow;
  uint64_t ncfg, nfeas;
  /* single-config extraction */
  int extract; uint64_t want; int *out_a, *out_lv; int got;
  /* window scores: (T, E) of every configuration of [lo, hi), NaN if infeasible */
  double *outT, *outE;
} ctx_t;

static void pareto_add(ctx_t *C, uint64_t idx, double T, double E) {
  for (int i = 0; i < C->par_n; i++)
    if (C->par[i].t <= T && C->par[i].e <= E) return;   /* dominated or equal */
  int w = 0;
  for (int i = 0; i < C->par_n; i++)
    if (!(T <= C->par[i].t && E <= C->par[i].e)) C->par[w++] = C->par[i];
  C->par_n = w;
  if (C->par_n >= C->par_cap) { C->par_overflow = 1; return; }
  C->par[C->par_n].idx = idx; C->par[C->par_n].t = T; C->par[C->par_n].e = E;
  C->par_n++;
}

static void leaf(ctx_t *C, int k, uint64_t base) {
  const or_query *q = C->q;
  int nd = q->scope == 0 ? q->n : k;
  u128 ndig = ipow((u128)q->L, nd);
  u128 lo = q->lo > base ? q->lo - base : 0;
  u128 hi = (u128)q->hi - base < ndig ? (u128)q->hi - base : ndig;
  int pl[64], digit[64];
  for (u128 v = lo; v < hi; v++) {
    u128 x = v;
    for (int j = nd - 1; j >= 0; j--) { digit[j] = (int)(x % q->L); x /= q->L; }
    for (int i = 0; i < q->n; i++)
      pl[i] = q->lev[q->scope == 0 ? digit[i] : digit[C->a[i]]];
    uint64_t idx = base + (uint64_t)v;
    if (C->extract) {
      if (idx == C->want) {
        for (int i = 0; i < q->n; i++) { C->out_a[i] = C->a[i]; }
        for (int j = 0; j < nd; j++) C->out_lv[j] = digit[j];
        C->got = 1;
      }
      continue;
    }
    C->ncfg++;
    double T, E;
    if (!oracle_score_config(C->P, q, q->n, C->a, k, pl, &T, &E)) {
      if (C->outT) { C->outT[idx - q->lo] = __builtin_nan(""); C->outE[idx - q->lo] = __builtin_nan(""); }
      continue;
    }
    C->nfeas++;
    if (C->outT) { C->outT[idx - q->lo] = T; C->outE[idx - q->lo] = E; }
    for (int w = 0; w < q->nw; w++) {
      double F = objective(C->tseq, C->eseq, T, E, q->wa[w], q->wb[w]);
      if (!C->best[w].found || F > C->best[w].f) {   /* strict: lowest index wins ties */
        C->best[w].found = 1; C->best[w].f = F; C->best[w].idx = idx;
        C->best[w].t = T; C->best[w].e = E;
      }
    }
    if (q->want_pareto) pareto_add(C, idx, T, E);
  }
}

/* place element i given b open groups; base = index of the first config in subtree */
static void rec(ctx_t *C, int i, int b, uint64_t base) {
  const or_query *q = C->q;
  if (i == q->n) { leaf(C, b, base); return; }
  int cap = q->c;
  for (int j = 0; j <= b; j++) {
    if (j == b && b >= q->g) break;
    if (j < b && C->sz[j] >= cap) continue;
    C->a[i] = j;
    C->sz[j]++;
    int nb = j == b ? b + 1 : b;
    u128 cnt = subtree(i + 1, nb, C->sz);
    if ((u128)base + cnt > q->lo && base < q->hi) rec(C, i + 1, nb, base);
    C->sz[j]--;
    if ((u128)base + cnt >= (u128)q->hi) return;
    base += (uint64_t)cnt;
  }
}

/* Full/window search.  Returns 0 ok, -4 Pareto capacity overflow. */
int oracle_search(const or_profile *P, const or_query *q, int l100,
                  or_best *best, or_point *pareto, int pareto_cap, int *npareto,
                  uint64_t *nconfigs, uint64_t *nfeasible) {
  ctx_t *C = calloc(1, sizeof(ctx_t));
  C->P = P; C->q = q; C->best = best;
  for (int w = 0; w < q->nw; w++) memset(&best[w], 0, sizeof(or_best));
  C->par = pareto; C->par_cap = pareto_cap;
  oracle_constants(P, q, l100, &C->tseq, &C->eseq);
  count_setup(q);
  C->a[0] = 0; C->sz[0] = 1;
  if (q->n >= 1 && q->lo < q->hi) rec(C, 1, 1, 0);
  *npareto = C->par_n; *nconfigs = C->ncfg; *nfeasible = C->nfeas;
  int ovf = C->par_overflow;
  free(C);
  return ovf ? -4 : 0;
}

/* fp64 canonical (T, E) of every configuration of the window [q->lo, q->hi)
 * into outT / outE (index - lo; NaN if infeasible), same enumeration as
 * oracle_search.  Returns the number of configurations. */
uint64_t oracle_score_window(const or_profile *P, const or_query *q, double *outT, double *outE) {
  ctx_t *C = calloc(1, sizeof(ctx_t));
  C->P = P; C->q = q; C->outT = outT; C->outE = outE;
  or_best dummy[8];
  C->best = dummy;
  or_query q2 = *q; q2.nw = 0; q2.want_pareto = 0;
  C->q = &q2;
  count_setup(&q2);
  C->a[0] = 0; C->sz[0] = 1;
  if (q2.n >= 1 && q2.lo < q2.hi) rec(C, 1, 1, 0);
  uint64_t n = C->ncfg;
  free(C);
  return n;
}

/* Decode index -> (RGS a[n], level digits lv[n or k]); returns k or -1. */
int oracle_config(const or_query *q0, uint64_t idx, int *a, int *lv) {
  or_query q = *q0; q.lo = idx; q.hi = idx + 1;
  ctx_t *C = calloc(1, sizeof(ctx_t));
  C->q = &q; C->extract = 1; C->want = idx; C->out_a = a; C->out_lv = lv;
  count_setup(&q);
  C->a[0] = 0; C->sz[0] = 1;
  rec(C, 1, 1, 0);
  int k = -1;
  if (C->got) { k = 0; for (int i = 0; i < q.n; i++) if (a[i] + 1 > k) k = a[i] + 1; }
  free(C);
  return k;
}

/* F of one configuration, for tests */
double oracle_objective(double tseq, double eseq, double T, double E, int a, int b) {
  return objective(tseq, eseq, T, E, a, b);
}
