/*
 * oracle/dpcert.c -- O3: exact subset-DP certificate of the PER_GPU optimum
 * values and Pareto-front values (TEST INFRASTRUCTURE ONLY; same usage rules
 * as enum.c, shares no code with the CUDA path).
 *
 * Used where O1 cannot enumerate (c4: 2.07e14 configurations).  A PER_GPU
 * configuration is a sequence of groups in block order (group j contains the
 * smallest workflow not in groups 0..j-1), each with its own level; in the
 * canonical score T = max_g T_g and
 * E = ((0 + E_0) + E_1) + ...  in exactly that group order.  So the set of
 * reachable (T, E) after covering workflow set S with k groups obeys
 *   F(S u B, k+1) >= { (max(T, T_B(mu)), fl(E + E_B(mu))) : (T,E) in F(S,k) }
 * for every feasible group B containing min(~S), |B| <= C, and level mu.
 * Both maps are monotone (IEEE rounding is monotone), so Pareto-dominated
 * partial states can be pruned without losing any final Pareto point.  The
 * final front at S = all workflows (k <= G) is the exact set of distinct
 * Pareto (T, E) values of the whole space, and max F_w over it is the exact
 * optimum value of every product metric (F is decreasing in T and E).
 * Group tuples T_B, E_B follow the canonical per-group order of enum.c.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
  int n, lp;
  const int *level_pct;
  const float *t, *p, *u, *bw;
  const int *mem;
  const float *d;
  int mem_cap;
  float ps;
} or_profile;

typedef struct { double t, e; } pt;
typedef struct { pt *p; int n, cap, clean; } flist;

static int cmp_pt(const void *a, const void *b) {
  const pt *x = a, *y = b;
  if (x->t != y->t) return x->t < y->t ? -1 : 1;
  if (x->e != y->e) return x->e < y->e ? -1 : 1;
  return 0;
}

static void prune(flist *f) {  /* sort by T asc, keep strictly decreasing E */
  if (f->n == 0) { f->clean = 0; return; }
  qsort(f->p, f->n, sizeof(pt), cmp_pt);
  int w = 0;
  for (int i = 0; i < f->n; i++)
    if (w == 0 || f->p[i].e < f->p[w - 1].e) f->p[w++] = f->p[i];
  f->n = w;
  f->clean = w;
}

static void push(flist *f, double t, double e) {
  if (f->n == f->cap) {
    if (f->n >= 64) prune(f);
    if (f->cap == 0 || 2 * f->n > f->cap) {
      f->cap = f->cap ? 2 * f->cap : 16;
      f->p = realloc(f->p, sizeof(pt) * f->cap);
    }
  }
  f->p[f->n].t = t;
  f->p[f->n].e = e;
  f->n++;
}

/* canonical per-group tuple (members = bits of B ascending, all at profile level pl) */
static int group_tuple(const or_profile *P, unsigned B, int pl, double *Tg_out, double *Eg_out) {
  const int lp = P->lp, n = P->n;
  long long M = 0;
  for (int i = 0; i < n; i++) if (B >> i & 1) M += P->mem[i];
  if (M > (long long)P->mem_cap) return 0;
  double U = 0.0, Bw = 0.0;
  for (int i = 0; i < n; i++) if (B >> i & 1) {
    U = U + (double)P->u[i * lp + pl];
    Bw = Bw + (double)P->bw[i * lp + pl];
  }
  double c = 1.0;
  if (U > c) c = U;
  if (Bw > c) c = Bw;
  double Tg = 0.0;
  for (int i = 0; i < n; i++) if (B >> i & 1) {
    double sigma = 1.0;
    for (int j = 0; j < n; j++) if ((B >> j & 1) && j != i)
      sigma = sigma + (double)P->d[((size_t)(i * lp + pl) * P->n + j) * lp + pl];
    double tau = ((double)P->t[i * lp + pl] * sigma) * c;
    if (tau > Tg) Tg = tau;
  }
  const double ps = (double)P->ps;
  double D = 0.0;
  for (int i = 0; i < n; i++) if (B >> i & 1)
    D = D + ((double)P->p[i * lp + pl] - ps) * (double)P->t[i * lp + pl];
  *Tg_out = Tg;
  *Eg_out = ps * Tg + D;
  return 1;
}

/* n workflows (the profile's first n), g GPUs, c clients max, L levels
 * (profile level indices lev[]).  Writes the final front (T asc) to out;
 * returns its size, or -1 if out_cap is too small / n too large. */
int oracle_dpcert(const or_profile *P0, int n, int g, int c, int L, const int *lev,
                  double *out_t, double *out_e, int out_cap) {
  if (n < 1 || n > 20) return -1;
  or_profile Pv = *P0;
  const or_profile *P = &Pv;
  Pv.n = P0->n;  /* strides use the profile's N */
  const unsigned full = (1u << n) - 1;
  const size_t NS = (size_t)1 << n;
  double *gT = malloc(sizeof(double) * NS * L), *gE = malloc(sizeof(double) * NS * L);
  unsigned char *gok = calloc(NS, 1);
  for (unsigned B = 1; B <= full; B++) {
    if (__builtin_popcount(B) > c) continue;
    int ok = 1;
    for (int m = 0; m < L && ok; m++)
      ok = group_tuple(P, B, lev[m], &gT[(size_t)B * L + m], &gE[(size_t)B * L + m]);
    gok[B] = (unsigned char)ok;
  }
  flist *F = calloc(NS * (size_t)(g + 1), sizeof(flist));
  push(&F[0], 0.0, 0.0);
  for (unsigned S = 0; S < full; S++) {
    const unsigned rest = full & ~S;
    const unsigned low = rest & (0u - rest);
    const unsigned others = rest & ~low;
    for (int k = 0; k < g; k++) {
      flist *f = &F[(size_t)S * (g + 1) + k];
      if (f->n == 0) continue;
      prune(f);
      /* all B = low | sub, sub subset of others */
      unsigned sub = others;
      for (;;) {
        const unsigned B = low | sub;
        if (gok[B]) {
          flist *to = &F[(size_t)(S | B) * (g + 1) + k + 1];
          for (int m = 0; m < L; m++) {
            const double tb = gT[(size_t)B * L + m], eb = gE[(size_t)B * L + m];
            for (int i = 0; i < f->n; i++) {
              const double T = f->p[i].t > tb ? f->p[i].t : tb;
              push(to, T, f->p[i].e + eb);
            }
          }
        }
        if (sub == 0) break;
        sub = (sub - 1) & others;
      }
      free(f->p);
      f->p = 0;
      f->n = f->cap = 0;
    }
  }
  flist fin = {0, 0, 0, 0};
  for (int k = 1; k <= g; k++) {
    flist *f = &F[(size_t)full * (g + 1) + k];
    for (int i = 0; i < f->n; i++) push(&fin, f->p[i].t, f->p[i].e);
    free(f->p);
  }
  prune(&fin);
  int nout = fin.n;
  if (nout <= out_cap)
    for (int i = 0; i < nout; i++) { out_t[i] = fin.p[i].t; out_e[i] = fin.p[i].e; }
  else
    nout = -1;
  free(fin.p);
  free(F);
  free(gT);
  free(gE);
  free(gok);
  return nout;
}

/*
 * O4: the same certificate for PER_CLIENT level scope (every client its own
 * level, the literal reading of BASELINE.json's "per-client
 * active-thread percentage", PAPER.md L75 granularity).  A group's tuple now
 * depends on its members' level vector: for every feasible group B the Pareto
 * front PF(B) of (T_B, E_B) over all L^|B| level vectors is enumerated (plain
 * loops, canonical order of enum.c), then the block-order DP of oracle_dpcert
 * runs over those fronts.  Pruning dominated level vectors of a group is
 * exact for the same reason as above (max and + are monotone under rounding).
 *
 * The two phases are separate entry points so that the first (sum_B L^|B|
 * level vectors: 5^16 = 1.5e11 for n = 16, L = 4) can run in several
 * processes over disjoint ranges of B (oracle.dp_certificate(procs=...)):
 *   oracle_client_fronts(B_lo, B_hi)  -> PF(B) for B in [B_lo, B_hi)
 *   oracle_client_dp(fronts)          -> the block-order DP
 * oracle_dpcert_client composes them in one process.
 */

/* canonical per-group tuple of group m[0] < m[1] < ... < m[s-1] (ascending
 * members), member m[x] at profile level pl[x]; same order as enum.c */
static void group_tuple_members(const or_profile *P, const int *m, int s, const int *pl, double *Tg_out,
                                double *Eg_out) {
  const int lp = P->lp;
  double U = 0.0, Bw = 0.0;
  for (int x = 0; x < s; x++) {
    U = U + (double)P->u[m[x] * lp + pl[x]];
    Bw = Bw + (double)P->bw[m[x] * lp + pl[x]];
  }
  double c = 1.0;
  if (U > c) c = U;
  if (Bw > c) c = Bw;
  /* sigma_x = 1 + sum over y ascending, y != x: the y loop is outside so the
   * s sums advance together (each one still adds its terms in ascending y) */
  double sigma[32];
  const float *row[32];
  for (int x = 0; x < s; x++) {
    sigma[x] = 1.0;
    row[x] = P->d + (size_t)(m[x] * lp + pl[x]) * P->n * lp;
  }
  for (int y = 0; y < s; y++) {
    const int col = m[y] * lp + pl[y];
    for (int x = 0; x < s; x++) if (x != y) sigma[x] = sigma[x] + (double)row[x][col];
  }
  double Tg = 0.0;
  for (int x = 0; x < s; x++) {
    double tau = ((double)P->t[m[x] * lp + pl[x]] * sigma[x]) * c;
    if (tau > Tg) Tg = tau;
  }
  const double ps = (double)P->ps;
  double D = 0.0;
  for (int x = 0; x < s; x++)
    D = D + ((double)P->p[m[x] * lp + pl[x]] - ps) * (double)P->t[m[x] * lp + pl[x]];
  *Tg_out = Tg;
  *Eg_out = ps * Tg + D;
}

/* The same L tuples as group_tuple_members for the L levels of the last
 * member m[s-1] (pl[0..s-2] fixed): every canonical sum adds the last
 * member's term last (members ascending), so the sums over m[0..s-2] are
 * formed once and the last member's term is added per level -- the same
 * operations in the same order, hence bitwise the same results (pinned:
 * tests/test_oracle_cert.py::test_client_fronts_batched_equals_plain). */
static void group_tuples_last(const or_profile *P, const int *m, int s, const int *pl, int L, const int *lev,
                              double *Tg_out, double *Eg_out) {
  const int lp = P->lp, z = s - 1, mz = m[s - 1];
  double U0 = 0.0, Bw0 = 0.0, D0 = 0.0;
  const double ps = (double)P->ps;
  double sig0[32];
  const float *row[32];
  for (int x = 0; x < z; x++) {
    U0 = U0 + (double)P->u[m[x] * lp + pl[x]];
    Bw0 = Bw0 + (double)P->bw[m[x] * lp + pl[x]];
    D0 = D0 + ((double)P->p[m[x] * lp + pl[x]] - ps) * (double)P->t[m[x] * lp + pl[x]];
    sig0[x] = 1.0;
    row[x] = P->d + (size_t)(m[x] * lp + pl[x]) * P->n * lp;
  }
  for (int y = 0; y < z; y++) {
    const int col = m[y] * lp + pl[y];
    for (int x = 0; x < z; x++) if (x != y) sig0[x] = sig0[x] + (double)row[x][col];
  }
  for (int j = 0; j < L; j++) {
    const int cz = mz * lp + lev[j];
    const double U = U0 + (double)P->u[cz], Bw = Bw0 + (double)P->bw[cz];
    double c = 1.0;
    if (U > c) c = U;
    if (Bw > c) c = Bw;
    double Tg = 0.0;
    for (int x = 0; x < z; x++) {
      const double sigma = sig0[x] + (double)row[x][cz];
      const double tau = ((double)P->t[m[x] * lp + pl[x]] * sigma) * c;
      if (tau > Tg) Tg = tau;
    }
    const float *rz = P->d + (size_t)cz * P->n * lp;
    double sigma = 1.0;
    for (int y = 0; y < z; y++) sigma = sigma + (double)rz[m[y] * lp + pl[y]];
    const double tau = ((double)P->t[cz] * sigma) * c;
    if (tau > Tg) Tg = tau;
    const double D = D0 + ((double)P->p[cz] - ps) * (double)P->t[cz];
    Tg_out[j] = Tg;
    Eg_out[j] = ps * Tg + D;
  }
}

/* PF(B) for B in [B_lo, B_hi) (groups of the first n workflows, |B| <= c):
 * off[B - B_lo] .. off[B - B_lo + 1] index the points of PF(B) in out_t /
 * out_e (T ascending, E strictly decreasing; empty if B is not feasible).
 * batched = 0: every level vector through group_tuple_members (the plain
 * form); 1: the last member's L levels at once (group_tuples_last).
 * Returns the number of points written, or -1 if out_cap is too small. */
long long oracle_client_fronts(const or_profile *P, int n, int c, int L, const int *lev, unsigned B_lo,
                               unsigned B_hi, double *out_t, double *out_e, long long *off,
                               long long out_cap, int batched) {
  long long w = 0;
  flist f = {0, 0, 0, 0};
  for (unsigned B = B_lo; B < B_hi; B++) {
    off[B - B_lo] = w;
    const int s = __builtin_popcount(B);
    if (B == 0 || s > c || B >> n) continue;
    int m[32], pl[32];
    int k = 0;
    long long M = 0;
    for (int i = 0; i < n; i++) if (B >> i & 1) { m[k++] = i; M += P->mem[i]; }
    if (M > (long long)P->mem_cap) continue;   /* memory (L87, L91): same for every vector */
    /* every level vector: digits dg[0..s-1] counted in base L (last member
     * fastest), member m[x] at profile level lev[dg[x]]; batched: the last
     * digit is swept inside group_tuples_last */
    const int nd = batched ? s - 1 : s;
    int dg[32];
    for (int x = 0; x < s; x++) { dg[x] = 0; pl[x] = lev[0]; }
    f.n = 0;
    for (;;) {
      if (batched) {
        double Tg[64], Eg[64];
        group_tuples_last(P, m, s, pl, L, lev, Tg, Eg);
        for (int j = 0; j < L; j++) push(&f, Tg[j], Eg[j]);
      } else {
        double Tg, Eg;
        group_tuple_members(P, m, s, pl, &Tg, &Eg);
        push(&f, Tg, Eg);
      }
      int x = nd - 1;
      while (x >= 0 && dg[x] == L - 1) { dg[x] = 0; pl[x] = lev[0]; x--; }
      if (x < 0) break;
      dg[x]++;
      pl[x] = lev[dg[x]];
    }
    prune(&f);
    if (w + f.n > out_cap) { free(f.p); return -1; }
    for (int i = 0; i < f.n; i++) { out_t[w] = f.p[i].t; out_e[w] = f.p[i].e; w++; }
  }
  off[B_hi - B_lo] = w;
  free(f.p);
  return w;
}

/* The block-order DP over given per-group fronts PF(B), B in [0, 2^n):
 * points pf_t/pf_e[off[B] .. off[B+1]).  Final front (T asc) to out. */
int oracle_client_dp(int n, int g, const double *pf_t, const double *pf_e, const long long *off,
                     double *out_t, double *out_e, int out_cap) {
  if (n < 1 || n > 20) return -1;
  const unsigned full = (1u << n) - 1;
  const size_t NS = (size_t)1 << n;
  flist *F = calloc(NS * (size_t)(g + 1), sizeof(flist));
  push(&F[0], 0.0, 0.0);
  for (unsigned S = 0; S < full; S++) {
    const unsigned rest = full & ~S;
    const unsigned low = rest & (0u - rest);
    const unsigned others = rest & ~low;
    for (int k = 0; k < g; k++) {
      flist *f = &F[(size_t)S * (g + 1) + k];
      if (f->n == 0) continue;
      prune(f);
      unsigned sub = others;
      for (;;) {
        const unsigned B = low | sub;
        if (off[B + 1] > off[B]) {
          flist *to = &F[(size_t)(S | B) * (g + 1) + k + 1];
          for (long long q = off[B]; q < off[B + 1]; q++) {
            const double tb = pf_t[q], eb = pf_e[q];
            for (int i = 0; i < f->n; i++) {
              const double T = f->p[i].t > tb ? f->p[i].t : tb;
              push(to, T, f->p[i].e + eb);
            }
          }
        }
        if (sub == 0) break;
        sub = (sub - 1) & others;
      }
      free(f->p);
      f->p = 0;
      f->n = f->cap = 0;
    }
  }
  flist fin = {0, 0, 0, 0};
  for (int k = 1; k <= g; k++) {
    flist *f = &F[(size_t)full * (g + 1) + k];
    for (int i = 0; i < f->n; i++) push(&fin, f->p[i].t, f->p[i].e);
    free(f->p);
  }
  prune(&fin);
  int nout = fin.n;
  if (nout <= out_cap)
    for (int i = 0; i < nout; i++) { out_t[i] = fin.p[i].t; out_e[i] = fin.p[i].e; }
  else
    nout = -1;
  free(fin.p);
  free(F);
  return nout;
}

int oracle_dpcert_client(const or_profile *P, int n, int g, int c, int L, const int *lev,
                         double *out_t, double *out_e, int out_cap) {
  if (n < 1 || n > 16) return -1;
  const size_t NS = (size_t)1 << n;
  long long cap = 1 << 20;
  long long *off = malloc(sizeof(long long) * (NS + 1));
  double *pt_ = 0, *pe_ = 0;
  long long np;
  for (;;) {
    pt_ = realloc(pt_, sizeof(double) * cap);
    pe_ = realloc(pe_, sizeof(double) * cap);
    np = oracle_client_fronts(P, n, c, L, lev, 0, (unsigned)NS, pt_, pe_, off, cap, 0);
    if (np >= 0) break;
    cap *= 4;
  }
  const int nout = oracle_client_dp(n, g, pt_, pe_, off, out_t, out_e, out_cap);
  free(off);
  free(pt_);
  free(pe_);
  return nout;
}
