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
 * active-thread percentage").  A group's tuple now depends on its members'
 * level vector: for every feasible group B the Pareto front PF(B) of
 * (T_B, E_B) over all L^|B| level vectors is enumerated (plain loops,
 * canonical order of enum.c), then the block-order DP of oracle_dpcert runs
 * over those fronts.  Pruning dominated level vectors of a group is exact for
 * the same reason as above (max and + are monotone under rounding).
 */
static int group_tuple_client(const or_profile *P, unsigned B, const int *pl, double *Tg_out,
                              double *Eg_out) {
  const int lp = P->lp, n = P->n;
  long long M = 0;
  for (int i = 0; i < n; i++) if (B >> i & 1) M += P->mem[i];
  if (M > (long long)P->mem_cap) return 0;
  double U = 0.0, Bw = 0.0;
  for (int i = 0; i < n; i++) if (B >> i & 1) {
    U = U + (double)P->u[i * lp + pl[i]];
    Bw = Bw + (double)P->bw[i * lp + pl[i]];
  }
  double c = 1.0;
  if (U > c) c = U;
  if (Bw > c) c = Bw;
  double Tg = 0.0;
  for (int i = 0; i < n; i++) if (B >> i & 1) {
    double sigma = 1.0;
    for (int j = 0; j < n; j++) if ((B >> j & 1) && j != i)
      sigma = sigma + (double)P->d[((size_t)(i * lp + pl[i]) * P->n + j) * lp + pl[j]];
    double tau = ((double)P->t[i * lp + pl[i]] * sigma) * c;
    if (tau > Tg) Tg = tau;
  }
  const double ps = (double)P->ps;
  double D = 0.0;
  for (int i = 0; i < n; i++) if (B >> i & 1)
    D = D + ((double)P->p[i * lp + pl[i]] - ps) * (double)P->t[i * lp + pl[i]];
  *Tg_out = Tg;
  *Eg_out = ps * Tg + D;
  return 1;
}

int oracle_dpcert_client(const or_profile *P0, int n, int g, int c, int L, const int *lev,
                         double *out_t, double *out_e, int out_cap) {
  if (n < 1 || n > 14) return -1;
  or_profile Pv = *P0;
  const or_profile *P = &Pv;
  const unsigned full = (1u << n) - 1;
  const size_t NS = (size_t)1 << n;
  flist *PF = calloc(NS, sizeof(flist));   /* per-group front over level vectors */
  for (unsigned B = 1; B <= full; B++) {
    const int s = __builtin_popcount(B);
    if (s > c) continue;
    int mem[32], pl[64];
    int m = 0;
    for (int i = 0; i < n; i++) if (B >> i & 1) mem[m++] = i;
    long long nv = 1;
    for (int k = 0; k < s; k++) nv *= L;
    for (long long v = 0; v < nv; v++) {
      long long x = v;
      for (int k = s - 1; k >= 0; k--) { pl[mem[k]] = lev[x % L]; x /= L; }
      double Tg, Eg;
      if (!group_tuple_client(P, B, pl, &Tg, &Eg)) break;   /* memory: same for every vector */
      push(&PF[B], Tg, Eg);
    }
    prune(&PF[B]);
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
      unsigned sub = others;
      for (;;) {
        const unsigned B = low | sub;
        const flist *pb = &PF[B];
        if (pb->n) {
          flist *to = &F[(size_t)(S | B) * (g + 1) + k + 1];
          for (int q = 0; q < pb->n; q++) {
            const double tb = pb->p[q].t, eb = pb->p[q].e;
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
  for (size_t B = 0; B < NS; B++) free(PF[B].p);
  free(PF);
  return nout;
}
