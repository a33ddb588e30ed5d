// host_core.cpp -- host side of the search: validation, the DP count table,
// rank/unrank, the sequential baselines, the fp64 canonical score, the staged
// device tables and error bounds, and the exact cross-rank merge.
//
// Compiled with -ffp-contract=off (no FMA contraction): every fp64 operation
// below rounds once, in the written order, so host_score / host_constants are
// bitwise equal to the device fp64 refine and to the CPU oracle (which is a
// separate implementation under oracle/, sharing no code with this file).
//
// PAPER.md = /root/reference/PAPER.md; R<n> = DESIGN.md "Readings of the paper".
#include <algorithm>
#include <cmath>
#include <cstring>
#include <map>

#include "sched_internal.hpp"

namespace sched {

// ------------------------------------------------------------ validation
int validate_profile(const sched_profile *in, Profile *P) {
  if (!in || !P) return SCHED_E_INVALID;
  const int n = in->n_workflows, lp = in->n_levels;
  if (n < 1 || n > kMaxN || lp < 1 || lp > SCHED_MAX_PROFILE_LEVELS) return SCHED_E_INVALID;
  if (!in->level_pct || !in->solo_time_s || !in->solo_power_w || !in->sm_util || !in->bw_util ||
      !in->max_mem_mib || !in->corun_slowdown)
    return SCHED_E_INVALID;
  if (!(std::isfinite(in->static_power_w) && in->static_power_w >= 0.f)) return SCHED_E_INVALID;
  if (in->mem_capacity_mib <= 0) return SCHED_E_INVALID;
  P->n = n;
  P->lp = lp;
  P->pct.assign(in->level_pct, in->level_pct + lp);
  P->l100 = -1;
  for (int l = 0; l < lp; l++) {
    if (P->pct[l] <= 0 || P->pct[l] > 100) return SCHED_E_INVALID;
    if (l > 0 && P->pct[l] <= P->pct[l - 1]) return SCHED_E_INVALID;
    if (P->pct[l] == 100) P->l100 = l;
  }
  if (P->l100 < 0) return SCHED_E_INVALID;  // sequential baseline runs at 100% (R16)
  const size_t nl = (size_t)n * lp;
  P->t.assign(in->solo_time_s, in->solo_time_s + nl);
  P->p.assign(in->solo_power_w, in->solo_power_w + nl);
  P->u.assign(in->sm_util, in->sm_util + nl);
  P->bw.assign(in->bw_util, in->bw_util + nl);
  P->d.assign(in->corun_slowdown, in->corun_slowdown + nl * nl);
  P->mem.assign(in->max_mem_mib, in->max_mem_mib + n);
  P->mem_cap = in->mem_capacity_mib;
  P->ps = in->static_power_w;
  for (size_t k = 0; k < nl; k++) {
    if (!(std::isfinite(P->t[k]) && P->t[k] > 0.f && P->t[k] < 1e30f)) return SCHED_E_INVALID;
    // static power may not exceed average power: keeps every energy term >= 0 (R8)
    if (!(std::isfinite(P->p[k]) && P->p[k] >= P->ps && P->p[k] < 1e30f)) return SCHED_E_INVALID;
    if (!(std::isfinite(P->u[k]) && P->u[k] >= 0.f && P->u[k] < 1e6f)) return SCHED_E_INVALID;
    if (!(std::isfinite(P->bw[k]) && P->bw[k] >= 0.f && P->bw[k] < 1e6f)) return SCHED_E_INVALID;
  }
  for (size_t k = 0; k < nl * nl; k++)
    if (!(std::isfinite(P->d[k]) && P->d[k] >= 0.f && P->d[k] < 1e6f)) return SCHED_E_INVALID;
  for (int i = 0; i < n; i++)
    if (P->mem[i] < 0) return SCHED_E_INVALID;
  return SCHED_OK;
}

int resolve_query_shape(const sched_query *q, int n_profile_levels, Query *Q) {
  if (!q || !Q) return SCHED_E_INVALID;
  std::memset(Q, 0, sizeof *Q);
  if (q->n < 1 || q->n > kMaxN || q->g < 1 || q->g > kMaxG) return SCHED_E_INVALID;
  if (q->max_clients < 1 || q->max_clients > SCHED_MAX_CLIENTS) return SCHED_E_INVALID;
  if (q->level_scope != SCHED_PER_CLIENT && q->level_scope != SCHED_PER_GPU) return SCHED_E_INVALID;
  if (q->n_weights < 0 || q->n_weights > kMaxW) return SCHED_E_INVALID;
  if (q->n_weights > 0 && !q->weights) return SCHED_E_INVALID;
  Q->n = q->n;
  Q->g = q->g;
  Q->c = std::min(q->max_clients, q->n);
  Q->scope = q->level_scope;
  Q->nw = q->n_weights;
  int L = 0;
  for (int l = 0; l < 32; l++) {
    if (!(q->level_mask >> l & 1u)) continue;
    if (l >= n_profile_levels || L >= kMaxL) return SCHED_E_INVALID;
    Q->lev[L++] = l;
  }
  if (L < 1) return SCHED_E_INVALID;
  Q->L = L;
  for (int w = 0; w < Q->nw; w++) {
    int a = q->weights[2 * w], b = q->weights[2 * w + 1];
    if (a < 0 || b < 0 || a > SCHED_MAX_EXPONENT || b > SCHED_MAX_EXPONENT || a + b < 1)
      return SCHED_E_INVALID;
    Q->wa[w] = a;
    Q->wb[w] = b;
  }
  Q->count = q->shard_count;
  Q->rank = q->shard_rank;
  if (Q->count < 1 || Q->rank < 0 || Q->rank >= Q->count) return SCHED_E_INVALID;
  Q->chunk_log2 = q->chunk_log2 == 0 ? 24 : q->chunk_log2;  // 2^24: profiles/r01_chunk_sweep.txt
  if (Q->chunk_log2 < 12 || Q->chunk_log2 > 40) return SCHED_E_INVALID;
  Q->want_pareto = q->want_pareto != 0;
  Q->cand_cap = q->candidate_cap == 0 ? (1u << 20) : q->candidate_cap;
  Q->lo = q->index_lo;
  Q->hi = q->index_hi;
  if (q->model_flags & ~(uint32_t)(SCHED_MODEL_COUNT_IDLE | SCHED_MODEL_NO_INTERFERENCE | SCHED_MODEL_POWER_CAP |
                                    SCHED_MODEL_TIME_SLICE))
    return SCHED_E_INVALID;
  if ((q->model_flags & SCHED_MODEL_TIME_SLICE) && (q->model_flags & SCHED_MODEL_NO_INTERFERENCE))
    return SCHED_E_INVALID;  // R30: the hard rule is about concurrent clients
  Q->model = q->model_flags;
  Q->pcap = q->power_cap_w;
  if ((Q->model & SCHED_MODEL_POWER_CAP) && !(std::isfinite(Q->pcap) && Q->pcap > 0.f)) return SCHED_E_INVALID;
  return SCHED_OK;
}

int resolve_query(const Profile *P, const sched_query *q, Query *Q, uint64_t *total) {
  if (!P) return SCHED_E_INVALID;
  int st = resolve_query_shape(q, P->lp, Q);
  if (st) return st;
  if (Q->n > P->n) return SCHED_E_INVALID;
  if ((Q->model & SCHED_MODEL_POWER_CAP) && !(Q->pcap > P->ps)) return SCHED_E_INVALID;
  Space sp;
  st = build_space(*Q, &sp);
  if (st) return st;
  if (Q->hi == UINT64_MAX || Q->hi > sp.total) Q->hi = sp.total;
  if (Q->lo > Q->hi) return SCHED_E_INVALID;
  if (total) *total = sp.total;
  return SCHED_OK;
}

// ------------------------------------------------------------ DP count table
namespace {
typedef unsigned __int128 u128;
const u128 kSat = (u128)1 << 100;

struct Builder {
  const Query &q;
  Space &sp;
  std::map<std::vector<int>, int> ids;
  std::vector<u128> W;
  bool too_many = false;
  Builder(const Query &qq, Space &s) : q(qq), sp(s) {}

  // key = [i, b, hist[1..c-1]] (capped) or [i, b] (uncapped)
  int get(const std::vector<int> &key) {
    auto it = ids.find(key);
    if (it != ids.end()) return it->second;
    const int id = (int)W.size();
    if (id >= 65534) { too_many = true; return 0; }
    ids.emplace(key, id);
    W.push_back(0);
    sp.trans.resize((size_t)(id + 1) * sp.tc, kNoState);
    const int i = key[0], b = key[1];
    u128 w = 0;
    if (i == q.n) {
      int e = q.scope == SCHED_PER_CLIENT ? q.n : b;
      w = 1;
      for (int k = 0; k < e; k++) w *= (u128)q.L;
    } else {
      if (b < q.g) {  // open a new group (it has size 1)
        std::vector<int> nk = key;
        nk[0] = i + 1;
        nk[1] = b + 1;
        if (sp.capped && q.c > 1) nk[2 + 0] += 1;  // hist[1] lives at index 2
        int s2 = get(nk);
        sp.trans[(size_t)id * sp.tc + 0] = (uint16_t)s2;
        w += W[s2];
      }
      if (sp.capped) {
        for (int z = 1; z < q.c; z++) {  // join a group of size z
          if (key[2 + z - 1] == 0) continue;
          std::vector<int> nk = key;
          nk[0] = i + 1;
          nk[2 + z - 1] -= 1;
          if (z + 1 < q.c) nk[2 + z] += 1;  // else the group becomes full
          int s2 = get(nk);
          sp.trans[(size_t)id * sp.tc + z] = (uint16_t)s2;
          w += (u128)key[2 + z - 1] * W[s2];  // any of the hist[z] groups of size z
        }
      } else if (b >= 1) {
        std::vector<int> nk = key;
        nk[0] = i + 1;
        int s2 = get(nk);
        sp.trans[(size_t)id * sp.tc + 1] = (uint16_t)s2;
        w += (u128)b * W[s2];  // any of the b open groups
      }
    }
    if (w > kSat) w = kSat;
    W[id] = w;
    return id;
  }
};
}  // namespace

int build_space(const Query &q, Space *sp) {
  sp->n = q.n;
  sp->g = q.g;
  sp->c = q.c;
  sp->L = q.L;
  sp->scope = q.scope;
  sp->capped = q.c < q.n;
  sp->tc = sp->capped ? q.c : 2;
  sp->trans.clear();
  Builder B(q, *sp);
  std::vector<int> root(sp->capped ? 2 + (q.c - 1) : 2, 0);
  root[0] = 1;
  root[1] = 1;
  if (sp->capped && q.c > 1) root[2] = 1;
  sp->root = B.get(root);
  if (B.too_many) return SCHED_E_TOO_LARGE;
  u128 tot = B.W[sp->root];
  if (tot > ((u128)1 << 63)) return SCHED_E_TOO_LARGE;
  sp->total = (uint64_t)tot;
  sp->W.resize(B.W.size());
  for (size_t k = 0; k < B.W.size(); k++) sp->W[k] = (uint64_t)B.W[k];
  return SCHED_OK;
}

int host_unrank(const Space &sp, uint64_t idx, int8_t *a, int8_t *digits, int *k_out) {
  if (idx >= sp.total) return SCHED_E_INVALID;
  uint64_t r = idx;
  int s = sp.root, b = 1;
  int sz[kMaxG] = {0};
  a[0] = 0;
  sz[0] = 1;
  for (int i = 1; i < sp.n; i++) {
    int chosen = -1;
    for (int j = 0; j <= b; j++) {
      int col;
      if (j < b) {
        if (sp.capped) {
          if (sz[j] >= sp.c) continue;
          col = sz[j];
        } else {
          col = 1;
        }
      } else {
        if (b >= sp.g) break;
        col = 0;
      }
      uint16_t s2 = sp.trans[(size_t)s * sp.tc + col];
      if (s2 == kNoState) continue;
      uint64_t w = sp.W[s2];
      if (r < w) {
        chosen = j;
        s = s2;
        break;
      }
      r -= w;
    }
    if (chosen < 0) return SCHED_E_INVALID;
    a[i] = (int8_t)chosen;
    if (chosen == b) sz[b++] = 1;
    else sz[chosen]++;
  }
  const int nd = sp.scope == SCHED_PER_CLIENT ? sp.n : b;
  for (int d = nd - 1; d >= 0; d--) {
    digits[d] = (int8_t)(r % (uint64_t)sp.L);
    r /= (uint64_t)sp.L;
  }
  if (r != 0) return SCHED_E_INVALID;
  *k_out = b;
  return SCHED_OK;
}

int host_rank(const Space &sp, const int8_t *a, const int8_t *digits, uint64_t *out) {
  if (a[0] != 0) return SCHED_E_INVALID;
  uint64_t idx = 0;
  int s = sp.root, b = 1;
  int sz[kMaxG] = {0};
  sz[0] = 1;
  for (int i = 1; i < sp.n; i++) {
    const int ai = a[i];
    if (ai < 0 || ai > b || ai >= sp.g) return SCHED_E_INVALID;
    int found = 0;
    for (int j = 0; j <= b; j++) {
      int col;
      if (j < b) {
        if (sp.capped) {
          if (sz[j] >= sp.c) {
            if (j == ai) return SCHED_E_INVALID;
            continue;
          }
          col = sz[j];
        } else {
          col = 1;
        }
      } else {
        if (b >= sp.g) break;
        col = 0;
      }
      uint16_t s2 = sp.trans[(size_t)s * sp.tc + col];
      if (s2 == kNoState) {
        if (j == ai) return SCHED_E_INVALID;
        continue;
      }
      if (j == ai) {
        s = s2;
        found = 1;
        break;
      }
      idx += sp.W[s2];
    }
    if (!found) return SCHED_E_INVALID;
    if (ai == b) sz[b++] = 1;
    else sz[ai]++;
  }
  const int nd = sp.scope == SCHED_PER_CLIENT ? sp.n : b;
  uint64_t v = 0;
  for (int d = 0; d < nd; d++) {
    if (digits[d] < 0 || digits[d] >= sp.L) return SCHED_E_INVALID;
    v = v * (uint64_t)sp.L + (uint64_t)digits[d];
  }
  if (sp.W[s] == 0) return SCHED_E_INVALID;
  *out = idx + v;
  return SCHED_OK;
}

// ------------------------------------------------------------ fp64 canonical model
// Sequential baseline ("jobs are scheduled individually on GPUs
// in queue order with no parallel overlap"; R6, R16): list schedule at 100%.
void host_constants(const Profile &P, const Query &q, double *tseq, double *eseq) {
  const double ps = (double)P.ps, capd = (double)q.pcap - ps;
  const bool cap = q.model & SCHED_MODEL_POWER_CAP;
  double fin[kMaxG];
  for (int g = 0; g < q.g; g++) fin[g] = 0.0;
  for (int i = 0; i < q.n; i++) {
    const size_t k = (size_t)i * P.lp + P.l100;
    double t = (double)P.t[k];
    if (cap) {  // R28: a solo task above P_cap runs dyn / (P_cap - P_s)
      const double tc = (((double)P.p[k] - ps) * t) / capd;
      if (tc > t) t = tc;
    }
    int best = 0;
    for (int g = 1; g < q.g; g++)
      if (fin[g] < fin[best]) best = g;
    fin[best] = fin[best] + t;
  }
  double T = 0.0;
  for (int g = 0; g < q.g; g++)
    if (fin[g] > T) T = fin[g];
  double E = 0.0;
  if (q.model & SCHED_MODEL_COUNT_IDLE) {  // R26: E_seq = g P_s T_seq + sum dyn
    double D = 0.0;
    for (int i = 0; i < q.n; i++) {
      const size_t k = (size_t)i * P.lp + P.l100;
      D = D + ((double)P.p[k] - ps) * (double)P.t[k];
    }
    E = ((double)q.g * ps) * T + D;
  } else {
    for (int i = 0; i < q.n; i++) {
      const size_t k = (size_t)i * P.lp + P.l100;
      const double t = (double)P.t[k], p = (double)P.p[k];
      double e = p * t;
      if (cap) {
        const double dyn = (p - ps) * t, tc = dyn / capd;
        if (tc > t) e = ps * tc + dyn;
      }
      E = E + e;
    }
  }
  if (P.tseq_base > 0.0) T = P.tseq_base;  // R29: the unsplit queue's baselines
  if (P.eseq_base > 0.0) E = P.eseq_base;
  *tseq = T;
  *eseq = E;
}

// ------------------------------------------------------------ task splits (R29)
// Workflow i = tasks[i] identical independent tasks (Table III "# Iter.",
// R17); a split runs it as p_i | tasks[i] concurrent clients of
// tasks[i]/p_i tasks each ("split them into multiple
// parallel workflows"; Figs 4-5 "s-p").  Split vectors are ranked
// lexicographically, divisors ascending, workflow 0 most significant.
int split_vectors(int n, const int32_t *tasks, const int32_t *max_split, std::vector<std::vector<int>> *out) {
  if (!tasks || n < 1 || n > kMaxN) return SCHED_E_INVALID;
  std::vector<std::vector<int>> ch(n);
  uint64_t total = 1;
  for (int i = 0; i < n; i++) {
    if (tasks[i] < 1 || tasks[i] > (1 << 20)) return SCHED_E_INVALID;
    const int lim = max_split ? max_split[i] : tasks[i];
    if (lim < 1) return SCHED_E_INVALID;
    for (int d = 1; d <= tasks[i] && d <= lim && d <= kMaxN; d++)
      if (tasks[i] % d == 0) ch[i].push_back(d);
    total *= ch[i].size();
    if (total > (1u << 20)) return SCHED_E_TOO_LARGE;
  }
  out->clear();
  std::vector<int> pos(n, 0);
  for (;;) {  // odometer, last workflow fastest
    std::vector<int> v(n);
    int sum = 0;
    for (int i = 0; i < n; i++) sum += (v[i] = ch[i][pos[i]]);
    if (sum > kMaxN) return SCHED_E_TOO_LARGE;  // more clients than a query takes: cap with max_split
    out->push_back(v);
    int i = n - 1;
    while (i >= 0 && ++pos[i] == (int)ch[i].size()) pos[i--] = 0;
    if (i < 0) break;
  }
  return SCHED_OK;
}

// Expanded client queue (workflow-major): client of workflow i runs
// fl32((t_i * s_i) / K_i) at every level, same power / SM / BW / memory;
// co-run d between clients of workflows i, j is d[i,l][j,m] (siblings: the
// profile's diagonal block, the self co-run slowdown).
int expand_split(const Profile &P, int n, const int32_t *tasks, const std::vector<int> &split, Profile *E) {
  std::vector<int> own;
  for (int i = 0; i < n; i++)
    for (int r = 0; r < split[i]; r++) own.push_back(i);
  const int m = (int)own.size(), lp = P.lp;
  if (m < 1 || m > kMaxN) return SCHED_E_TOO_LARGE;
  E->n = m;
  E->lp = lp;
  E->pct = P.pct;
  E->l100 = P.l100;
  E->mem_cap = P.mem_cap;
  E->ps = P.ps;
  E->tseq_base = E->eseq_base = 0.0;
  E->t.resize((size_t)m * lp);
  E->p.resize((size_t)m * lp);
  E->u.resize((size_t)m * lp);
  E->bw.resize((size_t)m * lp);
  E->mem.resize(m);
  E->d.resize((size_t)m * lp * m * lp);
  for (int a = 0; a < m; a++) {
    const int i = own[a];
    const double K = (double)tasks[i], s = (double)(tasks[i] / split[i]);
    for (int l = 0; l < lp; l++) {
      const size_t src = (size_t)i * lp + l, dst = (size_t)a * lp + l;
      E->t[dst] = (float)(((double)P.t[src] * s) / K);
      E->p[dst] = P.p[src];
      E->u[dst] = P.u[src];
      E->bw[dst] = P.bw[src];
      for (int b = 0; b < m; b++)
        for (int mm = 0; mm < lp; mm++)
          E->d[(dst * m + b) * lp + mm] = P.d[(src * P.n + own[b]) * lp + mm];
    }
    E->mem[a] = P.mem[i];
  }
  return SCHED_OK;
}

// Canonical score (PAPER.md L87 predicate + memory clause, L91, L96).
int host_score(const Profile &P, const Query &q, const int8_t *a, int k, const int8_t *digits,
               double *Tout, double *Eout) {
  const int n = q.n, lp = P.lp;
  int pl[kMaxN];
  for (int i = 0; i < n; i++)
    pl[i] = q.lev[q.scope == SCHED_PER_CLIENT ? digits[i] : digits[a[i]]];
  for (int g = 0; g < k; g++) {
    long long M = 0;
    for (int i = 0; i < n; i++)
      if (a[i] == g) M += P.mem[i];
    if (M > (long long)P.mem_cap) return 0;
  }
  const double ps = (double)P.ps;
  double T = 0.0, E = 0.0, Dall = 0.0;
  for (int g = 0; g < k; g++) {
    double U = 0.0, B = 0.0;
    for (int i = 0; i < n; i++)
      if (a[i] == g) {
        U = U + (double)P.u[(size_t)i * lp + pl[i]];
        B = B + (double)P.bw[(size_t)i * lp + pl[i]];
      }
    if ((q.model & SCHED_MODEL_NO_INTERFERENCE) && (U > 1.0 || B > 1.0)) return 0;  // R27
    double c = 1.0;
    if (U > c) c = U;
    if (B > c) c = B;
    double Tg = 0.0;
    if (q.model & SCHED_MODEL_TIME_SLICE) {  // R30: slices one after another, solo profile
      for (int i = 0; i < n; i++) {
        if (a[i] != g) continue;
        const size_t r = (size_t)i * lp + pl[i];
        double tau = (double)P.t[r];
        if (q.model & SCHED_MODEL_POWER_CAP) {
          const double tc = (((double)P.p[r] - ps) * (double)P.t[r]) / ((double)q.pcap - ps);
          if (tc > tau) tau = tc;
        }
        Tg = Tg + tau;
      }
    }
    for (int i = 0; i < n && !(q.model & SCHED_MODEL_TIME_SLICE); i++) {
      if (a[i] != g) continue;
      double sigma = 1.0;
      for (int j = 0; j < n; j++)
        if (a[j] == g && j != i)
          sigma = sigma + (double)P.d[((size_t)(i * lp + pl[i]) * P.n + j) * lp + pl[j]];
      double tau = ((double)P.t[(size_t)i * lp + pl[i]] * sigma) * c;
      if (tau > Tg) Tg = tau;
    }
    double D = 0.0;
    for (int i = 0; i < n; i++)
      if (a[i] == g) {
        const size_t r = (size_t)i * lp + pl[i];
        D = D + ((double)P.p[r] - ps) * (double)P.t[r];
      }
    if ((q.model & SCHED_MODEL_POWER_CAP) && !(q.model & SCHED_MODEL_TIME_SLICE)) {  // R28
      const double tc = D / ((double)q.pcap - ps);
      if (tc > Tg) Tg = tc;
    }
    const double Eg = ps * Tg + D;
    if (Tg > T) T = Tg;
    E = E + Eg;
    Dall = Dall + D;
  }
  if (q.model & SCHED_MODEL_COUNT_IDLE) E = ((double)q.g * ps) * T + Dall;  // R26
  *Tout = T;
  *Eout = E;
  return 1;
}

double host_objective(double tseq, double eseq, double T, double E, int a, int b) {
  const double X = tseq / T, Y = eseq / E;
  double F = 1.0;
  for (int i = 0; i < a; i++) F = F * X;
  for (int i = 0; i < b; i++) F = F * Y;
  return F;
}

// ------------------------------------------------------------ staged tables
static uint32_t align_up(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }


int build_stage(const Profile &P, const Query &q, const Space &sp, std::vector<unsigned char> *blob,
                DevParams *dp) {
  std::memset(dp, 0, sizeof *dp);
  const int n = q.n, L = q.L, R = n * L, ds = R | 1;
  double tseq, eseq;
  host_constants(P, q, &tseq, &eseq);
  dp->n = n;
  dp->g = q.g;
  dp->c = q.c;
  dp->L = L;
  dp->scope = q.scope;
  dp->nw = q.nw;
  dp->capped = sp.capped;
  dp->tc = sp.tc;
  dp->R = R;
  dp->ds = ds;
  dp->root = sp.root;
  dp->nstates = (int)sp.W.size();
  dp->ps = (double)P.ps;
  dp->tseq = tseq;
  dp->eseq = eseq;
  dp->phat = (float)((double)P.ps * tseq / eseq);
  dp->model = q.model;
  dp->capd = (double)q.pcap - (double)P.ps;
  dp->kcap = (q.model & SCHED_MODEL_POWER_CAP) ? (float)(eseq / (dp->capd * tseq)) : 0.f;
  dp->gps = (double)q.g * (double)P.ps;
  dp->kidle = (float)(dp->gps * tseq / eseq);
  dp->kidle0 = (q.model & SCHED_MODEL_COUNT_IDLE) ? dp->kidle : 0.f;
  dp->mem_cap = P.mem_cap;
  dp->want_pareto = q.want_pareto;
  dp->wb_pos = 1;
  for (int w = 0; w < q.nw; w++) {
    dp->wb_pos &= q.wb[w] >= 1 ? 1 : 0;
    dp->wa[w] = q.wa[w];
    dp->wb[w] = q.wb[w];
  }
  // ---- fp32 error bounds ----
  // relative error of the hot loop's T/T_seq and E/E_seq against the fp64
  // canonical values, u = 2^-24, generous constants (all terms are >= 0).
  const double u = std::ldexp(1.0, -24);
  const double eT = (3.0 * q.c + 8.0) * u;
  const double eE = (3.0 * q.c + 8.0 + n + q.g + 8.0) * u;
  for (int w = 0; w < q.nw; w++) {
    const double eta = q.wa[w] * eT + q.wb[w] * eE + (q.wa[w] + q.wb[w] + 2.0) * u;
    dp->delta[w] = (float)(4.0 * eta);
    dp->mul[w] = 1.f + dp->delta[w];
    // log-domain pre-screen of the run-time-weight tile kernel (search_tile.cuh
    // rt_screen): a*lg2(T) + b*lg2(E) <= lg2(thr * mul) + lmargin whenever the
    // exact proxy test passes, for |lg2| <= 32 of every operand: each __log2f
    // is within 2^-17 absolute there (2 ulp relative), the fp32 proxy within
    // (a+b) u of T^a E^b, the FMUL/FFMA within |L| 2^-23 -- (a+b+1) 2^-15
    // covers the sum with room
    dp->fa[w] = (float)q.wa[w];
    dp->fb[w] = (float)q.wb[w];
    dp->lmargin[w] = (float)std::ldexp((double)(q.wa[w] + q.wb[w] + 1), -15);
  }
  dp->gamma = (float)(2.0 * std::max(eT, eE) + 4.0 * u);
  dp->tlb_scale = std::nextafter(tseq / (1.0 + 2.0 * eT), 0.0);
  {
    float f = (float)dp->tlb_scale;
    if ((double)f > dp->tlb_scale) f = std::nextafter(f, 0.f);
    dp->tlb_scale_f = f;
  }
  // ---- tables ----
  uint32_t off = 0;
  auto take = [&](uint32_t bytes, uint32_t al) {
    off = align_up(off, al);
    uint32_t o = off;
    off += bytes;
    return o;
  };
  dp->off_th = take(4 * R, 16);
  dp->off_u = take(4 * R, 16);
  dp->off_bw = take(4 * R, 16);
  dp->off_dh = take(4 * R, 16);
  dp->off_traw = take(4 * R, 16);
  dp->off_praw = take(4 * R, 16);
  dp->off_mem = take(4 * n, 16);
  dp->off_d = take(4 * R * ds, 16);
  dp->off_W = take(8 * (uint32_t)sp.W.size(), 16);
  dp->off_trans = take(2 * (uint32_t)sp.trans.size(), 16);
  dp->blob_bytes = align_up(off, 16);
  if (dp->blob_bytes > 150 * 1024) return SCHED_E_TOO_LARGE;
  blob->assign(dp->blob_bytes, 0);
  unsigned char *B = blob->data();
  float *th = (float *)(B + dp->off_th), *uu = (float *)(B + dp->off_u);
  float *bw = (float *)(B + dp->off_bw), *dh = (float *)(B + dp->off_dh);
  float *traw = (float *)(B + dp->off_traw), *praw = (float *)(B + dp->off_praw);
  int *mem = (int *)(B + dp->off_mem);
  float *d = (float *)(B + dp->off_d);
  float tlow = 0.f;
  for (int i = 0; i < n; i++) {
    mem[i] = P.mem[i];
    float tmin = 3e38f;
    for (int l = 0; l < L; l++) {
      const int r = i * L + l;
      const size_t k = (size_t)i * P.lp + q.lev[l];
      th[r] = (float)((double)P.t[k] / tseq);
      uu[r] = P.u[k];
      bw[r] = P.bw[k];
      dh[r] = (float)((((double)P.p[k] - (double)P.ps) * (double)P.t[k]) / eseq);
      traw[r] = P.t[k];
      praw[r] = P.p[k];
      tmin = std::min(tmin, th[r]);
    }
    tlow = std::max(tlow, tmin);
    for (int j = 0; j < n; j++)
      for (int l = 0; l < L; l++)
        for (int m = 0; m < L; m++) {
          const int r = i * L + l, r2 = j * L + m;
          d[(size_t)r * ds + r2] =
              i == j ? 0.f : P.d[((size_t)(i * P.lp + q.lev[l]) * P.n + j) * P.lp + q.lev[m]];
        }
  }
  {
    const double tl = (double)tlow * 0.5 * tseq;
    uint64_t b;
    std::memcpy(&b, &tl, 8);
    set_buckets(*dp, kBucketShift, (uint32_t)(b >> kBucketShift));
  }
  std::memcpy(B + dp->off_W, sp.W.data(), 8 * sp.W.size());
  std::memcpy(B + dp->off_trans, sp.trans.data(), 2 * sp.trans.size());
  // ---- work split: chunks c with c % count == rank ----
  dp->lo = q.lo;
  dp->hi = q.hi;
  dp->shard_count = q.count;
  dp->chunk_log2 = q.chunk_log2;
  dp->unit_log2 = std::min(kUnitLog2, q.chunk_log2);
  dp->n_owned = 0;
  dp->first_chunk = 0;
  if (q.hi > q.lo) {
    const uint64_t c0 = q.lo >> q.chunk_log2, c1 = (q.hi - 1) >> q.chunk_log2;
    const uint64_t R64 = (uint64_t)q.count;
    const uint64_t f = c0 + ((uint64_t)q.rank + R64 - c0 % R64) % R64;
    dp->first_chunk = f;
    dp->n_owned = f > c1 ? 0 : (c1 - f) / R64 + 1;
  }
  dp->n_units = dp->n_owned << (dp->chunk_log2 - dp->unit_log2);
  dp->unit_stride = 1;
  dp->cand_cap = q.cand_cap;
  dp->gtab_ok = ((uint64_t)L << n) * sizeof(GroupRec) <= ((uint64_t)384 << 20);
  {  // interleave lanes when partitions hold enough level vectors to keep lanes together
    double per = 1.0;
    const int nd = q.scope == SCHED_PER_CLIENT ? n : std::min(q.g, n);
    for (int k = 0; k < nd; k++) per *= L;
    dp->lane_strided = per >= 64.0;
  }
  return SCHED_OK;
}

// ------------------------------------------------------------ merge
int merge_picks(int n_ranks, int nw, const sched_pick *rank_best, const sched_pick *rank_pareto,
                const uint64_t *rank_np, sched_pick *best, sched_pick *pareto, uint64_t cap,
                uint64_t *np) {
  if (n_ranks < 1 || nw < 0 || nw > kMaxW) return SCHED_E_INVALID;
  if (nw > 0 && (!rank_best || !best)) return SCHED_E_INVALID;
  for (int w = 0; w < nw; w++) {
    sched_pick b;
    std::memset(&b, 0, sizeof b);
    for (int r = 0; r < n_ranks; r++) {
      const sched_pick &x = rank_best[(size_t)r * nw + w];
      if (!x.valid) continue;
      if (!b.valid || x.score64 > b.score64 || (x.score64 == b.score64 && x.index < b.index)) b = x;
    }
    best[w] = b;
  }
  std::vector<sched_pick> all;
  if (rank_np) {
    uint64_t off = 0;
    for (int r = 0; r < n_ranks; r++) {
      for (uint64_t k = 0; k < rank_np[r]; k++)
        if (rank_pareto[off + k].valid) all.push_back(rank_pareto[off + k]);
      off += rank_np[r];
    }
  }
  std::sort(all.begin(), all.end(), [](const sched_pick &x, const sched_pick &y) {
    if (x.makespan_s != y.makespan_s) return x.makespan_s < y.makespan_s;
    if (x.energy_j != y.energy_j) return x.energy_j < y.energy_j;
    return x.index < y.index;
  });
  std::vector<sched_pick> front;
  for (const auto &x : all)
    if (front.empty() || x.energy_j < front.back().energy_j) front.push_back(x);
  if (np) *np = front.size();
  if (front.size() > cap) return SCHED_E_CAPACITY;
  for (size_t k = 0; k < front.size(); k++) pareto[k] = front[k];
  return SCHED_OK;
}

}  // namespace sched
