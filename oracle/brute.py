"""O2: brute force over all G^N GPU labelings (TEST INFRASTRUCTURE ONLY, N <= 6).

Independent of enum.c: the space is built by canonicalising every labeling
of the N workflows onto G GPUs (GPUs are interchangeable -> relabel blocks by
first occurrence, "groups ... on available GPUs"), the index
order is obtained by SORTING the distinct (RGS, level digits) tuples
(reading R4: RGS lexicographic, then digits most-significant first), and
each configuration is scored by a separate pure-Python fp64 transcription
of the canonical score (PAPER.md L87, L91, L96,
L116).  Python floats are IEEE binary64 with one rounding per operation.
"""
from __future__ import annotations

import itertools

PER_CLIENT = 0


def space(n, g, c, L, scope):
    """Sorted list of (rgs, digits) for the whole space."""
    rgss = set()
    for lab in itertools.product(range(g), repeat=n):
        m = {}
        rgs = tuple(m.setdefault(x, len(m)) for x in lab)
        k = len(m)
        sizes = [rgs.count(b) for b in range(k)]
        if max(sizes) <= c:
            rgss.add(rgs)
    out = []
    for rgs in sorted(rgss):
        k = max(rgs) + 1
        nd = n if scope == PER_CLIENT else k
        for dig in itertools.product(range(L), repeat=nd):
            out.append((rgs, dig))
    return out


COUNT_IDLE, NO_INTERFERENCE, POWER_CAP, TIME_SLICE = 1, 2, 4, 8   # scoring-model variants (R26-R28, R30)


def _capped(t, dyn, capd):
    """solo / group time under the power cap: max(t, dyn / (P_cap - P_s))"""
    tc = dyn / capd
    return tc if tc > t else t


def t_seq(t100, g, p100=None, ps=0.0, model=0, pcap=0.0):
    fin = [0.0] * g
    for i, ti in enumerate(t100):
        if model & POWER_CAP:
            ti = _capped(ti, (p100[i] - ps) * ti, pcap - ps)
        j = min(range(g), key=lambda x: (fin[x], x))
        fin[j] = fin[j] + ti
    return max(fin)


def e_seq(p100, t100, ps=0.0, model=0, pcap=0.0, g=1, ts=0.0):
    e = 0.0
    if model & COUNT_IDLE:
        for pi, ti in zip(p100, t100):
            e = e + (pi - ps) * ti
        return (g * ps) * ts + e
    for pi, ti in zip(p100, t100):
        ei = pi * ti
        if model & POWER_CAP:
            dyn = (pi - ps) * ti
            tc = _capped(ti, dyn, pcap - ps)
            if tc != ti:
                ei = ps * tc + dyn
        e = e + ei
    return e


def score(prof, n, rgs, lv_prof, model=0, pcap=0.0, g=1):
    """lv_prof[i]: profile level index of workflow i. -> (feasible, T, E)."""
    t = prof.solo_time_s.astype(float)
    p = prof.solo_power_w.astype(float)
    u = prof.sm_util.astype(float)
    bw = prof.bw_util.astype(float)
    d = prof.corun_slowdown.astype(float)
    ps = float(prof.static_power_w)
    k = max(rgs) + 1
    groups = [[i for i in range(n) if rgs[i] == b] for b in range(k)]
    for grp in groups:
        if sum(int(prof.max_mem_mib[i]) for i in grp) > int(prof.mem_capacity_mib):
            return False, None, None
    T = 0.0
    E = 0.0
    Dall = 0.0
    for grp in groups:
        U = 0.0
        B = 0.0
        for i in grp:
            U = U + u[i, lv_prof[i]]
            B = B + bw[i, lv_prof[i]]
        if model & NO_INTERFERENCE and (U > 1.0 or B > 1.0):
            return False, None, None
        cg = max(max(1.0, U), B)
        Tg = 0.0
        if model & TIME_SLICE:
            # R30: no MPS, the members take turns on the
            # whole GPU at their solo profile; each slice capped on its own
            for i in grp:
                ti = t[i, lv_prof[i]]
                if model & POWER_CAP:
                    ti = _capped(ti, (p[i, lv_prof[i]] - ps) * ti, float(pcap) - ps)
                Tg = Tg + ti
        else:
            for i in grp:
                s = 1.0
                for j in grp:
                    if j != i:
                        s = s + d[i, lv_prof[i], j, lv_prof[j]]
                tau = (t[i, lv_prof[i]] * s) * cg
                Tg = max(Tg, tau)
        D = 0.0
        for i in grp:
            D = D + (p[i, lv_prof[i]] - ps) * t[i, lv_prof[i]]
        if model & POWER_CAP and not model & TIME_SLICE:
            Tg = _capped(Tg, D, float(pcap) - ps)
        T = max(T, Tg)
        E = E + (ps * Tg + D)
        Dall = Dall + D
    if model & COUNT_IDLE:
        E = (g * ps) * T + Dall
    return True, T, E


def search(prof, q):
    pct = [int(x) for x in prof.level_pct]
    lev = [pct.index(v) for v in q.levels]
    l100 = pct.index(100)
    t100 = [float(prof.solo_time_s[i, l100]) for i in range(q.n)]
    p100 = [float(prof.solo_power_w[i, l100]) for i in range(q.n)]
    model = getattr(q, "model", 0)
    pcap = float(getattr(q, "power_cap", 0.0))
    ps = float(prof.static_power_w)
    ts = t_seq(t100, q.g, p100, ps, model, pcap)
    es = e_seq(p100, t100, ps, model, pcap, q.g, ts)
    sp = space(q.n, q.g, min(q.c, q.n), len(q.levels), q.scope)
    best = [None] * len(q.weights)
    feas = []
    for idx, (rgs, dig) in enumerate(sp):
        lvp = [lev[dig[i]] if q.scope == PER_CLIENT else lev[dig[rgs[i]]] for i in range(q.n)]
        ok, T, E = score(prof, q.n, rgs, lvp, model, pcap, q.g)
        if not ok:
            continue
        feas.append((idx, T, E))
        X = ts / T
        Y = es / E
        for w, (a, b) in enumerate(q.weights):
            F = 1.0
            for _ in range(a):
                F = F * X
            for _ in range(b):
                F = F * Y
            if best[w] is None or F > best[w][1]:
                best[w] = (idx, F, T, E)
    # Pareto by O(n^2) definition: not dominated by any feasible config;
    # one (lowest) index per distinct (T, E).
    pts = {}
    for idx, T, E in feas:
        dom = any((T2 <= T and E2 <= E) and (T2 < T or E2 < E) for _, T2, E2 in feas)
        if not dom and (T, E) not in pts:
            pts[(T, E)] = idx
    pareto = sorted([(i, T, E) for (T, E), i in pts.items()], key=lambda x: (x[1], x[2], x[0]))
    return dict(best=best, pareto=pareto, nconfigs=len(sp), nfeasible=len(feas),
                tseq=ts, eseq=es, space=sp)
