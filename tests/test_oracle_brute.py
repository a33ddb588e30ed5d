"""O1 (enum.c) pinned against O2 (brute force over all G^N labelings, N <= 6).

O2 defines the index order by sorting the canonicalised space and scores
with an independent pure-Python transcription; O1 must agree bitwise on
counts, best index / value per weight, and the Pareto set.  Windows of O1
must merge to the full result (the parallel oracle relies on it).
"""
import random

import pytest

import oracle
import oracle.brute as br
from synth import make_profile, Query, PER_CLIENT, PER_GPU

W = ((1, 0), (0, 1), (1, 1), (2, 1), (1, 2), (3, 1))

CASES = []
for n in range(1, 7):
    for g in (1, 2, 3, 4):
        for c in sorted({1, 2, n}):
            if g * c < n:
                continue
            for levels in ((100,), (50, 100), (25, 75, 100)):
                for scope in (PER_CLIENT, PER_GPU):
                    if scope == PER_CLIENT and len(levels) ** n > 256:
                        continue
                    CASES.append((n, g, c, levels, scope))


@pytest.mark.parametrize("n,g,c,levels,scope", CASES)
def test_enum_equals_bruteforce(n, g, c, levels, scope):
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=100 + n * 7 + g)
    q = Query(n, g, c, levels, scope, W, True)
    a = oracle.search(prof, q)
    b = br.search(prof, q)
    assert a["nconfigs"] == b["nconfigs"] == oracle.count(q)
    assert a["nfeasible"] == b["nfeasible"]
    assert a["best"] == b["best"]           # bitwise: (idx, F, T, E)
    assert a["pareto"] == b["pareto"]
    assert a["tseq"] == b["tseq"] and a["eseq"] == b["eseq"]


def test_enum_memory_infeasibility_matches():
    # WarpX (61453 MiB) cannot share with BerkeleyGW (30157 MiB) on 80 GiB
    # (PAPER.md L87 memory clause; Table II)
    prof = make_profile(5, levels=(50, 100), seed=3, archetypes=[11, 2, 0, 12, 5])
    q = Query(5, 3, 5, (50, 100), PER_GPU, W, True)
    a = oracle.search(prof, q)
    b = br.search(prof, q)
    assert a["nfeasible"] < a["nconfigs"]
    assert a["best"] == b["best"] and a["pareto"] == b["pareto"]
    for rgs, dig in b["space"]:
        ok, _, _ = br.score(prof, 5, rgs, [1] * 5)
        together = rgs[0] == rgs[1] or rgs[3] == rgs[1] or rgs[0] == rgs[3]
        assert ok == (not together)


def test_config_decode_matches_sorted_space():
    for (n, g, c, levels, scope) in [(5, 3, 2, (50, 100), PER_GPU), (4, 2, 4, (50, 100), PER_CLIENT),
                                     (6, 4, 3, (25, 75, 100), PER_GPU)]:
        q = Query(n, g, c, levels, scope, ())
        sp = br.space(n, g, c, len(levels), scope)
        for idx, (rgs, dig) in enumerate(sp):
            a, d = oracle.config(q, idx)
            assert tuple(a) == rgs and tuple(d) == dig


def test_windows_merge_to_full():
    rnd = random.Random(7)
    prof = make_profile(7, levels=(25, 50, 75, 100), seed=11)
    for scope, levels in ((PER_GPU, (25, 50, 75, 100)), (PER_CLIENT, (50, 100))):
        q = Query(7, 3, 4, levels, scope, W, True)
        full = oracle.search(prof, q)
        tot = oracle.count(q)
        cuts = sorted({0, tot} | {rnd.randrange(tot) for _ in range(9)})
        parts = [oracle.search(prof, q.with_range(a, b)) for a, b in zip(cuts, cuts[1:])]
        m = oracle.merge(parts)
        assert m["best"] == full["best"]
        assert m["pareto"] == full["pareto"]
        assert m["nconfigs"] == full["nconfigs"] == tot
