"""O3 (subset-DP certificate) pinned against O1 (full enumeration) on every
PER_GPU space small enough to enumerate: Pareto-front values and the
optimum of every weight must be bitwise equal.  The stored c3/c4/c5
certificates (tests/golden) must be reproducible from oracle/ alone."""
import json
import os

import pytest

import oracle
from synth import Query, config, make_profile, PER_GPU

W = ((1, 1), (2, 1), (1, 0), (0, 1), (1, 3))


@pytest.mark.parametrize("n,g,c,levels,seed", [
    (5, 2, 3, (50, 100), 1), (6, 3, 3, (25, 50, 100), 2), (7, 4, 7, (50, 100), 3),
    (8, 3, 3, (25, 50, 75, 100), 4), (9, 4, 4, (50, 100), 5), (8, 8, 8, (100,), 6),
    (9, 5, 2, (25, 100), 7), (10, 4, 3, (100,), 9),   # last: the c5 shape (L = 1, C = 3)
])
def test_certificate_equals_enumeration(n, g, c, levels, seed):
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed)
    q = Query(n, g, c, levels, PER_GPU, W, True)
    r = oracle.search(prof, q)
    cert = oracle.dp_certificate(prof, q)
    assert [(t, e) for _, t, e in r["pareto"]] == cert["front"]
    assert [b[1] for b in r["best"]] == cert["best"]


def test_certificate_handles_infeasible_groups():
    prof = make_profile(6, levels=(50, 100), seed=3, archetypes=[11, 2, 0, 12, 5, 1])
    q = Query(6, 3, 6, (50, 100), PER_GPU, W, True)
    r = oracle.search(prof, q)
    cert = oracle.dp_certificate(prof, q)
    assert r["nfeasible"] < r["nconfigs"]
    assert [(t, e) for _, t, e in r["pareto"]] == cert["front"]


@pytest.mark.parametrize("name", ["c3", "c4", "c5"])
def test_golden_certificates_reproduce(name):
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", f"{name}_certificate.json")))
    prof, q = config(name)
    cert = oracle.dp_certificate(prof, q)
    assert [[t.hex(), e.hex()] for t, e in cert["front"]] == g["front_T_E"]
    assert [b.hex() for b in cert["best"]] == g["best_score64"]


@pytest.mark.parametrize("n,g,c,levels,seed", [
    (5, 2, 3, (25, 50, 75, 100), 700), (6, 3, 3, (50, 100), 701), (7, 3, 7, (25, 50, 75, 100), 702),
    (6, 4, 2, (50, 100), 703), (5, 5, 5, (25, 50, 75, 100), 704), (6, 6, 6, (25, 50, 75, 100), 706),
    (8, 3, 3, (50, 100), 707),
])
def test_client_certificate_equals_enumeration(n, g, c, levels, seed):
    """O4 (PER_CLIENT subset DP over per-group level-vector fronts) == O1 full
    enumeration: front values and every weight's optimum, bitwise.  Catches:
    a level-vector order or member-level mix-up in the per-client group tuple,
    a dropped level vector, or pruning a vector that reaches the front."""
    from synth import PER_CLIENT
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed)
    q = Query(n, g, c, levels, PER_CLIENT, W, True)
    r = oracle.search(prof, q)
    cert = oracle.dp_certificate(prof, q)
    assert [(t, e) for _, t, e in r["pareto"]] == cert["front"]
    assert [b[1] if b else None for b in r["best"]] == cert["best"]


@pytest.mark.parametrize("n,c,levels,seed", [
    (7, 7, (25, 50, 75, 100), 710), (8, 4, (50, 100), 711), (6, 6, (25, 75, 100), 712), (9, 3, (100,), 713),
])
def test_client_fronts_batched_equals_plain(n, c, levels, seed):
    """O4 phase 1: the batched per-group fronts (last member's levels swept
    inside group_tuples_last, prefix sums shared) equal the plain form
    (every level vector through group_tuple_members) bitwise for every group,
    including groups made infeasible by memory (WarpX / BerkeleyGW rows)."""
    from synth import PER_CLIENT
    arch = [11, 2, 0, 12, 5, 1, 7, 9, 3][:n]
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed, archetypes=arch)
    q = Query(n, n, c, levels, PER_CLIENT, W, True)
    off0, t0, e0 = oracle._client_fronts((prof, q, 0, 1 << n, 0))
    off1, t1, e1 = oracle._client_fronts((prof, q, 0, 1 << n, 1))
    assert off0.tolist() == off1.tolist()
    assert t0.tobytes() == t1.tobytes() and e0.tobytes() == e1.tobytes()
    assert (off0[1:] == off0[:-1]).any()   # some group infeasible (memory)


def test_client_certificate_parallel_equals_serial():
    """The process-pool form of O4 (phase 1 split over group ranges) equals
    the one-process O4 bitwise."""
    from synth import PER_CLIENT
    prof = make_profile(9, levels=(25, 50, 75, 100), seed=720)
    q = Query(9, 4, 9, (50, 100), PER_CLIENT, W, True)
    a = oracle.dp_certificate(prof, q)
    b = oracle.dp_certificate(prof, q, procs=3)
    assert a["front"] == b["front"] and a["best"] == b["best"]


@pytest.mark.parametrize("n,g,c,seed", [(9, 5, 9, 730), (10, 4, 4, 731), (10, 8, 3, 732)])
def test_client_certificate_equals_enumeration_n9_n10(n, g, c, seed):
    """O4 == O1 (full enumeration, process pool) at the largest PER_CLIENT
    sizes the enumerator covers in seconds: n = 9, 10 with 2 levels per
    client (pin O4 beyond n = 8 before trusting it at n = 16)."""
    from synth import PER_CLIENT
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=seed)
    q = Query(n, g, c, (50, 100), PER_CLIENT, W, True)
    r = oracle.search_parallel(prof, q)
    cert = oracle.dp_certificate(prof, q, procs=2)
    assert [(t, e) for _, t, e in r["pareto"]] == cert["front"]
    assert [b[1] if b else None for b in r["best"]] == cert["best"]


def test_client_n16_certificate_consistent_with_per_gpu_certificate():
    """The literal per-client c4 certificate (O4, n = 16) against the PER_GPU
    c4 certificate (O3), two independent computations: every PER_GPU
    configuration is also a PER_CLIENT configuration (all clients of a group
    at the group's level), so every PER_GPU front point is weakly dominated
    by a per-client front point and every per-client optimum is >= the
    PER_GPU one.  Also: the stored baselines equal the oracle's constants."""
    g16 = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "c4_client_n16_certificate.json")))
    g4 = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "c4_certificate.json")))
    f16 = [(float.fromhex(t), float.fromhex(e)) for t, e in g16["front_T_E"]]
    f4 = [(float.fromhex(t), float.fromhex(e)) for t, e in g4["front_T_E"]]
    assert f16 == sorted(f16) and all(a[1] > b[1] for a, b in zip(f16, f16[1:]))   # a staircase
    for t, e in f4:
        assert any(t2 <= t and e2 <= e for t2, e2 in f16)
    w16 = [tuple(w) for w in g16["weights"]]
    for w, b in zip(g4["weights"], g4["best_score64"]):
        assert float.fromhex(g16["best_score64"][w16.index(tuple(w))]) >= float.fromhex(b)
    prof, q = config("c4")
    ts, es = oracle.constants(prof, q)
    assert g16["tseq"] == ts.hex() and g16["eseq"] == es.hex()
    # the optimum of each weight is attained on the stored front
    for (a, b), best in zip(w16, g16["best_score64"]):
        assert max(oracle.objective(ts, es, t, e, a, b) for t, e in f16) == float.fromhex(best)
