"""Seeded randomized parity sweep over every fast kernel (parity
first): 160 cases mixing queue sizes, GPU counts, client caps, level sets,
level scopes, weight sets (compiled-in and run-time exponents, Pareto on /
off), the power-cap variant, index windows at random offsets and chunk sizes
that split partitions across units -- each result bitwise against the
oracle (test_gpu_parity.check).  The kernel path is whatever the library
picks; the test records that every fast path was exercised."""
import collections
import random

import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import make_profile, Query, PER_CLIENT, PER_GPU
from test_gpu_parity import check

pytestmark = pytest.mark.gpu

ALLW = [(1, 0), (0, 1), (1, 1), (2, 1), (1, 2), (3, 1), (1, 3), (4, 4), (2, 3), (0, 2)]


def _case(t):
    rnd = random.Random(7000 + t)
    kind = t % 4
    if kind == 0:     # PER_GPU, 4 levels: the tile kernel
        n, g = rnd.randint(6, 10), rnd.randint(5, 8)
        c, levels, scope = rnd.randint(2, n), (25, 50, 75, 100), PER_GPU
    elif kind == 1:   # PER_CLIENT, 4 levels, groups <= 4 clients: the group-table kernel
        n, g = rnd.randint(6, 9), rnd.randint(3, 8)
        c, levels, scope = rnd.randint(max(1, -(-n // g)), 4), (25, 50, 75, 100), PER_CLIENT
    elif kind == 2:   # one level: the suffix kernel
        n, g = rnd.randint(8, 12), rnd.randint(4, 8)
        c, levels, scope = rnd.randint(max(2, -(-n // g)), 4), (100,), PER_GPU
    else:             # anything: small mixed spaces
        n, g = rnd.randint(3, 8), rnd.randint(1, 6)
        c = rnd.randint(max(1, -(-n // g)), n)
        levels = tuple(sorted(rnd.sample((25, 50, 75, 100), rnd.randint(1, 4))))
        scope = rnd.choice((PER_GPU, PER_CLIENT))
    ws = tuple(rnd.sample(ALLW, rnd.randint(0, 6)))
    pareto = rnd.random() < 0.7 or not ws
    model = 4 if rnd.random() < 0.15 else 0
    arch = [rnd.choice((0, 1, 3, 5, 2, 11)) for _ in range(n)] if rnd.random() < 0.3 else None
    return t, n, g, c, levels, scope, ws, pareto, model, arch, rnd.randint(0, 1 << 30)


PATHS = collections.Counter()


@pytest.mark.parametrize("t", range(160))
def test_fuzz(t):
    t, n, g, c, levels, scope, ws, pareto, model, arch, r = _case(t)
    try:
        prof = make_profile(n, levels=(25, 50, 75, 100), seed=8000 + t, g=g, c=c, archetypes=arch)
    except RuntimeError:
        pytest.skip("no feasible profile for this archetype mix")
    q = Query(n, g, c, levels, scope, ws, pareto, model=model, power_cap=180.0)
    tot = S.count(q)
    rnd = random.Random(r)
    if tot > 3_000_000 or rnd.random() < 0.5:   # a window
        lo = rnd.randrange(max(1, tot - 1))
        q = q.with_range(lo, min(tot, lo + rnd.randint(1, 400_000)))
    cl = rnd.choice((12, 14, 16, 24))
    res = S.Scheduler(prof).search(q, chunk_log2=cl)
    PATHS[res.stats["kernel_path"]] += 1
    check(res, oracle.search(prof, q), q)


def test_fuzz_exercised_every_fast_path():
    if sum(PATHS.values()) < 100:
        pytest.skip("run together with test_fuzz")
    assert {1, 3, 6} <= set(PATHS), PATHS
