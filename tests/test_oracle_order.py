"""Index-order pins (reading R4: RGS lexicographic, then level digits MSB-first).

First / last configurations follow from the definition of lexicographic
order by hand (SURVEY 8(c) pins), independent of any counting code.
"""
import oracle
import oracle.counts as cn
from synth import CONFIGS


def _q(name):
    return CONFIGS[name]["query"]


def test_first_configs():
    q = _q("c3")   # C = 4: greedy fill of the lowest blocks
    a, d = oracle.config(q, 0)
    assert tuple(a) == (0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 2, 2) and d == [0, 0, 0]
    q = _q("c4")   # C >= N: everything in block 0, level digit 0
    a, d = oracle.config(q, 0)
    assert a == [0] * 16 and d == [0]
    a, d = oracle.config(q, 3)    # one block -> 4 level vectors, then next RGS
    assert a == [0] * 16 and d == [3]
    a, d = oracle.config(q, 4)
    assert a == [0] * 15 + [1] and d == [0, 0]


def test_last_configs():
    for name, rgs in (("c4", (0, 1, 2, 3, 4, 5, 6, 7) + (7,) * 8),
                      ("c3", (0, 1, 2, 3, 4, 5, 6, 7, 7, 7, 7, 6)),
                      ("c5", (0, 1, 2, 3, 4, 5, 6, 7, 7, 7, 6, 6, 5, 5, 4, 4, 3, 3, 2, 2))):
        q = _q(name)
        tot = cn.count_configs(q.n, q.g, min(q.c, q.n), len(q.levels), q.scope)
        a, d = oracle.config(q, tot - 1)
        assert tuple(a) == rgs
        assert all(x == len(q.levels) - 1 for x in d)


def test_c2_per_client_digits():
    q = _q("c2")   # PER_CLIENT, L = 4, N = 8: 4^8 level vectors per partition
    a, d = oracle.config(q, 4 ** 8 - 1)
    assert a == [0] * 8 and d == [3] * 8
    a, d = oracle.config(q, 4 ** 8 + 6)
    assert a == [0] * 7 + [1] and d == [0] * 6 + [1, 2]
