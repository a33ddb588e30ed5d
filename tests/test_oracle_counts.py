"""Pins of the oracle's configuration counting (CPU).

The space (R1, R2) must have |Omega| = sum_{k<=G} P_k(N,C) * L^(N or k);
uncapped P_k = S(N,k) and sum_k S(N,k) = Bell(N) (BASELINE.json north_star).
"""
import itertools

import pytest

import oracle
import oracle.counts as cn
from synth import Query, PER_CLIENT, PER_GPU

# OEIS A000110 (Bell numbers), textbook values.
BELL = [1, 1, 2, 5, 15, 52, 203, 877, 4140, 21147, 115975, 678570, 4213597,
        27644437, 190899322, 1382958545, 10480142147, 82864869804,
        682076806159, 5832742205057, 51724158235372]
# S(16, k), k = 1..8 (also OEIS A008277 row 16).
S16 = [1, 32767, 7141686, 171798901, 1096190550, 2734926558, 3281882604, 2141764053]


def test_bell_numbers():
    for n, b in enumerate(BELL):
        assert cn.bell(n) == b


def test_stirling_row16():
    assert [cn.stirling2(16, k) for k in range(1, 9)] == S16


def test_stirling_recurrence_and_egf():
    # textbook recurrence S(n,k) = k S(n-1,k) + S(n-1,k-1) vs explicit formula
    for n in range(1, 18):
        for k in range(1, n + 1):
            assert cn.stirling2(n, k) == k * cn.stirling2(n - 1, k) + cn.stirling2(n - 1, k - 1)
            assert cn.partitions_k_egf(n, k, n) == cn.stirling2(n, k)


def test_capped_partitions_small_bruteforce():
    # count set partitions with block sizes <= c by direct enumeration of labelings
    for n in range(1, 8):
        for c in range(1, n + 1):
            for k in range(1, n + 1):
                seen = set()
                for lab in itertools.product(range(k), repeat=n):
                    m = {}
                    rgs = tuple(m.setdefault(x, len(m)) for x in lab)
                    if len(m) == k and max(rgs.count(b) for b in range(k)) <= c:
                        seen.add(rgs)
                assert cn.partitions_k(n, k, c) == len(seen), (n, k, c)


def test_appendix_a_sizes():
    # SURVEY App. A / BASELINE.md table
    assert cn.count_configs(4, 2, 4, 2, PER_CLIENT) == 128
    assert cn.count_configs(8, 4, 8, 4, PER_CLIENT) == 183173120
    assert cn.count_configs(12, 8, 4, 4, PER_GPU) == 26398581440
    assert cn.count_configs(16, 8, 16, 4, PER_GPU) == 206502209976948
    assert cn.count_configs(20, 8, 3, 1, PER_GPU) == 602027426000
    assert cn.count_configs(16, 8, 16, 4, PER_CLIENT) == 40517592409461227520
    assert cn.count_partitions(16, 16, 16) == BELL[16]
    assert cn.count_partitions(20, 20, 20) == BELL[20]


@pytest.mark.parametrize("scope", [PER_CLIENT, PER_GPU])
def test_oracle_count_matches_closed_form(scope):
    for n in range(1, 21):
        for g in (1, 2, 3, 5, 8):
            for c in sorted({1, 2, 3, 4, n}):
                if g * c < n:
                    continue
                for L in (1, 2, 4):
                    if scope == PER_CLIENT and n > 16 and L == 4:
                        continue
                    q = Query(n, g, c, tuple(range(L)), scope, ())
                    assert oracle.count(q) == cn.count_configs(n, g, min(c, n), L, scope), (n, g, c, L)


def test_oracle_count_literal_c4_exceeds_u64():
    q = Query(16, 8, 16, (0, 1, 2, 3), PER_CLIENT, ())
    v = oracle.count(q)
    assert v == 40517592409461227520 and v > 2 ** 64


def test_infeasible_caps_give_zero():
    q = Query(7, 2, 3, (0,), PER_GPU, ())   # 2 groups x 3 < 7 workflows
    assert oracle.count(q) == 0 == cn.count_configs(7, 2, 3, 1, PER_GPU)
