"""Closed-form configuration counts (TEST INFRASTRUCTURE ONLY).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may
import anything under oracle/.  This file shares no code with the CUDA path.

The configuration space (R1, R2; BASELINE.json north_star "Sigma
Stirling S(N,k), k <= G, x MPS-level combinations, and the Bell numbers"):
  * a set partition of the N queued workflows into k <= G unlabeled groups
    ("select groups of queued workflows to co-schedule on available GPUs",
    PAPER.md L87, Sec. IV-B), each group of size <= C (MPS client limit,
    PAPER.md L35, L92);
  * PER_CLIENT: one MPS level per workflow  -> L^N level vectors;
    PER_GPU:    one MPS level per group      -> L^k level vectors.

Closed forms, evaluated exactly with Python integers / Fractions:
  S(n,k) = (1/k!) sum_j (-1)^j C(k,j) (k-j)^n      (Stirling 2nd kind)
  Bell(n) = sum_k S(n,k)
  P_k(N,C) = N! [x^N] (sum_{s=1..C} x^s/s!)^k / k!   (EGF, capped block size)
"""
from __future__ import annotations

from fractions import Fraction
from math import comb, factorial

PER_CLIENT = 0
PER_GPU = 1


def stirling2(n: int, k: int) -> int:
    """Explicit inclusion-exclusion formula (no recursion)."""
    if n == 0 and k == 0:
        return 1
    if k == 0 or k > n:
        return 0
    s = sum((-1) ** j * comb(k, j) * (k - j) ** n for j in range(k + 1))
    assert s % factorial(k) == 0
    return s // factorial(k)


def bell(n: int) -> int:
    return sum(stirling2(n, k) for k in range(n + 1))


def _poly_pow_coeff(base: list, k: int, n: int) -> Fraction:
    """[x^n] (sum_i base[i] x^i)^k with Fraction coefficients."""
    res = [Fraction(0)] * (n + 1)
    res[0] = Fraction(1)
    for _ in range(k):
        nxt = [Fraction(0)] * (n + 1)
        for i, ri in enumerate(res):
            if ri == 0:
                continue
            for j, bj in enumerate(base):
                if i + j > n:
                    break
                if bj:
                    nxt[i + j] += ri * bj
        res = nxt
    return res[n]


def partitions_k(n: int, k: int, c: int) -> int:
    """Number of set partitions of n labelled items into exactly k blocks of size <= c."""
    if n == 0:
        return 1 if k == 0 else 0
    if c >= n:
        return stirling2(n, k)
    base = [Fraction(0)] + [Fraction(1, factorial(s)) for s in range(1, c + 1)]
    v = Fraction(factorial(n)) * _poly_pow_coeff(base, k, n) / factorial(k)
    assert v.denominator == 1
    return int(v)


def partitions_k_egf(n: int, k: int, c: int) -> int:
    """Same as partitions_k but always via the EGF (used to cross-check Stirling)."""
    if n == 0:
        return 1 if k == 0 else 0
    base = [Fraction(0)] + [Fraction(1, factorial(s)) for s in range(1, min(c, n) + 1)]
    v = Fraction(factorial(n)) * _poly_pow_coeff(base, k, n) / factorial(k)
    assert v.denominator == 1
    return int(v)


def count_configs(n: int, g: int, c: int, n_levels: int, scope: int) -> int:
    """|Omega(N, G, C, L, scope)| exactly."""
    tot = 0
    for k in range(1, min(g, n) + 1):
        pk = partitions_k(n, k, c)
        tot += pk * (n_levels ** n if scope == PER_CLIENT else n_levels ** k)
    return tot


def count_partitions(n: int, g: int, c: int) -> int:
    return sum(partitions_k(n, k, c) for k in range(1, min(g, n) + 1))
