"""The five BASELINE.json workloads (BJ:L7-L11) as query descriptions.

Input description only (no method arithmetic).  Readings for the unstated
parts (level scope, c3 levels, weights) are DESIGN.md R2, R3, R14.
"""
from __future__ import annotations

import dataclasses

PER_CLIENT = 0
PER_GPU = 1


@dataclasses.dataclass(frozen=True)
class Query:
    n: int
    g: int
    c: int
    levels: tuple            # searched MPS active-thread % (subset of the profile grid)
    scope: int               # PER_CLIENT | PER_GPU
    weights: tuple           # ((a, b), ...) exponents of X^a * Y^b
    want_pareto: bool = True
    index_lo: int = 0
    index_hi: int | None = None   # None = |Omega|
    model: int = 0                # scoring-model variant bits (R26-R28): 1 COUNT_IDLE,
    power_cap: float = 0.0        # 2 NO_INTERFERENCE, 4 POWER_CAP (P_cap in W), 8 TIME_SLICE (R30)
    tseq_base: float = 0.0        # > 0: sequential baselines supplied by the caller (the
    eseq_base: float = 0.0        # unsplit queue of a split search, R29)

    def with_range(self, lo, hi):
        return dataclasses.replace(self, index_lo=lo, index_hi=hi)


CONFIGS = {
    # BJ:L7  4 workflows, 2 GPUs, MPS levels {50,100}%
    "c1": dict(query=Query(4, 2, 4, (50, 100), PER_CLIENT,
                           ((1, 0), (0, 1), (1, 1), (2, 1)), True),
               profile=dict(n=4, levels=(50, 100), seed=0)),
    # BJ:L8  8 workflows, 4 GPUs, {25,50,75,100}%, throughput objective
    "c2": dict(query=Query(8, 4, 8, (25, 50, 75, 100), PER_CLIENT,
                           ((1, 0),), False),
               profile=dict(n=8, levels=(25, 50, 75, 100), seed=0)),
    # BJ:L9  12 workflows, 8 GPUs, <=4 clients/GPU, throughput+energy Pareto
    "c3": dict(query=Query(12, 8, 4, (25, 50, 75, 100), PER_GPU,
                           ((1, 1),), True),
               profile=dict(n=12, levels=(25, 50, 75, 100), seed=0)),
    # BJ:L10 16 workflows, 8 GPUs, 4 levels, full Pareto set, sharded 8xB200
    "c4": dict(query=Query(16, 8, 16, (25, 50, 75, 100), PER_GPU,
                           ((1, 1), (2, 1)), True),
               profile=dict(n=16, levels=(25, 50, 75, 100), seed=0)),
    # BJ:L11 20 workflows, 8 GPUs, <=3 clients/GPU, objective-weight sweep
    "c5": dict(query=Query(20, 8, 3, (100,), PER_GPU,
                           ((1, 0), (3, 1), (2, 1), (1, 1), (1, 2), (1, 3), (0, 1)),
                           True),
               profile=dict(n=20, levels=(100,), seed=0)),
}


def config(name: str):
    """(profile, query) for a named workload, seeded (graded seed 0)."""
    from .profiles import make_profile
    spec = CONFIGS[name]
    q = spec["query"]
    prof = make_profile(g=q.g, c=q.c, **spec["profile"])
    return prof, q
