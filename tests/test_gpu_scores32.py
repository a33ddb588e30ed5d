"""The fp32 hot loop's score of EVERY configuration, not only of the picks
(VERDICT r1 weak 1(d)): sched_debug_scores32 runs the bench's tile kernel
over an index window and writes each configuration's (T/T_seq, E/E_seq) as
the tile loop computes them in fp32; the oracle's fp64 canonical (T, E) of
the same configurations (oracle.score_window) must agree within the north
star's 1e-5 relative -- and within the DESIGN.md section 5 bounds eps_T =
(3C+8) 2^-24, eps_E = (3C+N+G+16) 2^-24 that the exactness argument uses --
with memory-infeasible configurations on both sides the same."""
import random

import numpy as np
import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config, make_profile, requeue, Query, PER_GPU
from test_gpu_parity import _windows

pytestmark = pytest.mark.gpu

U = 2.0 ** -24


def _check_window(prof, q, lo, hi):
    qw = q.with_range(lo, hi)
    sch = S.Scheduler(prof)
    got = sch.debug_scores32(qw).cpu().numpy().astype(np.float64)
    T, E = oracle.score_window(prof, qw)
    ts, es = oracle.constants(prof, q)
    feas = ~np.isnan(T)
    assert np.array_equal(feas, ~np.isnan(got[:, 0])) and np.array_equal(feas, ~np.isnan(got[:, 1]))
    if not feas.any():
        return 0, 0.0, 0.0
    rt = np.abs(got[feas, 0] / (T[feas] / ts) - 1.0)
    re = np.abs(got[feas, 1] / (E[feas] / es) - 1.0)
    c = min(q.c, q.n)
    assert rt.max() <= min(1e-5, (3 * c + 8) * U), rt.max()
    assert re.max() <= min(1e-5, (3 * c + q.n + q.g + 16) * U), re.max()
    # the product metrics computed from them (X^a Y^b, a + b <= 3) stay within 1e-5 too
    x32, y32 = 1.0 / got[feas, 0], 1.0 / got[feas, 1]
    x64, y64 = ts / T[feas], es / E[feas]
    for a, b in ((1, 1), (2, 1), (1, 0), (0, 1)):
        assert np.abs((x32 ** a * y32 ** b) / (x64 ** a * y64 ** b) - 1).max() <= 1e-5
    return int(feas.sum()), float(rt.max()), float(re.max())


@pytest.mark.parametrize("name", ["c4", "c3", "mem_c4", "dup_c4"])
def test_every_configuration_fp32_within_bound(name):
    if name in ("c4", "c3"):
        prof, q = config(name)
    elif name == "mem_c4":
        _, q = config("c4")
        prof = make_profile(16, levels=(25, 50, 75, 100), seed=3, g=8, c=16,
                            archetypes=[11, 0, 3, 2, 5, 9, 1, 12, 3, 4, 2, 6, 0, 5, 7, 1])
    else:
        prof, q = config("c4")
        prof = requeue(prof, list(range(8)) * 2)
    q = Query(q.n, q.g, q.c, q.levels, PER_GPU, ((1, 1),), False)
    tot = S.count(q)
    rnd = random.Random(len(name))
    nf, mt, me = 0, 0.0, 0.0
    for lo, hi in _windows(tot, 1 << 24, rnd, 200_000):
        a, b, c = _check_window(prof, q, max(0, lo), min(tot, hi))
        nf, mt, me = nf + a, max(mt, b), max(me, c)
    print(f"{name}: {nf} feasible configurations, max rel err T {mt:.3g}, E {me:.3g}")
    assert nf > 0
