"""GPU parity of the scoring-model variants (include/sched.h SCHED_MODEL_*,
DESIGN.md R26 COUNT_IDLE, R27 NO_INTERFERENCE, R28 POWER_CAP, R30
TIME_SLICE) on every
kernel path that accepts them, against the oracle (same bar as
test_gpu_parity.check: bitwise picks, Pareto set and counts)."""
import dataclasses
import random

import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import config, make_profile, Query, PER_CLIENT, PER_GPU
from test_gpu_parity import check

pytestmark = pytest.mark.gpu

W = ((1, 0), (0, 1), (1, 1), (2, 1))
MODELS = [1, 2, 4, 3, 5, 6, 7, 8, 9, 12, 13]


@pytest.mark.parametrize("model", MODELS)
@pytest.mark.parametrize("seed", range(3))
def test_variants_small_generic_and_auto(model, seed, monkeypatch):
    """Small PER_CLIENT / PER_GPU spaces (L = 2..4): the default path choice
    and the generic kernel must both equal the oracle."""
    rnd = random.Random(1000 * model + seed)
    n = rnd.randint(4, 7)
    g = rnd.randint(2, 4)
    levels = (50, 100) if seed % 2 else (25, 50, 75, 100)
    scope = PER_CLIENT if (seed == 0 and len(levels) ** n <= 4096) else PER_GPU
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=300 + seed)
    q = Query(n, g, n, levels, scope, W, True, model=model, power_cap=150.0)
    ref = oracle.search(prof, q)
    check(S.Scheduler(prof).search(q), ref, q)
    monkeypatch.setenv("SCHED_KERNEL", "generic")
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == 0
    check(res, ref, q)


@pytest.mark.parametrize("model", [2, 4, 6, 8, 12])
@pytest.mark.parametrize("kernel,path", [("sfx", 3), ("dfs", 2)])
def test_variants_partition_kernels(model, kernel, path, monkeypatch):
    """L = 1: NO_INTERFERENCE / POWER_CAP / TIME_SLICE enter through the
    group table on the suffix and pair kernels."""
    monkeypatch.setenv("SCHED_KERNEL", kernel)
    prof = make_profile(10, levels=(100,), seed=41, g=5, c=3)
    sweep = ((1, 0), (3, 1), (2, 1), (1, 1), (1, 2), (1, 3), (0, 1))   # a weight set the pair kernel is built for
    q = Query(10, 5, 3, (100,), PER_GPU, sweep, True, model=model, power_cap=140.0)
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == path
    check(res, oracle.search(prof, q), q)


@pytest.mark.parametrize("model", [4, 8, 12])
def test_power_cap_tile_kernel(model, monkeypatch):
    """POWER_CAP / TIME_SLICE on the PER_GPU L = 4 tile kernel (group-local,
    through the group table)."""
    monkeypatch.setenv("SCHED_KERNEL", "tile")
    prof = make_profile(9, levels=(25, 50, 75, 100), seed=42)
    q = Query(9, 6, 3, (25, 50, 75, 100), PER_GPU, ((1, 1), (2, 1)), True, model=model, power_cap=130.0)
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == 1
    check(res, oracle.search(prof, q), q)


@pytest.mark.parametrize("name,model", [("c4", 4), ("c5", 6), ("c3", 1), ("c2", 2), ("c4", 8), ("c2", 12), ("c5", 8), ("c3", 12)])
def test_variants_big_windows(name, model):
    """Windows of the BASELINE workloads under a variant (P_cap = 300 W, the
    paper's A100X cap), in the default launch configuration."""
    prof, q = config(name)
    q = dataclasses.replace(q, model=model, power_cap=300.0 if name != "c5" else 200.0)
    tot = S.count(q)
    sch = S.Scheduler(prof)
    rnd = random.Random(3)
    for lo in [0, tot - 50_000] + [rnd.randrange(tot - 50_000) for _ in range(2)]:
        qw = q.with_range(lo, lo + 50_000)
        check(sch.search(qw), oracle.search(prof, qw), qw)


@pytest.mark.parametrize("model", [1, 5, 9, 13])
@pytest.mark.parametrize("levels", [(25, 50, 75, 100), (50, 75, 100)])
def test_count_idle_tile_kernel(model, levels):
    """COUNT_IDLE (R26: every GPU draws P_s for the whole makespan, E = G P_s T
    + sum D_g) and its combinations with POWER_CAP / TIME_SLICE on the PER_GPU
    tile kernel (round 2: the group records carry D_g, the kernel adds the
    idle term per configuration and to every tile corner): small full spaces
    and c4 windows, bitwise against the oracle."""
    prof = make_profile(9, levels=(25, 50, 75, 100), seed=43)
    q = Query(9, 6, 4, levels, PER_GPU, ((1, 1), (2, 1), (1, 0), (0, 1)), True, model=model, power_cap=130.0)
    res = S.Scheduler(prof).search(q)
    assert res.stats["kernel_path"] == 1
    check(res, oracle.search(prof, q), q)
    prof4, q4 = config("c4")
    q4 = dataclasses.replace(q4, levels=levels, model=model, power_cap=300.0)
    tot = S.count(q4)
    sch = S.Scheduler(prof4)
    rnd = random.Random(model)
    for lo in [0, tot - 100_000, (1 << 24) - 50_000] + [rnd.randrange(tot - 100_000) for _ in range(2)]:
        qw = q4.with_range(lo, lo + 100_000)
        r = sch.search(qw)
        assert r.stats["kernel_path"] == 1
        check(r, oracle.search(prof4, qw), qw)
