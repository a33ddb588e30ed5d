"""GPU parity of the scheduling-configuration search (sched_search_splits;
SURVEY 8(f) N3, R29) against oracle O5 (oracle/split.py): per
weight the fp64 score, split rank and index bitwise; the Pareto set as
(T, E, split rank, index) bitwise; configuration counts exactly."""
import pytest

import oracle
from oracle import split as O5
import paper_conf_sc_weaverkmeh0m24_b200 as S
from synth import make_profile, Query, PER_CLIENT, PER_GPU

pytestmark = pytest.mark.gpu

W = ((1, 0), (0, 1), (1, 1), (2, 1))
LAMMPS_4X, ATHENAPK_4X = 10, 1   # synth TABLE_II rows


def check(res, ref, q, tasks):
    rc, best, par, st, ns = res
    assert ns == len(ref["splits"])
    assert st["n_configs"] == ref["nconfigs"]
    assert (st["t_seq_s"], st["e_seq_j"]) == (ref["tseq"], ref["eseq"])
    for w in range(len(q.weights)):
        r = ref["best"][w]
        b = best[w]
        if r is None:
            assert not b.pick.valid
            continue
        assert b.pick.valid
        assert (b.pick.score64, b.split_rank, b.pick.index, b.pick.makespan_s, b.pick.energy_j) == \
            (r[0], r[1], r[2], r[3], r[4]), w
        assert tuple(b.split[i] for i in range(q.n)) == ref["splits"][r[1]]
        assert b.n_clients == sum(ref["splits"][r[1]])
    got = [(p.pick.makespan_s, p.pick.energy_j, p.split_rank, p.pick.index) for p in par]
    assert got == [tuple(x) for x in ref["pareto"]]


@pytest.mark.parametrize("n,tasks,g,c,levels,scope,seed", [
    (3, (4, 2, 2), 2, 4, (50, 100), PER_CLIENT, 0),
    (3, (2, 3, 1), 3, 3, (25, 50, 75, 100), PER_GPU, 1),
    (4, (2, 2, 2, 2), 4, 4, (25, 50, 75, 100), PER_GPU, 2),
    (2, (6, 4), 4, 16, (100,), PER_GPU, 3),
])
def test_splits_vs_oracle(n, tasks, g, c, levels, scope, seed):
    prof = make_profile(n, levels=(25, 50, 75, 100), seed=400 + seed)
    q = Query(n, g, c, levels, scope, W, True)
    check(S.Scheduler(prof).search_splits(q, tasks), O5.search_splits(prof, q, tasks), q, tasks)


def test_splits_cardinality_lammps_athenapk():
    """The paper's cardinality / scheduling-configuration experiment shape
    (LAMMPS and AthenaPK workflows, 4 tasks each, split
    '4-1', '2-2', '1-4'), on its 2 GPUs (L63), per-client MPS levels."""
    prof = make_profile(2, levels=(50, 100), seed=7, archetypes=[LAMMPS_4X, ATHENAPK_4X])
    q = Query(2, 2, 8, (50, 100), PER_CLIENT, W, True)
    check(S.Scheduler(prof).search_splits(q, (4, 4)), O5.search_splits(prof, q, (4, 4)), q, (4, 4))


@pytest.mark.parametrize("model", [1, 2, 4])
def test_splits_model_variants(model):
    prof = make_profile(3, levels=(50, 100), seed=11)
    q = Query(3, 2, 6, (50, 100), PER_GPU, W, True, model=model, power_cap=150.0)
    check(S.Scheduler(prof).search_splits(q, (2, 2, 3)), O5.search_splits(prof, q, (2, 2, 3)), q, (2, 2, 3))


def test_splits_max_split_and_all_ones():
    """max_split caps the split (all ones = the plain search, same indices)."""
    prof = make_profile(4, levels=(50, 100), seed=12)
    q = Query(4, 2, 4, (50, 100), PER_CLIENT, W, True)
    rc, best, par, st, ns = S.Scheduler(prof).search_splits(q, (4, 6, 2, 3), max_split=(1, 1, 1, 1))
    assert ns == 1
    ref = S.Scheduler(prof).search(q)
    assert [(b.pick.index, b.pick.score64) for b in best] == [(b.index, b.score64) for b in ref.best]
    assert [(p.pick.index, p.pick.makespan_s) for p in par] == [(p.index, p.makespan_s) for p in ref.pareto]
