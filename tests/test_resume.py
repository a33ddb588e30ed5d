"""Checkpoint / resume and coverage of long searches (resume.py).
CPU: the window search is played by the oracle (O1 on each index window),
so the checkpoint format, resume logic, exact merge (sched_merge, host
only) and coverage checks run without a GPU; the merged result must equal
the oracle's one-shot search bitwise.  GPU: the same with sched_search."""
import dataclasses

import pytest

import oracle
import paper_conf_sc_weaverkmeh0m24_b200 as S
from paper_conf_sc_weaverkmeh0m24_b200 import resume as R
from synth import make_profile, Query, PER_CLIENT, PER_GPU

W = ((1, 0), (0, 1), (1, 1), (2, 1))


class _Res:
    def __init__(self, best, pareto, stats):
        self.best, self.pareto, self.stats = best, pareto, stats


def _oracle_search_fn(prof, nw):
    def fn(qw):
        r = oracle.search(prof, qw)
        ts, es = r["tseq"], r["eseq"]
        best = []
        for b in r["best"]:
            p = S.Pick()
            if b:
                p.index, p.score64, p.makespan_s, p.energy_j = b[0], b[1], b[2], b[3]
                p.x64, p.y64, p.valid = ts / b[2], es / b[3], 1
            best.append(p)
        par = []
        for idx, t, e in r["pareto"]:
            p = S.Pick()
            p.index, p.makespan_s, p.energy_j, p.x64, p.y64, p.valid = idx, t, e, ts / t, es / e, 1
            par.append(p)
        return _Res(best, par, {"n_configs": r["nconfigs"], "n_feasible": r["nfeasible"]})
    return fn


def _case():
    prof = make_profile(6, levels=(25, 50, 75, 100), seed=11)
    return prof, Query(6, 3, 6, (50, 100), PER_CLIENT, W, True)


def _same(out, ref):
    best, par, st = out
    assert [b.index if b.valid else None for b in best] == [b[0] if b else None for b in ref["best"]]
    assert [b.score64 for b in best if b.valid] == [b[1] for b in ref["best"] if b]
    assert [(p.index, p.makespan_s, p.energy_j) for p in par] == ref["pareto"]
    assert st["n_configs"] == ref["nconfigs"] and st["n_feasible"] == ref["nfeasible"]


def test_windows_tile_the_space():
    for total, n, a in [(128, 5, 1), (10 ** 9, 64, 1 << 22), (7, 64, 4), (1 << 22, 3, 1 << 22)]:
        ws = R.windows_of(total, n, a)
        assert ws[0][0] == 0 and ws[-1][1] == total
        assert all(w[1] == v[0] for w, v in zip(ws, ws[1:]))
        assert all(lo % a == 0 for lo, _ in ws)


def test_interrupted_then_resumed_equals_one_shot(tmp_path):
    prof, q = _case()
    ck = str(tmp_path / "ck.jsonl")
    fn = _oracle_search_fn(prof, len(q.weights))
    assert R.search_resumable(None, prof, q, ck, n_windows=9, align=64, max_windows=3, search_fn=fn) is None
    calls = []
    out = R.search_resumable(None, prof, q, ck, n_windows=9, align=64,
                             search_fn=lambda qw: calls.append(qw.index_lo) or fn(qw))
    assert out[2]["resumed"] == 3 and out[2]["windows"] == 9 and len(calls) == 6
    _same(out, oracle.search(prof, q))
    # a third run finds everything in the checkpoint: no search at all
    out2 = R.search_resumable(None, prof, q, ck, n_windows=9, align=64, search_fn=lambda qw: 1 / 0)
    _same(out2, oracle.search(prof, q))


def test_torn_line_and_other_search_ignored(tmp_path):
    prof, q = _case()
    ck = tmp_path / "ck.jsonl"
    fn = _oracle_search_fn(prof, len(q.weights))
    R.search_resumable(None, prof, q, str(ck), n_windows=4, align=64, max_windows=2, search_fn=fn)
    q2 = dataclasses.replace(q, weights=((1, 1),))       # another search in the same file
    R.search_resumable(None, prof, q2, str(ck), n_windows=4, align=64, max_windows=1,
                       search_fn=_oracle_search_fn(prof, 1))
    with open(ck, "a") as f:
        f.write('{"fp": "' + R.fingerprint(prof, q) + '", "lo": 0, "hi"')   # torn write
    out = R.search_resumable(None, prof, q, str(ck), n_windows=4, align=64, search_fn=fn)
    assert out[2]["resumed"] == 2
    _same(out, oracle.search(prof, q))


def test_changed_window_split_not_counted_as_resumed(tmp_path):
    """Records of another window split (n_windows / align changed between
    runs) are neither merged nor counted as resumed, and a warning names them."""
    prof, q = _case()
    ck = str(tmp_path / "ck.jsonl")
    fn = _oracle_search_fn(prof, len(q.weights))
    R.search_resumable(None, prof, q, ck, n_windows=4, align=64, max_windows=2, search_fn=fn)
    with pytest.warns(RuntimeWarning, match="another window split"):
        out = R.search_resumable(None, prof, q, ck, n_windows=7, align=32, search_fn=fn)
    assert out[2]["resumed"] == 0 and out[2]["stale"] == 2
    _same(out, oracle.search(prof, q))


def test_truncated_window_raises_coverage_error(tmp_path):
    """Fault injection: a window search that silently scores fewer
    configurations than its range must not produce an 'optimum'."""
    prof, q = _case()
    fn = _oracle_search_fn(prof, len(q.weights))
    second = R.windows_of(S.count(q), 5, 64)[1][0]
    bad = lambda qw: fn(qw.with_range(qw.index_lo, qw.index_hi - 1)) if qw.index_lo == second else fn(qw)  # noqa: E731
    with pytest.raises(R.CoverageError):
        R.search_resumable(None, prof, q, str(tmp_path / "ck.jsonl"), n_windows=5, align=64, search_fn=bad)


def test_fingerprint_separates_profiles_and_queries():
    prof, q = _case()
    f0 = R.fingerprint(prof, q)
    assert f0 == R.fingerprint(prof, q.with_range(5, 9))             # the window is not part of it
    assert f0 != R.fingerprint(prof, dataclasses.replace(q, g=2))
    p2 = make_profile(6, levels=(25, 50, 75, 100), seed=12)
    assert f0 != R.fingerprint(p2, q)


@pytest.mark.gpu
def test_gpu_resumed_search_equals_one_shot(tmp_path):
    prof = make_profile(9, levels=(25, 50, 75, 100), seed=42)
    q = Query(9, 6, 3, (25, 50, 75, 100), PER_GPU, ((1, 1), (2, 1)), True)
    sch = S.Scheduler(prof)
    ck = str(tmp_path / "ck.jsonl")
    assert R.search_resumable(sch, prof, q, ck, n_windows=7, max_windows=2, align=1 << 20) is None
    best, par, st = R.search_resumable(sch, prof, q, ck, n_windows=7, align=1 << 20)
    one = sch.search(q)
    assert st["resumed"] == 2 and st["n_configs"] == one.stats["n_configs"]
    assert [b.index for b in best] == one.best_indices and [b.score64 for b in best] == [b.score64 for b in one.best]
    assert [(p.index, p.makespan_s, p.energy_j) for p in par] == [(p.index, p.makespan_s, p.energy_j) for p in one.pareto]
