"""The NCCL leg of the multi-GPU layer on one GPU.

Every gpurun box has one B200, so the 2/4/8-rank NCCL runs happen only on the
driver's box; here the same code runs over a real NCCL process group of one
rank: bench.py under torch.distributed.run (--nproc-per-node 1: process
group, NCCL barrier / all_gather / all_reduce, per-step coverage check) and
dist.sharded_search + exchange against the oracle.
"""
import json
import os
import socket
import subprocess
import sys
import textwrap

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _env():
    e = dict(os.environ)
    for k in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT", "TORCHELASTIC_RUN_ID"):
        e.pop(k, None)
    e["NCCL_DEBUG"] = "INFO"
    return e


def test_bench_under_torchrun_one_rank_nccl():
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=1",
           "--master-addr", "127.0.0.1", f"--master-port={_port()}", os.path.join(ROOT, "bench.py"),
           "--gpus", "1", "--steps", "1", "--warmup", "3", "--no-cpu-baseline", "--no-secondary"]
    r = subprocess.run(cmd, capture_output=True, text=True, env=_env(), timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [json.loads(x) for x in r.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1
    line = lines[0]
    assert line["n_gpus"] == 1 and line["config"]["coverage"].startswith("ok: 1 steps")
    assert line["value"] > 1e12
    assert "NCCL INFO" in r.stdout + r.stderr      # the collectives really went through NCCL


_WORKER = textwrap.dedent("""
    import json, os, sys
    sys.path.insert(0, {root!r})
    import torch, torch.distributed as dist
    import oracle
    import paper_conf_sc_weaverkmeh0m24_b200 as S
    from paper_conf_sc_weaverkmeh0m24_b200 import dist as D
    from synth import Query, make_profile, PER_GPU
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method="tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    prof = make_profile(9, levels=(25, 50, 75, 100), seed=31)
    q = Query(9, 4, 4, (25, 50, 75, 100), PER_GPU, ((1, 1), (2, 1), (1, 0)), True)
    sch = S.Scheduler(prof)
    out = []
    for s_idx in range(3):                      # every slice of a 3-slice cut, then merged
        best, par, res, n_all = D.sharded_search(sch, q, chunk_log2=12, slices=(s_idx, 3))
        out.append(([(b.index, b.score64) if b.valid else None for b in best],
                    [(p.index, p.makespan_s, p.energy_j) for p in par], n_all))
    ref = oracle.search(prof, q)
    print(json.dumps({{"slices": out, "ref_best": [(b[0], b[1]) if b else None for b in ref["best"]],
                      "ref_pareto": ref["pareto"], "n": ref["nconfigs"],
                      "backend": dist.get_backend()}}))
    dist.destroy_process_group()
""")


def test_sharded_search_over_nccl_one_rank():
    import oracle
    import paper_conf_sc_weaverkmeh0m24_b200 as S
    from synth import Query, make_profile, PER_GPU
    code = _WORKER.format(root=ROOT, port=_port())
    r = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=_env(), timeout=600,
                       cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([x for x in r.stdout.splitlines() if x.startswith("{")][-1])
    assert d["backend"] == "nccl"
    assert sum(s[2] for s in d["slices"]) == d["n"]          # coverage over the three slices
    # merge the three slices' results exactly (sched_merge) and compare with the oracle
    from paper_conf_sc_weaverkmeh0m24_b200.sched import Pick
    prof = make_profile(9, levels=(25, 50, 75, 100), seed=31)
    q = Query(9, 4, 4, (25, 50, 75, 100), PER_GPU, ((1, 1), (2, 1), (1, 0)), True)
    ts, es = oracle.constants(prof, q)
    sl_best, sl_par = [], []
    for best, par, _ in d["slices"]:
        bl = []
        for b in best:
            p = Pick()
            if b is not None:
                p.valid, (p.index, p.score64) = 1, b
            bl.append(p)
        sl_best.append(bl)
        pl = []
        for idx, T, E in par:
            p = Pick()
            p.valid, p.index, p.makespan_s, p.energy_j = 1, idx, T, E
            pl.append(p)
        sl_par.append(pl)
    mb, mp = S.merge(sl_best, sl_par, len(q.weights))
    assert [(b.index, b.score64) for b in mb] == [tuple(x) for x in d["ref_best"]]
    assert [(p.index, p.makespan_s, p.energy_j) for p in mp] == [tuple(x) for x in d["ref_pareto"]]
