"""bench.py's multi-GPU launcher on CPU: `--gpus 2` without torchrun
re-launches itself with two ranks (torch.distributed.run, gloo in the dry
run), every step's shards are exchanged and the coverage check passes
(BASELINE.json metric "at 1/2/4/8 B200")."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None):
    e = dict(os.environ)
    for k in ("RANK", "WORLD_SIZE", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        e.pop(k, None)
    e.update(env or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True,
                          text=True, env=e, timeout=300)


def test_gpus2_self_launches_two_ranks_with_coverage():
    r = _run(["--dry-run", "--gpus", "2", "--steps", "3", "--warmup", "1"])
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [json.loads(x) for x in r.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1                       # rank 0 prints one line
    line = lines[0]
    assert line["n_gpus"] == 2 and line["coverage"].startswith("ok: 3 steps, sum over 2 rank(s)")


def test_gpus1_dry_run_single_process():
    r = _run(["--dry-run", "--gpus", "1", "--steps", "2", "--warmup", "1"])
    assert r.returncode == 0, r.stderr[-2000:]
    assert json.loads(r.stdout.strip().splitlines()[-1])["n_gpus"] == 1


def test_world_size_must_match_gpus():
    r = _run(["--dry-run", "--gpus", "4"], env={"WORLD_SIZE": "2", "RANK": "0"})
    assert r.returncode == 2 and "WORLD_SIZE=2" in r.stderr
