#!/usr/bin/env python
"""Benchmark: exhaustive co-scheduling configuration search on B200.

  python bench.py [--gpus N --steps K --warmup W] [--impl ours|reference] [--full]

Workload (BASELINE.json configs[3], BJ:L10): c4 = 16 workflows x 8 GPUs x 4
MPS levels {25,50,75,100}% (PER_GPU, R2), objectives [TxE],
[TxTxE] + full Pareto set.  The 2.065e14-configuration index space is cut
into 64 cyclic slices of 2^24-index chunks; one step = one slice (1/64 of the
space) split over the N ranks (strong scaling), including the NCCL exchange
and exact merge.  64 steps are the complete search (`--full` runs them all).
After the timed region the configurations scored by all ranks are checked
against each step's slice (coverage).

Multi-GPU: `--gpus N` (N > 1) started without torchrun re-launches itself
under `torch.distributed.run --nproc-per-node N` (one rank per GPU, NCCL);
started under torchrun, WORLD_SIZE must equal N, and the process group (and
the NCCL exchange) is used even at one rank.  `--dry-run` runs the same
rank / exchange / coverage plumbing on CPU (gloo) with a stub in place of the
kernels (no scoring) -- the CPU test of the launcher.

One JSON line on rank 0 (driver contract).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "configurations scored/sec (whole box) at 1/2/4/8 B200; time-to-optimal-schedule"
UNIT = "configs/s"
SLICES = 64
CHUNK_LOG2 = 24   # 2^24-index chunks: tools/chunk_sweep.py (c4 step 669.8 -> 653.0 ms vs 2^22)
DP_WARM = 5        # warm sched_front_dp calls after the cold one (time-to-optimal)
OPS_PER_CONFIG = 4   # T max, E add, 2 min-reductions (c4 tile kernel, per configuration)
SMS = 148
LANES_PER_SM_CLK = 4 * 32   # 4 SMSPs x 32 lanes issue slots per clock


def env():
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return None
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        rows = []
        for line in open(self.f.name):
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 9:
                continue
            try:
                rows.append((float(parts[1]), float(parts[2]), parts[5:9], parts[4]))
            except ValueError:
                continue
        os.unlink(self.f.name)
        if not rows:
            return None
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i, v in enumerate(r[2]) if v.lower() == "active"})
        load = [r[0] for r in rows] or [0.0]
        return {"sm_mhz": statistics.median(load), "sm_max_mhz": max(r[1] for r in rows),
                "samples": len(rows), "reasons": reasons}


def cpu_baseline(prof, q, seed=0, per_window=1_500_000, windows_per_core=2):
    """The oracle as it stands, on host cores, over a bounded random sample of
    index windows of the same workload."""
    import random
    import oracle
    from concurrent.futures import ProcessPoolExecutor
    cores = os.cpu_count() or 1
    tot = oracle.count(q)
    rnd = random.Random(seed)
    los = sorted(rnd.randrange(tot - per_window) for _ in range(cores * windows_per_core))
    qs = [q.with_range(lo, lo + per_window) for lo in los]
    t0 = time.perf_counter()
    with ProcessPoolExecutor(cores) as ex:
        parts = list(ex.map(oracle._search_star, [(prof, x, 1 << 16) for x in qs]))
    dt = time.perf_counter() - t0
    n = sum(p["nconfigs"] for p in parts)
    return {"value": n / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{len(qs)} random index windows x {per_window} configs of the same workload "
                      f"({n} configs, fp64 recursive enumerator oracle/enum.c, {dt:.1f} s wall)"}


def run_reference(args):
    """--impl reference: the oracle timed as the reference arm (rank 0 only)."""
    rank, world, _ = env()
    if rank != 0:
        return 0
    import random
    import oracle
    from concurrent.futures import ProcessPoolExecutor
    from synth import config
    prof, q = config(args.workload)
    cores = os.cpu_count() or 1
    tot = oracle.count(q)
    per = args.ref_window

    def step_windows(sigma):
        rnd = random.Random(1000 + sigma)
        nchunks = tot >> CHUNK_LOG2
        out = []
        for _ in range(cores):
            c = rnd.randrange(nchunks // SLICES) * SLICES + sigma % SLICES
            lo = (c << CHUNK_LOG2) + rnd.randrange((1 << CHUNK_LOG2) - per)
            out.append(q.with_range(lo, lo + per))
        return out

    with ProcessPoolExecutor(cores) as ex:
        def step(sigma):
            parts = list(ex.map(oracle._search_star, [(prof, x, 1 << 16) for x in step_windows(sigma)]))
            return sum(p["nconfigs"] for p in parts)
        for i in range(args.warmup):
            step(i)
        t0 = time.perf_counter()
        n = 0
        for i in range(args.steps):
            n += step(args.warmup + i)
        dt = time.perf_counter() - t0
    v = n / dt
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": f"{args.workload} (bounded sample per step: {cores} windows x {per} "
                                   f"configs of the step's chunk slice)", "slices": SLICES,
                       "chunk_log2": CHUNK_LOG2},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
                             "sample": f"{cores} windows x {per} configs per step"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def check_steps(step_cfg, first_sigma, space, world, dev):
    """Coverage: per timed step, the configurations scored by all ranks equal
    the index count of that step's slice (dist.check_coverage raises)."""
    import torch
    from paper_conf_sc_weaverkmeh0m24_b200.dist import check_coverage
    import torch.distributed as dist
    t = torch.tensor(step_cfg, dtype=torch.int64, device=dev)
    if dist.is_available() and dist.is_initialized():
        dist.all_reduce(t)
    for i, n in enumerate(t.tolist()):
        check_coverage(n, 0, space, CHUNK_LOG2, (first_sigma + i) % SLICES, SLICES, world)
    return f"ok: {len(step_cfg)} steps, sum over {world} rank(s) == slice index count"


def free_port():
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch(args):
    """--gpus N > 1 without torchrun: one rank per GPU under torch.distributed.run."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={free_port()}", os.path.abspath(__file__),
           *sys.argv[1:]]
    return subprocess.call(cmd)


def run_dry(args):
    """CPU (gloo) run of the multi-rank plumbing: rank/world from the launcher,
    per-rank shard of each step (a stub stands in for sched_search: it
    reports the shard's index count and no picks), exchange + merge, and the
    coverage check.  Tests the launcher without a GPU (no scoring happens)."""
    import torch.distributed as dist
    import paper_conf_sc_weaverkmeh0m24_b200 as S
    from paper_conf_sc_weaverkmeh0m24_b200.dist import exchange, slice_index_count
    from synth import config
    rank, world, _ = env()
    if world > 1:
        dist.init_process_group("gloo")
    _, q = config(args.workload)
    space = S.count(q)
    nw = len(q.weights)
    cfg = []
    for i in range(args.warmup + args.steps):
        sh = ((i % SLICES) * world + rank, SLICES * world)
        n = slice_index_count(0, space, CHUNK_LOG2, sh[0], sh[1])   # stub: the shard's count
        if world > 1:
            exchange([S.Pick() for _ in range(nw)], [], nw)
        if i >= args.warmup:
            cfg.append(n)
    coverage = check_steps(cfg, args.warmup, space, world, "cpu")
    if rank == 0:
        print(json.dumps({"dry_run": True, "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                          "workload": args.workload, "space_configs": space, "coverage": coverage,
                          "configs_per_step": sum(cfg) * world // max(1, len(cfg))}), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def secondary(S):
    """The other kernels on their BASELINE workloads, one device-timed search
    each after a warm-up (context for the headline, not the headline):
    the literal per-client c3 ("c3-client", 1/64 chunk slice; kernel_path 6)
    and the whole c5 space (7-weight sweep + Pareto; kernel_path 3)."""
    from synth import config, Query
    out = []
    prof3, q3 = config("c3")
    qc = Query(q3.n, q3.g, q3.c, q3.levels, 0, q3.weights, q3.want_pareto)
    prof5, q5 = config("c5")
    for name, prof, q, kw in (("c3-client (PER_CLIENT c3, 5.5e13 configs), 1/64 slice", prof3, qc,
                               {"shard": (5, 64), "chunk_log2": CHUNK_LOG2}),
                              ("c5 whole space (7-weight sweep + Pareto)", prof5, q5, {})):
        sch = S.Scheduler(prof)
        sch.search(q, **kw)
        r = sch.search(q, **kw)
        st = r.stats
        out.append({"workload": name, "configs": st["n_configs"], "search_ms": st["search_ms"],
                    "configs_per_s": st["n_configs"] / (st["search_ms"] / 1e3), "kernel_path": st["kernel_path"],
                    "feasible_fraction": st["n_feasible"] / max(1, st["n_configs"])})
        sch.close()
    # time-to-optimal of the literal per-client c4 (4.05e19 configurations: no
    # enumeration reaches it) by the device subset DP, warm
    prof4, q4 = config("c4")
    qc4 = Query(q4.n, q4.g, q4.c, q4.levels, 0, q4.weights, q4.want_pareto)
    sch = S.Scheduler(prof4)
    ws = sch.dp_workspace(qc4)
    sch.front_dp(qc4, workspace=ws)
    t0 = time.perf_counter()
    rc, best, front, st = sch.front_dp(qc4, workspace=ws)
    out.append({"workload": "c4 literal per-client (4.05e19 configurations), subset DP (time-to-optimal)",
                "wall_s": time.perf_counter() - t0, "device_ms": st["total_ms"], "front_points": len(front),
                "best_score64": [b.score64 for b in best], "kernel_path": st["kernel_path"]})
    sch.close()
    return out


def describe(name, q):
    """The workload's one-line description (BASELINE.json configs, synth/configs.py)."""
    idx = {"c1": 0, "c2": 1, "c3": 2, "c4": 3, "c5": 4}.get(name)
    w = ",".join("[" + "x".join(["T"] * a + ["E"] * b) + "]" for a, b in q.weights)
    lv = "{" + ",".join(str(x) for x in q.levels) + "}%"
    return (f"{name}: {q.n} workflows x {q.g} GPUs, <= {q.c} clients per GPU, MPS levels {lv} "
            f"{'PER_GPU' if q.scope == 1 else 'PER_CLIENT'}, objectives {w}"
            f"{' + Pareto' if q.want_pareto else ''}"
            + (f" (BASELINE configs[{idx}])" if idx is not None else ""))


def run_ours(args):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_weaverkmeh0m24_b200 as S
    from paper_conf_sc_weaverkmeh0m24_b200.dist import exchange
    from synth import config

    rank, world, local = env()
    # a process group whenever the launcher is torchrun (also at one rank:
    # `torchrun --nproc-per-node 1` exercises the NCCL exchange on one GPU)
    pg = world > 1 or "TORCHELASTIC_RUN_ID" in os.environ
    assert torch.cuda.is_available(), "bench.py needs a CUDA device"
    # BENCH_SHARE_GPU=1 (tests only): every rank uses cuda:0 with a gloo group,
    # to exercise the N > 1 path on a one-GPU box; NCCL otherwise.
    share = os.environ.get("BENCH_SHARE_GPU") == "1"
    local = 0 if share else local
    torch.cuda.set_device(local)
    if pg:
        if share:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    prof, q = config(args.workload)
    nw = len(q.weights)
    space = S.count(q)
    sched = S.Scheduler(prof)
    ws = sched.workspace(q)
    sched.stage(q, workspace=ws)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()

    def barrier():
        torch.cuda.synchronize()
        if pg:
            dist.barrier()
        torch.cuda.synchronize()

    def step(sigma, sch=sched, workspace=ws):
        res = sch.search(q, workspace=workspace, shard=((sigma % SLICES) * world + rank, SLICES * world),
                         chunk_log2=CHUNK_LOG2)
        if pg:
            best, par, _ = exchange(res.best, res.pareto, nw)
        else:
            best, par = res.best, res.pareto
        return res, best, par

    if args.full:
        return run_full(args, step, barrier, rank, world, space, nw)

    for i in range(args.warmup):
        step(i)
        flush.zero_()
    clocks = Clocks(local)
    barrier()
    clocks.start()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    ncfg = 0
    search_ms = 0.0
    main_ms = 0.0
    launches = 0
    refined = 0
    step_cfg = []
    nfeas = 0
    for i in range(args.steps):
        res, _, _ = step(args.warmup + i)
        step_cfg.append(res.stats["n_configs"])
        ncfg += res.stats["n_configs"]
        search_ms += res.stats["search_ms"]
        main_ms += res.stats["main_ms"]
        launches += res.stats["kernel_launches"]
        refined += res.stats["n_refined"]
        nfeas += res.stats["n_feasible"]
        flush.zero_()
    ev1.record(stream)
    barrier()
    clk = clocks.stop()
    elapsed = ev0.elapsed_time(ev1)
    rdev = "cpu" if share else "cuda"
    if pg:
        t = torch.tensor([elapsed, float(ncfg)], dtype=torch.float64, device=rdev)
        mx = t.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        elapsed_max, ncfg_all = float(mx[0]), int(t[1])
    else:
        elapsed_max, ncfg_all = elapsed, ncfg
    value = ncfg_all / (elapsed_max / 1e3)
    ms_per_step = elapsed_max / args.steps
    coverage = check_steps(step_cfg, args.warmup, space, world, rdev)

    # ---- end to end through the public API with host buffers ----
    e2e_steps = max(1, min(args.steps, 3))
    barrier()
    t0 = time.perf_counter()
    e_cfg = 0
    h2d = d2h = 0
    for i in range(e2e_steps):
        fresh = S.Scheduler(prof)            # host profile -> handle; search re-stages (H2D)
        res, best, par = step(args.warmup + args.steps + i, sch=fresh)
        e_cfg += res.stats["n_configs"]
        h2d += res.stats["h2d_bytes"]
        d2h += res.stats["d2h_bytes"]
        fresh.close()
    barrier()
    e_dt = time.perf_counter() - t0
    if pg:
        t = torch.tensor([e_dt, float(e_cfg)], dtype=torch.float64, device=rdev)
        mx = t.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        e_dt, e_cfg = float(mx[0]), int(t[1])
    e2e = {"value": e_cfg / e_dt, "unit": UNIT, "h2d_bytes_per_step": h2d // e2e_steps,
           "d2h_bytes_per_step": d2h // e2e_steps, "steps": e2e_steps,
           "note": "fresh handle per step: host profile copy, H2D staging from pinned memory, "
                   "kernels, D2H of counters/picks, NCCL exchange + merge; host wall clock"}

    if rank != 0:
        dist.destroy_process_group() if pg else None
        return 0
    # time-to-optimal-schedule of the same space by the device subset DP
    # (sched_front_dp): exact front + optimum per weight.
    # One cold call (first launch of the DP kernels in this process: lazy
    # module load included) and DP_WARM warm calls on a reused workspace.
    dp_runs = []
    dp_ws = None
    for i in range(1 + DP_WARM):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        rc_dp, best_dp, front_dp, st_dp = sched.front_dp(q, workspace=dp_ws)
        torch.cuda.synchronize()
        dp_runs.append((time.perf_counter() - t0, st_dp["total_ms"]))
        if dp_ws is None:
            dp_ws = sched.dp_workspace(q)
    warm = dp_runs[1:]
    dp = {"cold_wall_s": dp_runs[0][0], "cold_device_ms": dp_runs[0][1],
          "warm_wall_s_median": statistics.median(w for w, _ in warm),
          "warm_device_ms_median": statistics.median(d for _, d in warm), "warm_calls": len(warm),
          "status": rc_dp, "front_points": len(front_dp), "best_score64": [b.score64 for b in best_dp],
          "note": "sched_front_dp: per-group Pareto fronts + block-order subset DP, exact fp64; wall = "
                  "host clock around the C-ABI call (host prep, H2D, kernels, D2H, decode); device = "
                  "CUDA events around the kernels only"}
    peaks = measured_peaks()
    f_max = float(peaks.get("sm_max_mhz", 1965.0))
    peak = SMS * LANES_PER_SM_CLK * f_max * 1e6 / 1e12      # T thread-instr/s
    # the dominant kernel's launch: the main pass of k_tile (its CUDA events);
    # the whole search (seed pass, group table, finalize) for comparison
    achieved = OPS_PER_CONFIG * ncfg / (main_ms / 1e3) / 1e12
    achieved_search = OPS_PER_CONFIG * ncfg / (search_ms / 1e3) / 1e12
    traffic = None
    try:
        prof_sum = json.load(open(os.path.join(ROOT, "profiles", "r02_traffic.json")))
        traffic = prof_sum["dram_bytes_per_config"] * (ncfg / args.steps)
    except Exception:
        pass
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": describe(args.workload, q) +
                               f"; step = 1/{SLICES} cyclic chunk slice of the space split over ranks",
                   "space_configs": space, "slices": SLICES, "chunk_log2": CHUNK_LOG2,
                   "time_to_optimal_schedule_s_extrapolated": SLICES * ms_per_step / 1e3,
                   "time_to_optimal_schedule_subset_dp": dp,
                   "l2": "256 MiB L2 flush between steps; tables (~24 KiB) staged in smem",
                   "refine": "fp64 canonical re-score of near-best / possibly-Pareto configurations",
                   "n_refined_timed": refined, "seed": 0, "coverage": coverage,
                   "feasible_fraction_timed": nfeas / max(1, ncfg)},
        "clocks": clk,
        "e2e": e2e,
        "gpu_launches": launches,
        "roofline": {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Tops/s",
                     "frac": achieved / peak, "traffic": traffic,
                     "frac_whole_search": achieved_search / peak,
                     "kernel_ms_per_step": main_ms / args.steps, "search_ms_per_step": search_ms / args.steps,
                     "note": f"{OPS_PER_CONFIG} fp32 ops/config x configs of the step / the main-pass k_tile "
                             "launch (CUDA events around it, on its stream; frac_whole_search divides by "
                             "all of sched_search's kernels: seed pass, group table, finalize); "
                             f"peak = {SMS} SMs x 4 SMSP x 32 lanes x {f_max:.0f} MHz (sm_max_mhz, "
                             "MEASURED_PEAKS.json) issue slots"},
    }
    if world == 1 and not args.no_secondary:
        line["config"]["secondary"] = secondary(S)
    if world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(prof, q)
    print(json.dumps(line), flush=True)
    if pg:
        dist.destroy_process_group()
    return 0


def run_full(args, step, barrier, rank, world, space, nw):
    """Complete search (all 64 slices): time-to-optimal-schedule, merged result."""
    import torch
    import paper_conf_sc_weaverkmeh0m24_b200 as S
    step(0)
    barrier()
    t0 = time.perf_counter()
    bests, pars, ncfg = [], [], 0
    for sigma in range(SLICES):
        res, best, par = step(sigma)
        bests.append(best)
        pars.append(par)
        ncfg += res.stats["n_configs"]
    mb, mp = S.merge(bests, pars, nw)
    barrier()
    dt = time.perf_counter() - t0
    if rank == 0:
        print(json.dumps({"mode": "full", "metric": "time-to-optimal-schedule", "value": dt, "unit": "s",
                          "n_gpus": world, "space_configs": space, "configs_rank0": ncfg,
                          "configs_per_s": space / dt,
                          "best": [(b.index, b.score64) for b in mb],
                          "pareto": [(p.index, p.makespan_s, p.energy_j) for p in mp]}), flush=True)
    import torch.distributed as dist
    if dist.is_initialized():
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="c4")
    ap.add_argument("--full", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-secondary", action="store_true")
    ap.add_argument("--ref-window", type=int, default=400_000)
    ap.add_argument("--dry-run", action="store_true", help="CPU/gloo plumbing test, no kernels")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return relaunch(args)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus:
        sys.stderr.write(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}\n")
        return 2
    if args.dry_run:
        return run_dry(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())
