"""Summaries of ncu outputs for profiles/ (run here, no GPU needed).

  python tools/ncu_summary.py launches <launches.csv> <out.md>
  python tools/ncu_summary.py kernel <report.ncu-rep> <out.md> [configs_per_launch]
"""
import collections
import csv
import io
import json
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
    "launch__occupancy_limit_registers", "sm__warps_active.avg.per_cycle_active",
    "sm__inst_executed.avg.per_cycle_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__instruction_throughput.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "smsp__inst_executed.sum", "smsp__warps_eligible.avg.per_cycle_active",
    "sm__sass_thread_inst_executed_op_fp32_pred_on.sum", "smsp__thread_inst_executed_per_inst_executed.ratio",
]


def launches(path, out):
    rows = []
    txt = open(path).read()
    start = txt.index('"ID"')
    for r in csv.DictReader(io.StringIO(txt[start:])):
        if r["Metric Name"] == "gpu__time_duration.sum":
            rows.append((r["Kernel Name"].split("(")[0], float(r["Metric Value"])))
    agg = collections.OrderedDict()
    for name, ns in rows:
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += ns
    tot = sum(v[1] for v in agg.values())
    with open(out, "w") as f:
        f.write(f"# ncu launch list summary ({path})\n\n")
        f.write("`ncu --metrics gpu__time_duration.sum --clock-control none` over `bench.py --steps 2 --warmup 1`"
                " (cold-cache, serialised: compare shares, not absolutes)\n\n")
        f.write("| kernel | launches | total ms | mean ms | share |\n|---|---|---|---|---|\n")
        for name, (n, ns) in sorted(agg.items(), key=lambda x: -x[1][1]):
            f.write(f"| `{name}` | {n} | {ns / 1e6:.3f} | {ns / n / 1e6:.4f} | {ns / tot:.4%} |\n")
        f.write(f"\ntotal launches: {len(rows)}, total device time {tot / 1e6:.1f} ms\n")


def kernel(rep, out, configs=None):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw[raw.index('"ID"'):])))
    hdr, units = rows[0], rows[1]
    with open(out, "w") as f:
        f.write(f"# ncu --set full summary ({rep})\n\n")
        for vals in rows[2:]:
            name = vals[hdr.index("Kernel Name")]
            f.write(f"## `{name[:120]}`\n\n| metric | value | unit |\n|---|---|---|\n")
            d = {}
            for i, h in enumerate(hdr):
                if h in KEYS or (h.startswith("smsp__average_warps_issue_stalled") and h.endswith("per_issue_active.ratio")):
                    f.write(f"| {h} | {vals[i]} | {units[i]} |\n")
                    d[h] = (vals[i], units[i])
            if configs:
                def num(k):
                    v, u = d[k]
                    v = float(v.replace(",", ""))
                    return v * {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1}.get(u, 1)
                dram = num("dram__bytes_read.sum") + num("dram__bytes_write.sum")
                inst = num("smsp__inst_executed.sum")
                f.write(f"\nconfigs in the launch: {configs}; DRAM bytes/config: {dram / configs:.3e}; "
                        f"warp-instructions/config: {inst / configs:.4f} "
                        f"(thread-instr/config ~{32 * inst / configs:.2f})\n")
                json.dump({"dram_bytes_per_config": dram / configs, "thread_inst_per_config": 32 * inst / configs,
                           "source": rep}, open(out.replace(".md", ".json"), "w"), indent=1)
            f.write("\n")


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        kernel(sys.argv[2], sys.argv[3], int(sys.argv[4]) if len(sys.argv) > 4 else None)
