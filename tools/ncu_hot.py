"""Hot SASS regions of an ncu source page (csv from `ncu -i rep --page source --csv
--print-source sass`): instructions executed, average active threads, stall samples.
  python tools/ncu_hot.py page.csv [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ix = {k: i for i, k in enumerate(hdr)}
data = []
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    try:
        data.append((int(r[0], 16), r[1].strip(), float(r[ix["Warp Stall Sampling (All Samples)"]] or 0),
                     float(r[ix["Instructions Executed"]] or 0), float(r[ix["Avg. Threads Executed"]] or 0)))
    except ValueError:
        continue
tot_i = sum(d[3] for d in data)
tot_s = sum(d[2] for d in data)
tot_t = sum(d[3] * d[4] for d in data)
print(f"warp-instr {tot_i:.3e}  thread-instr {tot_t:.3e}  avg lanes {tot_t / tot_i:.2f}  samples {tot_s:.0f}")
# contiguous regions of 64 instructions
top = int(sys.argv[2]) if len(sys.argv) > 2 else 12
blk = {}
for a, s, st, ie, at in data:
    b = a // 0x400
    x = blk.setdefault(b, [0, 0, 0, a])
    x[0] += ie
    x[1] += ie * at
    x[2] += st
for b, (ie, th, st, a0) in sorted(blk.items(), key=lambda kv: -kv[1][0])[:top]:
    print(f"{b * 0x400:#8x}: warp-instr {ie / tot_i:6.1%}  lanes {th / max(ie, 1):5.1f}  stalls {st / tot_s:6.1%}")
