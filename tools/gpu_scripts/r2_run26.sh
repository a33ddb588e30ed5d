#!/bin/bash
# round 2, call 26: tile kernel CTA shapes: 256x2 (base), 384x2 (80 regs), 512x1 (128 regs)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in base T384 T512 base T384 T512; do echo "variant=$v" >> gpurun_out/r2z.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,pareto --reps 1 >> gpurun_out/r2z.jsonl 2>&1; done
echo done
