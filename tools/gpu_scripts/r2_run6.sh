#!/bin/bash
# round 2, call 6: threshold products in registers; timing of weight sets; full GPU suite
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python tools/time_slices.py c4 --sets c4,c1_set,c5_sweep,w10,w11,eight,pareto --reps 1 > gpurun_out/r2f_slices.jsonl 2>&1
timeout 600 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 2 >> gpurun_out/r2f_slices.jsonl 2>&1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r2f_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2f_gputests.log
echo done
