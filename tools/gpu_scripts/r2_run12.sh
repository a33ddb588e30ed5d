#!/bin/bash
# round 2, call 12: deferred tile loop (A/B)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for lm in 0 1; do echo "loopmode=$lm" >> gpurun_out/r2l_slices.jsonl; SCHED_TILE_LOOP=$lm timeout 600 python tools/time_slices.py c4 --sets c4,w11,pareto --reps 2 >> gpurun_out/r2l_slices.jsonl 2>&1; done
SCHED_TILE_LOOP=1 timeout 1200 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_parity.py -q -k "c4 or window or tile or sharded or dense or bench" > gpurun_out/r2l_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2l_tests.log
echo done
