#!/bin/bash
# round 2, call 29: 2 / 3 searched levels on the tile kernel: parity + timing vs the generic kernel
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_tile_weights.py -q -k "two_and_three" > gpurun_out/r2ac_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ac_tests.log
for lv in 50,75,100 50,100; do timeout 600 python tools/time_slices.py c4 --levels $lv --sets c4,pareto --reps 1 --slices 1024 >> gpurun_out/r2ac.jsonl 2>&1; SCHED_KERNEL=generic timeout 600 python tools/time_slices.py c4 --levels $lv --sets c4 --reps 1 --slices 8192 >> gpurun_out/r2ac.jsonl 2>&1; done
echo done
