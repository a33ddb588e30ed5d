#!/bin/bash
# round 2, call 30: 2 / 3 levels with last-two-group tiles
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_tile_weights.py -q -k "two_and_three" > gpurun_out/r2ad_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ad_tests.log
for lv in 50,75,100 50,100; do timeout 600 python tools/time_slices.py c4 --levels $lv --sets c4,pareto,w11 --reps 1 --slices 1024 >> gpurun_out/r2ad.jsonl 2>&1; done
echo done
