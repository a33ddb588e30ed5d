#!/bin/bash
# round 2, call 76: partition-wide staircase bound for compiled and run-time sets, not Pareto-only (PM2) vs NP
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in NP PM2 NP PM2 NP PM2; do echo "variant=$v" >> gpurun_out/r2bx.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,pareto,w11_21_12 --reps 1 >> gpurun_out/r2bx.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_PM2.so timeout 1500 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_fuzz.py -q -x > gpurun_out/r2bx_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bx_tests.log
echo done
