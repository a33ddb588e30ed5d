#!/bin/bash
# round 2, call 11: per-set tile loop choice; run-time-weight log pre-screen
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python tools/time_slices.py c4 --sets c4,w11,c1_set,c5_sweep,w10,pareto,eight,w11_21_12 --reps 2 > gpurun_out/r2k_slices.jsonl 2>&1
SCHED_TILE_RT=1 timeout 300 python tools/time_slices.py c4 --sets c4 --reps 1 >> gpurun_out/r2k_slices.jsonl 2>&1
timeout 1200 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_edge.py -q > gpurun_out/r2k_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2k_tests.log
echo done
