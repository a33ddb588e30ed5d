#!/bin/bash
# round 2, call 2: run-time weight tile kernel (parity + timing), tile parity regression
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_edge.py -q -x > gpurun_out/r2b_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2b_tests.log
timeout 600 python tools/time_slices.py c4 --sets c4,c1_set,c5_sweep,eight,w11,pareto --reps 2 > gpurun_out/r2b_slices.jsonl 2>&1
echo done
