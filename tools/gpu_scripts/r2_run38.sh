#!/bin/bash
# round 2, call 38: next partition's group records by cp.async during the current partition's tiles (PF = default build) vs N1
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in N1 PF N1 PF N1 PF; do echo "variant=$v" >> gpurun_out/r2al.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,c1_set,pareto --reps 1 >> gpurun_out/r2al.jsonl 2>&1; done
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tile_weights.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_scores32.py tests/test_gpu_variants.py -q -x > gpurun_out/r2al_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2al_tests.log
echo done
