#!/bin/bash
# round 2, call 37: tile loop over the lane's full tiles without bounds checks, ld.shared staircase screen,
# COUNT_IDLE as one FFMA (N1 = default build) vs HEAD (T3); RT4N with the staircase screen first; tile parity
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in T3 N1 T3 N1 T3 N1; do echo "variant=$v" >> gpurun_out/r2ak.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,w11_21_12,pareto --reps 1 >> gpurun_out/r2ak.jsonl 2>&1; done
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tile_weights.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_scores32.py tests/test_gpu_variants.py -q -x > gpurun_out/r2ak_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ak_tests.log
echo done
