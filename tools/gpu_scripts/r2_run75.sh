#!/bin/bash
# round 2, call 75: partition-wide staircase bound before the per-tile bucket lookup (PM = default) vs without (NP)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in NP PM NP PM NP PM; do echo "variant=$v" >> gpurun_out/r2bw.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,w11,pareto --reps 1 >> gpurun_out/r2bw.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_PM.so timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tile_weights.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_variants.py -q -x > gpurun_out/r2bw_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bw_tests.log
echo done
