#!/bin/bash
# round 2, call 83: tiles cleared by the partition-wide bound skip the weight screen too (SK) vs NS
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in NS SK NS SK NS SK; do echo "variant=$v" >> gpurun_out/r2ce.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,w11 --reps 1 >> gpurun_out/r2ce.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_SK.so timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tile_weights.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_scores32.py tests/test_gpu_variants.py -q -x > gpurun_out/r2ce_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ce_tests.log
echo done
