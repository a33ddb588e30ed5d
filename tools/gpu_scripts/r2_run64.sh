#!/bin/bash
# round 2, call 64: 256-configuration tiles for k >= 7 partitions (T256 = default build) vs 64-configuration tiles (N256)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in N256 T256 N256 T256 N256 T256; do echo "variant=$v" >> gpurun_out/r2bl.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c4 --sets c4,w11,w11_21_12 --reps 1 >> gpurun_out/r2bl.jsonl 2>&1; done
SCHED_SO_PATH=ab/lib_T256.so timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tile_weights.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py tests/test_gpu_variants.py tests/test_gpu_overflow.py -q -x > gpurun_out/r2bl_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bl_tests.log
echo done
