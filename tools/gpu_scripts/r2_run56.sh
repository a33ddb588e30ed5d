#!/bin/bash
# round 2, call 56: k_ctile2 staircase refreshed every 32 steps inside a partition (SY = default build) vs B; seed sizes
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_ctile2.py tests/test_gpu_fuzz.py -q -x > gpurun_out/r2bd_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bd_tests.log
for v in B SY B SY; do echo "variant=$v seed=16,32" >> gpurun_out/r2bd.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4,w11_21_12 --reps 1 >> gpurun_out/r2bd.jsonl 2>&1; done
for sd in "12,32" "14,32" "10,128" "16,8"; do echo "variant=SY seed=$sd" >> gpurun_out/r2bd.jsonl; SCHED_C2_SEED=$sd SCHED_SO_PATH=ab/lib_SY.so timeout 300 python tools/time_slices.py c3 --scope 0 --sets c4 --reps 2 >> gpurun_out/r2bd.jsonl 2>&1; done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2bd_launches.csv python tools/prof_search.py c3 --scope 0 --shard 5 64 > gpurun_out/r2bd_ncu.log 2>&1
echo done
