#!/bin/bash
# round 2, call 20: ctile2 exact tile corner from per-warp fp64 T tables (D) vs round-2 baseline (A)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for v in A D A D; do echo "variant=$v" >> gpurun_out/r2t.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_slices.py c3 --scope 0 --sets w11 --reps 1 >> gpurun_out/r2t.jsonl 2>&1; done
timeout 1500 python -m pytest tests/test_gpu_ctile2.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py -q > gpurun_out/r2t_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2t_tests.log
echo done
