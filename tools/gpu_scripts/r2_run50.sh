#!/bin/bash
# round 2, call 50: suffix table rows rebuilt in one batch (TB = default build) vs P2
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_sfx.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py -q -x > gpurun_out/r2ax_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ax_tests.log
for v in P2 TB P2 TB; do echo "variant=$v" >> gpurun_out/r2ax.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2ax.jsonl 2>&1; done
echo done
