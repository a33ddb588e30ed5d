#!/bin/bash
# round 2, call 49: pair tile as a loop over x_{M-2}'s options (P2 = default build) vs the unrolled 8x8 tile (PR)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_sfx.py tests/test_gpu_edge.py tests/test_gpu_fuzz.py -q -x > gpurun_out/r2aw_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2aw_tests.log
for v in PR P2 PR P2; do echo "variant=$v" >> gpurun_out/r2aw.jsonl; SCHED_SO_PATH=ab/lib_$v.so timeout 300 python tools/time_search.py c5 --reps 2 >> gpurun_out/r2aw.jsonl 2>&1; done
echo done
