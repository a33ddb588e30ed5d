#!/bin/bash
# round 2, call 33: COUNT_IDLE in the subset DP; DP regression
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_dp.py -q > gpurun_out/r2ag_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ag_tests.log
timeout 300 python tools/dp_cold.py c4 > gpurun_out/r2ag_dp.jsonl 2>&1
echo done
