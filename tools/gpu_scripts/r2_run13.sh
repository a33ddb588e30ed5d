#!/bin/bash
# round 2, call 13: fp32 scores of every configuration; tile timing after revert; full GPU suite
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_scores32.py -q -s > gpurun_out/r2m_scores32.log 2>&1
echo "rc=$?" >> gpurun_out/r2m_scores32.log
timeout 600 python tools/time_slices.py c4 --sets c4,w11,c1_set,pareto --reps 1 > gpurun_out/r2m_slices.jsonl 2>&1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r2m_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2m_gputests.log
echo done
