#!/bin/bash
# round 2, call 31: COUNT_IDLE on the tile kernel; regressions (tile, variants, weights); timing
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_variants.py tests/test_gpu_tile_weights.py tests/test_gpu_parity.py tests/test_gpu_scores32.py -q > gpurun_out/r2ae_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ae_tests.log
timeout 600 python tools/time_slices.py c4 --sets c4,c1_set,pareto --reps 1 > gpurun_out/r2ae.jsonl 2>&1
echo done
