#!/bin/bash
# round 2, call 82: final bench; cold DP check; tile parity after the vote-loop change
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2cd_bench.json 2> gpurun_out/r2cd_bench.err
timeout 1500 python -m pytest tests/test_gpu_tile_weights.py tests/test_gpu_dp.py tests/test_gpu_edge.py -q -x > gpurun_out/r2cd_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2cd_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2cd_smoke.log 2>&1
echo done
