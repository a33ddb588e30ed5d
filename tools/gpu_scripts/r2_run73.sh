#!/bin/bash
# round 2, call 73: bench with the main-pass roofline, smoke, parity spot checks
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2bu_smoke.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2bu_bench.json 2> gpurun_out/r2bu_bench.err
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_splits.py tests/test_gpu_dp.py tests/test_gpu_nccl.py -q -x > gpurun_out/r2bu_tests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bu_tests.log
echo done
