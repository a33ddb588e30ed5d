#!/bin/bash
# round 2, call 1: new GPU parity tests, the whole -m gpu suite, smoke, bench
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2_smi.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_edge.py -q -s -x > gpurun_out/r2_edge.log 2>&1
echo "edge rc=$?" >> gpurun_out/r2_edge.log
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r2_gputests.log 2>&1
echo "gpu rc=$?" >> gpurun_out/r2_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2_smoke.log 2>&1
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/r2_bench.json 2> gpurun_out/r2_bench.err
echo done
