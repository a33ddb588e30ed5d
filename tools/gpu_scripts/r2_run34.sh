#!/bin/bash
# round 2, call 34 (new session): checkpoint -- full GPU suite, smoke, bench, launch list
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2ah_smi.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r2ah_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ah_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2ah_smoke.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2ah_bench.json 2> gpurun_out/r2ah_bench.err
echo done
