#!/bin/bash
# round 2, call 28: checkpoint -- full GPU suite, smoke, bench
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r2ab_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2ab_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2ab_smoke.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2ab_bench.json 2> gpurun_out/r2ab_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r2ab_ref.json 2> gpurun_out/r2ab_ref.err
echo done
