#!/bin/bash
# round 2, call 80: final bench (twice) and the GPU suite's ctile2 / dp parts after the last change
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2cb_bench.json 2> gpurun_out/r2cb_bench.err
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r2cb_bench2.json 2> gpurun_out/r2cb_bench2.err
timeout 300 python tools/dp_cold.py c4 > gpurun_out/r2cb_dp.jsonl 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2cb_smoke.log 2>&1
echo done
