#!/bin/bash
# round 2, call 52: checkpoint after the suffix-kernel changes (M = 7, 512 x 1) -- full GPU suite, smoke,
# c5 timing, sanitizers over every kernel path, bench
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r2az_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2az_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2az_smoke.log 2>&1
timeout 300 python tools/time_search.py c5 --reps 3 > gpurun_out/r2az_c5.jsonl 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2az_bench.json 2> gpurun_out/r2az_bench.err
echo done
