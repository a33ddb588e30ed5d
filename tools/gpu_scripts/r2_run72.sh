#!/bin/bash
# round 2, call 72: final validation -- full GPU suite, smoke, bench, launch list of the bench's timed steps
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/r2bt_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2bt_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2bt_smoke.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2bt_bench.json 2> gpurun_out/r2bt_bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r2bt_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-secondary > gpurun_out/r2bt_ncu.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r2bt_ref.json 2> gpurun_out/r2bt_ref.err
echo done
