#!/bin/bash
# round 2, call 9: full GPU suite, smoke, bench, c5 timing, ctile2 ncu on a 1/64 c3-client slice
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r2i_gputests.log 2>&1
echo "rc=$?" >> gpurun_out/r2i_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2i_smoke.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r2i_bench.json 2> gpurun_out/r2i_bench.err
timeout 300 python tools/time_search.py c5 --reps 3 > gpurun_out/r2i_c5.jsonl 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_ctile2 --launch-skip 1 -c 1 -o gpurun_out/r02_ctile2_c3client_64 python tools/prof_search.py c3 --scope 0 --shard 5 64 > gpurun_out/r2i_ncu_ctile2.log 2>&1
echo done
