#!/bin/bash
# round 2, call 15: racecheck ctile2 after the syncwarp; ncu of the suffix kernel on c5
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 compute-sanitizer --tool racecheck --racecheck-report analysis --print-limit 20 python tools/sanitize_paths.py ctile2 > gpurun_out/r2o_racecheck_ctile2.log 2>&1
echo "rc=$?" >> gpurun_out/r2o_racecheck_ctile2.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sfx --launch-skip 1 -c 1 -o gpurun_out/r02_sfx_c5 python tools/prof_search.py c5 > gpurun_out/r2o_ncu_sfx.log 2>&1
echo done
