#!/bin/bash
# round 2, call 14: compute-sanitizer memcheck / racecheck / synccheck over every kernel path (incl. round-2 kernels)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  extra=""
  [ "$tool" = racecheck ] && extra="--racecheck-report analysis"
  timeout 1200 compute-sanitizer --tool $tool $extra --print-limit 20 python tools/sanitize_paths.py \
    > gpurun_out/r2n_sanitize_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/r2n_sanitize_$tool.log
done
echo done
