# compute-sanitizer memcheck / racecheck / synccheck over every kernel path
# (tools/sanitize_paths.py); logs under gpurun_out/sanitize_<tool>.log
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  extra=""
  [ "$tool" = racecheck ] && extra="--racecheck-report analysis"
  timeout 900 compute-sanitizer --tool $tool $extra --print-limit 20 python tools/sanitize_paths.py \
    > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize_$tool.log
  tail -4 gpurun_out/sanitize_$tool.log
done
