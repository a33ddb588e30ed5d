mkdir -p gpurun_out
for c in sfx dfs front_dp splits; do
  echo "== $c" >> gpurun_out/synccheck2.log
  timeout 600 compute-sanitizer --tool synccheck --print-limit 4 python tools/sanitize_paths.py $c >> gpurun_out/synccheck2.log 2>&1
  echo "rc=$?" >> gpurun_out/synccheck2.log
done
grep -v "Host Frame" gpurun_out/synccheck2.log | head -60
