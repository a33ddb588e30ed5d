python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python bench.py --full 2>&1 | tail -1 > gpurun_out/full_c4_v3.json; cut -c1-400 gpurun_out/full_c4_v3.json
for c in c1 c2 c3 c5; do python tools/time_search.py $c --reps 2 | tail -1; done > gpurun_out/full_spaces_v3.jsonl; cut -c1-200 gpurun_out/full_spaces_v3.jsonl
