python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
python tools/heuristic_gap.py > gpurun_out/heuristic_gap.md 2>&1; cat gpurun_out/heuristic_gap.md
python tools/splits_demo.py > gpurun_out/splits_demo.jsonl 2>&1; cut -c1-600 gpurun_out/splits_demo.jsonl
