# PER_CLIENT tile kernel: parity + timing
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "client_tile or c2_full or c1_full or small_spaces" 2>&1 | tail -3
python tools/time_search.py c2 --reps 3 | tail -1 | cut -c1-250
