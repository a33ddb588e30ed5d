# tile kernel v8 (FMNMX3 T, FADD E, bounds-free full steps): timing + parity
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
python tools/time_search.py c4 0 3298534883328 --reps 2 | cut -c1-200
python tools/time_search.py c4 100000000000000 3298534883328 | cut -c1-200
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_variants.py -x -q 2>&1 | tail -3
