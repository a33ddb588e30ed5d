python tools/time_search.py c4 0 3298534883328 --reps 2 | cut -c1-300
python tools/time_search.py c4 100000000000000 3298534883328 | cut -c1-300
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
