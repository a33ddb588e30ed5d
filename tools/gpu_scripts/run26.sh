python tools/time_search.py c4 0 3298534883328 --reps 2 | cut -c1-250
python tools/time_search.py c4 100000000000000 3298534883328 | cut -c1-250
timeout 600 python bench.py --no-cpu-baseline 2>&1 | tail -1 | cut -c1-300
