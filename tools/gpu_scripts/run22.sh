python tools/time_search.py c4 100000000000000 3298534883328 | cut -c1-400
python tools/time_search.py c4 100000000000000 549755813888 | cut -c1-400
