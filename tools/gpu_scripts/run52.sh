# subset-DP phase 1 nested low-member loops: parity + literal per-client c4 timing
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_dp.py -q -k "not 14" 2>&1 | tail -2
python tools/dp_c4client.py | cut -c1-200
