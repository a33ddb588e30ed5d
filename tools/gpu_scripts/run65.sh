python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_dp.py -q -s -k "c5 or enumeration" 2>&1 | grep -E "c5 DP|passed|failed|Error" | head
python tools/dp_c4client.py c5 gpu | cut -c1-300
