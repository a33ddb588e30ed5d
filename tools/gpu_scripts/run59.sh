python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "client_tile and 14" 2>&1 | grep -E "assert|Error|where|^E " | head -20
