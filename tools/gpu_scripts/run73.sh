python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_dp.py -q 2>&1 | tail -2
python tools/dp_c4client.py c5 gpu | cut -c1-100
python tools/dp_c4client.py c4 gpu | cut -c1-100
python tools/dp_c4client.py | cut -c1-100
