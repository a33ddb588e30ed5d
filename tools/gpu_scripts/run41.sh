# N3 split search parity + subset-DP literal per-client c4 timing
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_splits.py -x -q 2>&1 | tail -15
python tools/dp_c4client.py > gpurun_out/dp_c4client.json 2>&1; cut -c1-400 gpurun_out/dp_c4client.json
python tools/dp_c4client.py c4 gpu > gpurun_out/dp_c4gpu.json 2>&1; cut -c1-400 gpurun_out/dp_c4gpu.json
