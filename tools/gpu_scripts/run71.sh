# final round-1 validation: full GPU parity (incl. n = 14 per-client golden), smoke (c1 + c4 tile window), bench
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -3
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_r71.json 2> gpurun_out/bench_r71.err; tail -1 gpurun_out/bench_r71.json | cut -c1-200
python tools/dp_c4client.py | cut -c1-120
