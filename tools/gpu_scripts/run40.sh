# round-1 re-validation of the restored tree: build, GPU parity, smoke, bench
set -o pipefail
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/bench_r40.json 2> gpurun_out/bench_r40.err; tail -1 gpurun_out/bench_r40.json | cut -c1-3000
