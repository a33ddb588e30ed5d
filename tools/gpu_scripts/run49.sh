# N=2 bench path (two ranks sharing cuda:0 over gloo), reference arm under torchrun, DP golden n=13
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
BENCH_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | cut -c1-400
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 2>&1 | tail -1 | cut -c1-200
timeout 600 python -m pytest tests/test_gpu_dp.py -q -k "golden and 13" 2>&1 | tail -2
