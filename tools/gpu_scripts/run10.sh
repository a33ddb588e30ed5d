timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "tile_kernel_path" 2>&1 | grep -v "^  /\|Warning\|^$" | tail -40
