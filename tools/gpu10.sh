timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k full_width 2>&1 | tail -6
timeout 1200 python bench.py --steps 3 --warmup 3 2>&1 | tail -1
