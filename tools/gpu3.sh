set -x
timeout 600 python -m pytest tests/test_gpu_attention.py tests/test_gpu_parity.py -x -q 2>&1 | tail -15
timeout 900 python bench.py --steps 3 --warmup 3 2>&1 | tail -5
