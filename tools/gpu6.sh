timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_attention.py -x -q 2>&1 | tail -4
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -2
