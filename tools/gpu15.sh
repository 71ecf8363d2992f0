timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_attention.py -x -q 2>&1 | tail -4
timeout 300 python tools/attn_perf.py 2>&1 | grep '"variant": -1'
timeout 1200 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-projection 2>&1 | tail -1
