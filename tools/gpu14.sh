timeout 300 python -m pytest tests/test_gpu_attention.py -x -q 2>&1 | tail -4
timeout 300 python tools/attn_perf.py 2>&1 | tail -6
