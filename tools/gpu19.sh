timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q 2>&1 | tail -2
timeout 600 python tools/gemm_perf.py 2>&1 | tail -16
