timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q 2>&1 | tail -8
timeout 600 python tools/gemm_perf.py 0,1 2>&1 | tail -40
