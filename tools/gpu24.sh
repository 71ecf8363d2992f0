mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_norm.py tests/test_gpu_ce.py -x -q 2>&1 | tail -4
timeout 300 python tools/bw_perf.py 2>&1 | tail -40
