mkdir -p gpurun_out
timeout 600 python tools/gemm_step.py 2>&1 | tail -20
timeout 900 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_parity.py -x -q 2>&1 | tail -3
timeout 600 python tools/gemm_step.py 2>&1 | tail -20
