set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 300 python -m pytest tests/test_gpu_gemm.py -x -q 2>&1 | tail -5
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -40
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -5
