CUDA_LAUNCH_BLOCKING=1 timeout 120 python tools/dbg_gemm.py 2>&1 | grep -v Warning | tail -12
timeout 300 /usr/local/cuda/bin/compute-sanitizer --tool memcheck python tools/dbg_attn.py 2>&1 | head -30
