mkdir -p gpurun_out
timeout 600 python tools/gemm_step.py 2>&1 | tail -20
timeout 300 python tools/attn_bwd_exp.py 0 2>&1 | tail -5
timeout 300 python tools/attn_perf.py 2>&1 | tail -8
