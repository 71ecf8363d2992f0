timeout 600 python -m pytest tests/test_gpu_attention.py -x -q 2>&1 | tail -2
MARIO_DQI_CTAS=2 timeout 300 python tools/attn_bwd_exp.py 0 2>&1 | tail -2
MARIO_DQI_CTAS=1 timeout 300 python tools/attn_bwd_exp.py 0 2>&1 | tail -1
