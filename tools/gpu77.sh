MARIO_LIB=$PWD/ab/libmario_J.so timeout 600 python -m pytest tests/test_gpu_attention.py tests/test_gpu_parity.py -x -q 2>&1 | tail -1
for v in K J; do MARIO_LIB=$PWD/ab/libmario_$v.so timeout 300 python tools/attn_perf.py 2>&1 | grep '"variant": -1' | sed "s/^/$v /"; done
bash tools/gpu65.sh
