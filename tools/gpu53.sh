timeout 900 python -m pytest tests/test_gpu_gemm.py -x -q 2>&1 | tail -2
for i in 1 2; do timeout 600 python tools/gemm_step.py 2>&1 | tail -16 | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print(d.get('gemm','TOTAL'), d.get('us_epi', d.get('layer_ms')), d.get('tflops_epi', d.get('layer_total_tflops')))"; done
