for sk in 0 1; do STREAMK=$sk timeout 600 python tools/gemm_step.py 2>&1 | tail -16 | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('sk$sk', d.get('gemm','TOTAL'), d.get('us_epi', d.get('layer_ms')), d.get('tflops_epi', d.get('layer_total_tflops')))"; done
