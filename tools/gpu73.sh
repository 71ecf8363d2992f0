timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q 2>&1 | tail -1
for v in 0 1; do MARIO_GEMM_L2HINT=$v timeout 300 python tools/gemm_step.py 2>&1 | tail -16 | python -c "
import sys,json
t=[]
for l in sys.stdin:
    d=json.loads(l); t.append(f\"{d.get('gemm','TOTAL')}={d.get('us_epi', d.get('layer_ms'))}\")
print('hint$v', ' '.join(t))"; done
for i in 1 2; do for v in 0 1; do
MARIO_GEMM_L2HINT=$v timeout 900 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-projection 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']
print('hint$v', round(d['value'],3), 'clk', d['clocks']['sm_mhz'], ' '.join(f'{n}={round(v[\"ms\"],1)}' for n,v in k.items() if isinstance(v,dict)))"
done; done
