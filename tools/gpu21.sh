timeout 1500 python bench.py --steps 2 --warmup 3 --no-projection --no-cpu-baseline --no-e2e --graphs 0 2>&1 | tail -1 > gpurun_out/bench_kinds.json
python -c "
import json; d=json.load(open('gpurun_out/bench_kinds.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'gemm frac', d['roofline']['frac'])
tot=0
k=d['kernels']; print('breakdown step ms', k['step_ms'])
for n,v in k.items():
    if isinstance(v, dict): print(n, round(v['ms'],1), v['launches'], v['tflops']); tot+=v['ms']
print('sum kernels', tot)"
