timeout 1500 python bench.py --steps 2 --warmup 3 --no-projection --no-cpu-baseline --no-e2e --graphs 0 2>&1 | tail -1 > gpurun_out/bench_kinds.json
python -c "
import json; d=json.load(open('gpurun_out/bench_kinds.json'))
print('value', d['value'], 'ms', d['ms_per_step'])
tot=0
for k,v in d['kernels'].items(): print(k, round(v['ms_per_step'],1), v['launches_per_step']); tot+=v['ms_per_step']
print('sum kernels', tot)"
