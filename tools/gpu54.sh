mkdir -p gpurun_out
timeout 300 python tools/bw_perf.py 2 2>&1 | tail -12
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 1500 python bench.py --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/bench54.json
python -c "
import json; d=json.load(open('gpurun_out/bench54.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'gemm', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks'])
print('e2e', d['e2e'], 'eager', d.get('eager'))
for n,v in d['kernels'].items():
    if isinstance(v, dict): print(n, round(v['ms'],1), v['launches'], v['tflops'])"
