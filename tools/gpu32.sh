mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_gemm.py -x -q 2>&1 | tail -4
timeout 1500 python bench.py --steps 3 --warmup 3 --no-projection --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/bench32.json
python -c "
import json; d=json.load(open('gpurun_out/bench32.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'gemm', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks'])
print('e2e', d['e2e'], 'eager', d.get('eager'))
for n,v in d['kernels'].items():
    if isinstance(v, dict): print(n, round(v['ms'],1), v['launches'], v['tflops'])"
