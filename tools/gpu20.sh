timeout 600 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_parity.py -x -q 2>&1 | tail -2
timeout 1500 python bench.py --steps 3 --warmup 3 --no-projection --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/bench_latest.json
python -c "
import json; d=json.load(open('gpurun_out/bench_latest.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'gemm', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks'])
print('kernels', json.dumps(d['kernels'])); print('graph', d['graph_replay'])"
