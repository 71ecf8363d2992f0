mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_norm.py tests/test_gpu_ce.py tests/test_gpu_attention.py tests/test_gpu_parity.py -x -q 2>&1 | tail -15
timeout 1500 python bench.py --steps 3 --warmup 3 --no-projection --no-cpu-baseline 2>&1 | tail -1 > gpurun_out/bench23.json
python -c "
import json; d=json.load(open('gpurun_out/bench23.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'gemm', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks'])
print('e2e', d['e2e'], 'eager', d.get('eager'))
for n,v in d['kernels'].items():
    if isinstance(v, dict): print(n, round(v['ms'],1), v['launches'], v['tflops'])"
B="python bench.py --micro 2 --steps 1 --warmup 3 --graphs 0 --no-cpu-baseline --no-e2e --no-projection"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches4.csv $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pipe|softmax_ce_reg|colsum_final_wide" -s 30 -c 6 -o gpurun_out/prof_pipe4 $B > /dev/null 2>&1
echo done
