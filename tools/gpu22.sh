mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/smi.txt
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
cat gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 1500 python bench.py 2>&1 | tail -1 > gpurun_out/bench_full.json
python -c "
import json; d=json.load(open('gpurun_out/bench_full.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'gemm', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks'])
print('e2e', d['e2e'], 'eager', d.get('eager')); print('cpu', d.get('cpu_baseline'))
for n,v in d['kernels'].items():
    if isinstance(v, dict): print(n, round(v['ms'],1), v['launches'], v['tflops'])"
B="python bench.py --micro 2 --steps 1 --warmup 3 --graphs 0 --no-cpu-baseline --no-e2e --no-projection"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches3.csv $B > gpurun_out/launches3_stdout.log 2>&1
echo "launch list rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc2 -s 40 -c 6 -o gpurun_out/prof_gemm3 $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fa_bwd -s 4 -c 2 -o gpurun_out/prof_fabwd3 $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"norm|fa_fwd_tc|softmax_ce|colsum" -s 20 -c 8 -o gpurun_out/prof_misc3 $B > /dev/null 2>&1
echo done
