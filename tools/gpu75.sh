mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1500 python bench.py 2>&1 | tail -1 > gpurun_out/bench75.json
python -c "
import json; d=json.load(open('gpurun_out/bench75.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'roof', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks'])
print('e2e', d['e2e'], 'eager', d.get('eager')); print('cpu', d.get('cpu_baseline'))
for n,v in d['kernels'].items():
    if isinstance(v, dict): print(n, round(v['ms'],1), v['launches'], v['tflops'])"
B="python bench.py --micro 2 --steps 1 --warmup 3 --graphs 0 --no-cpu-baseline --no-e2e --no-projection"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches75.csv $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc2 -s 40 -c 4 -o gpurun_out/prof_gemm75 $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"fa_bwd_dkdv_ts|fa_bwd_dq_img" -s 2 -c 2 -o gpurun_out/prof_attnb75 $B > /dev/null 2>&1
echo done
