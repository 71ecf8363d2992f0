mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
timeout 1500 python bench.py 2>&1 | tail -1 > gpurun_out/bench43.json
python -c "
import json; d=json.load(open('gpurun_out/bench43.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'gemm', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks'])
print('e2e', d['e2e'], 'eager', d.get('eager')); print('cpu', d.get('cpu_baseline'))
for n,v in d['kernels'].items():
    if isinstance(v, dict): print(n, round(v['ms'],1), v['launches'], v['tflops'])"
B="python bench.py --micro 2 --steps 1 --warmup 3 --graphs 0 --no-cpu-baseline --no-e2e --no-projection"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches5.csv $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc2 -s 40 -c 4 -o gpurun_out/prof_gemm5 $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"fa_bwd_dkdv|fa_bwd_dq|fa_fwd2" -s 6 -c 3 -o gpurun_out/prof_attn5 $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:"norm_|softmax_ce|colsum|cast_k" -s 40 -c 8 -o gpurun_out/prof_bw5 $B > /dev/null 2>&1
echo done
