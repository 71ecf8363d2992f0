# HEAD evidence: default bench line, launch list of a lean step, --set full of the column-sum kernels
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 1500 python bench.py 2>&1 | tail -1 > gpurun_out/bench87.json
python -c "
import json; d=json.load(open('gpurun_out/bench87.json'))
print('value', d['value'], 'ms', d['ms_per_step'], 'roof', d['roofline']['achieved'], d['roofline']['frac'], 'clk', d['clocks'])
print('e2e', d['e2e'], 'eager', d.get('eager'))
for n,v in d['kernels'].items():
    if isinstance(v, dict): print(n, round(v['ms'],1), v['launches'], v['tflops'])"
timeout 900 python bench.py --impl reference --steps 1 --warmup 0 2>&1 | tail -1 > gpurun_out/ref87.json
cat gpurun_out/ref87.json | cut -c1-300
B="python bench.py --micro 2 --steps 1 --warmup 3 --graphs 0 --no-cpu-baseline --no-e2e --no-projection"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches87.csv $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"colsum_reduce|colsum_partial" -s 20 -c 4 -o gpurun_out/prof_colsum87 $B > /dev/null 2>&1
echo done
