# colsum partial grid (8 CTAs/SM, no unroll) vs the 4-row unroll: GPU suite on new2, alternating lean benches
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-projection"
for i in 1 2; do
  for v in new new2; do
    MARIO_LIB=ab/libmario_$v.so timeout 600 $B 2>&1 | tail -1 > gpurun_out/ab88_${v}_$i.json
    python -c "
import json; d=json.load(open('gpurun_out/ab88_${v}_$i.json'))
k=d['kernels']; print('$v', d['value'], d['ms_per_step'], 'colsum', round(k['colsum']['ms'],1), 'norm', round(k['norm']['ms'],1), 'gemm', round(k['gemm']['ms'],1), d['clocks']['sm_mhz'])"
  done
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:colsum -c 40 --csv --log-file gpurun_out/launches88.csv python bench.py --micro 2 --steps 1 --warmup 1 --graphs 0 --no-cpu-baseline --no-e2e --no-projection > /dev/null 2>&1
