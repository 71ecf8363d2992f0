# colsum_reduce A/B: full GPU suite on the new library, then alternating lean bench runs old/new
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-projection"
for i in 1 2; do
  for v in old new; do
    MARIO_LIB=ab/libmario_$v.so timeout 600 $B 2>&1 | tail -1 > gpurun_out/ab86_${v}_$i.json
    python -c "
import json; d=json.load(open('gpurun_out/ab86_${v}_$i.json'))
k=d['kernels']; print('$v', d['value'], d['ms_per_step'], 'colsum', round(k['colsum']['ms'],1), 'norm', round(k['norm']['ms'],1), 'gemm', round(k['gemm']['ms'],1), d['clocks']['sm_mhz'])"
  done
done
