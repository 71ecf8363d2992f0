# A/B of two library builds on one box, alternating: bench value + per-family ms
for i in 1 2; do for v in K J; do
MARIO_LIB=$PWD/ab/libmario_$v.so timeout 900 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-projection 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']
print('$v', round(d['value'],3), 'clk', d['clocks']['sm_mhz'], ' '.join(f'{n}={round(v[\"ms\"],1)}' for n,v in k.items() if isinstance(v,dict)))"
done; done
