timeout 600 python -m pytest tests/test_gpu_attention.py -x -q 2>&1 | tail -1
for v in 0 1; do MARIO_ATTN_L2HINT=$v timeout 300 python tools/attn_bwd_exp.py 0 2>&1 | tail -1 | sed "s/^/hint$v /"; MARIO_ATTN_L2HINT=$v timeout 300 python tools/attn_perf.py 2>&1 | grep '"variant": -1' | head -1 | sed "s/^/hint$v /"; done
for i in 1 2; do for v in 0 1; do
MARIO_ATTN_L2HINT=$v timeout 900 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-projection 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']
print('hint$v', round(d['value'],3), 'clk', d['clocks']['sm_mhz'], ' '.join(f'{n}={round(v[\"ms\"],1)}' for n,v in k.items() if isinstance(v,dict)))"
done; done
