# qkv-bias column sums from the attention kernels (MARIO_FUSE_QKVB=1) vs the separate column-sum pass (0)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_attention.py tests/test_gpu_s8.py -x -q > gpurun_out/t_s18.log 2>&1; echo "rc=$?" >> gpurun_out/t_s18.log
B="python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for v in 1 0 1 0; do
  MARIO_FUSE_QKVB=$v timeout 600 $B > gpurun_out/qb_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/qb_$v.json').read().strip().splitlines()[-1])
k=d['kernels']; print('fuse_qkvb=$v', round(d['value'],2), 'attn_bwd', round(k['attn_bwd']['ms'],1), 'colsum', round(k['colsum']['ms'],1), 'step', round(k['step_ms'],1), d['clocks']['sm_mhz'])" >> gpurun_out/ab_s18.txt
done
