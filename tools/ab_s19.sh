# fused qkv-bias sums with 16-byte column reads in the dK/dV epilogue: tests + bench A/B vs the column-sum pass
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "qkv_bias or full_width or lean" > gpurun_out/t_s19.log 2>&1; echo "rc=$?" >> gpurun_out/t_s19.log
B="python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for v in 1 0 1 0; do
  MARIO_FUSE_QKVB=$v timeout 600 $B > gpurun_out/qc_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/qc_$v.json').read().strip().splitlines()[-1])
k=d['kernels']; print('fuse_qkvb=$v', round(d['value'],2), 'attn_bwd', round(k['attn_bwd']['ms'],1), 'colsum', round(k['colsum']['ms'],1), 'step', round(k['step_ms'],1), d['clocks']['sm_mhz'])" >> gpurun_out/ab_s19.txt
done
