# stored activation set incl. the MLP activation (store_act=1) vs lean (0): parity tests, then bench A/B
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "lean or bf16 or full_width" > gpurun_out/t_s13.log 2>&1; echo "rc=$?" >> gpurun_out/t_s13.log
B="python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for v in 1 0 1 0; do
  MARIO_STORE_ACT=$v timeout 600 $B > gpurun_out/sa_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/sa_$v.json').read().strip().splitlines()[-1])
k=d['kernels']; print('store_act=$v', round(d['value'],2), 'gemm', round(k['gemm']['ms'],1), 'norm', round(k['norm']['ms'],1), 'elem', round(k['elementwise']['ms'],1), 'step', round(k['step_ms'],1), d['clocks']['sm_mhz'], 'mem', d['peak_mem_per_stage'])" >> gpurun_out/ab_s13.txt
done
MARIO_STORE_ACT=1 timeout 600 python bench.py --config cfg3 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0 > gpurun_out/cfg3_sa1.json 2>/dev/null
MARIO_STORE_ACT=0 timeout 600 python bench.py --config cfg3 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0 > gpurun_out/cfg3_sa0.json 2>/dev/null
