# Round-2 session-2 A/B (1 GPU): norm forward kernels per shape, then whole bench steps with the stored
# vs lean activation set (MARIO_STORE_NORM) and norm forward variant 2 (row pipeline) vs 3 (warp/row).
mkdir -p gpurun_out
timeout 300 python tools/norm_fwd_perf.py > gpurun_out/norm_fwd_perf.jsonl 2>&1
B="python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for v in "0 2" "1 2" "1 3" "0 2" "1 2" "1 3"; do set -- $v
  MARIO_STORE_NORM=$1 MARIO_NORM_VARIANT=$2 timeout 600 $B > gpurun_out/ab_$1$2.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/ab_$1$2.json').read().strip().splitlines()[-1])
k=d['kernels']; print('store=$1 normvar=$2', round(d['value'],2), 'norm', round(k['norm']['ms'],1), 'colsum', round(k['colsum']['ms'],1), 'step', round(k['step_ms'],1), d['clocks']['sm_mhz'])" >> gpurun_out/ab_s2.txt
done
