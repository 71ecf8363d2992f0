# norm backward CTAs per SM (3 by occupancy vs 1 or 2, with a deeper ring) on whole bench steps
mkdir -p gpurun_out
B="python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for v in "0 49152" "1 98304" "2 65536" "0 49152" "1 98304" "2 65536"; do set -- $v
  MARIO_NORM_BWD_CPS=$1 MARIO_NORM_BWD_RING=$2 MARIO_NORM_BWD_SMAX=8 timeout 600 $B > gpurun_out/nc_$1.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/nc_$1.json').read().strip().splitlines()[-1])
k=d['kernels']; print('cps=$1 ring=$2', round(d['value'],2), 'norm', round(k['norm']['ms'],1), 'step', round(k['step_ms'],1), d['clocks']['sm_mhz'])" >> gpurun_out/ab_normcps.txt
done
