# A/B of the norm kernel variants on whole bench steps (1 GPU): rows per iteration of the forward /
# backward row pipelines and the 1-D vs 2-D backward recompute (norm_apply).
mkdir -p gpurun_out
B="python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for v in "2 2 1" "2 2 2" "4 2 2" "4 4 2" "2 2 1" "4 4 2"; do set -- $v
  MARIO_NORM_FWD_R=$1 MARIO_NORM_BWD_R=$2 MARIO_NORM_APPLY=$3 timeout 600 $B > gpurun_out/nab_$1$2$3.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/nab_$1$2$3.json').read().strip().splitlines()[-1])
k=d['kernels']; print('fwdR=$1 bwdR=$2 apply=$3', round(d['value'],2), 'norm', round(k['norm']['ms'],1), 'step', round(k['step_ms'],1), d['clocks']['sm_mhz'])"
done
# GEMM: stream-K hybrid (last partial wave split by k-blocks) vs data-parallel tiles, per shape
timeout 600 python tools/gemm_step.py > gpurun_out/gemm_step_sk0.jsonl 2>&1
STREAMK=1 timeout 600 python tools/gemm_step.py > gpurun_out/gemm_step_sk1.jsonl 2>&1
paste -d' ' <(python -c "import json;[print(json.loads(l)['gemm'], json.loads(l)['us_epi']) for l in open('gpurun_out/gemm_step_sk0.jsonl') if 'gemm' in l]") <(python -c "import json;[print(json.loads(l)['us_epi']) for l in open('gpurun_out/gemm_step_sk1.jsonl') if 'gemm' in l]")
