# A/B of MARIO_GEMM_OVERLAP (independent backward wgrads on a side stream, non-persistent, filling the
# dgrad's last wave) on whole bench steps, plus bitwise checks with it on.
mkdir -p gpurun_out
MARIO_GEMM_OVERLAP=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_peer.py -q -m gpu -x \
  -k "bitwise or fp32_parity or bf16_parity or full_width" > gpurun_out/ov_tests.log 2>&1
tail -n 2 gpurun_out/ov_tests.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for i in 1 2; do for v in 0 1; do
  MARIO_GEMM_OVERLAP=$v timeout 600 $B > gpurun_out/ov_${v}_${i}.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/ov_${v}_${i}.json').read().strip().splitlines()[-1])
k=d['kernels']; print('overlap=$v', round(d['value'],2), 'ms', round(d['ms_per_step'],1), 'gemm', round(k['gemm']['ms'],1), d['clocks']['sm_mhz'])"
done; done
