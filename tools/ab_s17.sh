# attention D = rowsum(dO o O) fused into the dO GEMM epilogue (MARIO_FUSE_D=1) vs the separate kernel
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_gemm.py tests/test_gpu_attention.py tests/test_gpu_s8.py -x -q > gpurun_out/t_s17.log 2>&1; echo "rc=$?" >> gpurun_out/t_s17.log
B="python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for v in 1 0 1 0; do
  MARIO_FUSE_D=$v timeout 600 $B > gpurun_out/fd_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/fd_$v.json').read().strip().splitlines()[-1])
k=d['kernels']; print('fuse_D=$v', round(d['value'],2), 'gemm', round(k['gemm']['ms'],1), 'attn_bwd', round(k['attn_bwd']['ms'],1), 'step', round(k['step_ms'],1), d['clocks']['sm_mhz'])" >> gpurun_out/ab_s17.txt
done
