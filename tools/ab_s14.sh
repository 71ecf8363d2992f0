# column-sum reduction: 32-warp one-round-trip kernel vs the 16-warp one (MARIO_COLSUM_REDUCE=16), bench
# A/B; norm tests; ncu of fa_bwd_dq_img and fa_bwd_dkdv_n128 on the workspace path
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_norm.py tests/test_gpu_gemm.py -x -q > gpurun_out/t_s14.log 2>&1; echo "rc=$?" >> gpurun_out/t_s14.log
B="python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --emulate 0"
for v in 32 16 32 16; do
  MARIO_COLSUM_REDUCE=$v timeout 600 $B > gpurun_out/cr_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/cr_$v.json').read().strip().splitlines()[-1])
k=d['kernels']; print('colsum_reduce=$v', round(d['value'],2), 'norm', round(k['norm']['ms'],1), 'colsum', round(k['colsum']['ms'],1), 'step', round(k['step_ms'],1), d['clocks']['sm_mhz'])" >> gpurun_out/ab_s14.txt
done
for k in fa_bwd_dq_img fa_bwd_dkdv_n128; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o gpurun_out/profws_$k \
    python tools/attn_one_ws.py > gpurun_out/profws_$k.log 2>&1
  ncu -i gpurun_out/profws_$k.ncu-rep --page raw --csv > gpurun_out/rawws_$k.csv 2>/dev/null
  gzip -f gpurun_out/rawws_$k.csv
  rm -f gpurun_out/profws_$k.ncu-rep
done
