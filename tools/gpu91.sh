# evict_first on the GeLU' epilogue streams (MARIO_EPI_EF): GEMM + parity tests on ef1, A/B ef0/ef1, fc2 dgrad DRAM bytes
mkdir -p gpurun_out
MARIO_LIB=ab/libmario_ef1.so timeout 900 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_parity.py -m gpu -q -x 2>&1 | tail -2
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-projection"
for i in 1 2; do
  for v in ef0 ef1; do
    MARIO_LIB=ab/libmario_$v.so timeout 600 $B 2>&1 | tail -1 > gpurun_out/ab91_${v}_$i.json
    python -c "
import json; d=json.load(open('gpurun_out/ab91_${v}_$i.json'))
k=d['kernels']; print('$v', d['value'], d['ms_per_step'], 'gemm', round(k['gemm']['ms'],1), 'attn_bwd', round(k['attn_bwd']['ms'],1), 'norm', round(k['norm']['ms'],1), d['clocks']['sm_mhz'])"
  done
done
for v in ef0 ef1; do
MARIO_LIB=ab/libmario_$v.so timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:gemm_bf16_tc2 -s 200 -c 12 --csv --log-file gpurun_out/gemm91_$v.csv python bench.py --micro 2 --steps 1 --warmup 3 --graphs 0 --no-cpu-baseline --no-e2e --no-projection > /dev/null 2>&1
done
echo done
