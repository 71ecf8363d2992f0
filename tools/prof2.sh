mkdir -p gpurun_out
B="python bench.py --micro 2 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-projection"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches2.csv $B > gpurun_out/launches2_stdout.log 2>&1
echo "launch list rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fa_fwd_tc -c 1 -o gpurun_out/prof_fa_fwd $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc2 -s 10 -c 3 -o gpurun_out/prof_gemm2 $B > /dev/null 2>&1
echo done
