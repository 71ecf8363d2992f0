mkdir -p gpurun_out
B="python bench.py --micro 2 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B > gpurun_out/launches_stdout.log 2>&1
echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc -s 40 -c 3 -o gpurun_out/prof_gemm $B > gpurun_out/prof_gemm.log 2>&1
echo "gemm prof rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fa_ -s 6 -c 4 -o gpurun_out/prof_attn $B > gpurun_out/prof_attn.log 2>&1
echo "attn prof rc=$?"
ls -la gpurun_out
