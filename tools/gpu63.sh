mkdir -p gpurun_out
B="python bench.py --micro 2 --steps 1 --warmup 3 --graphs 0 --no-cpu-baseline --no-e2e --no-projection"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches63.csv $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc2 -s 40 -c 4 -o gpurun_out/prof_gemm63 $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"fa_bwd_dkdv_ts|fa_bwd_dq_img|fa_fwd2" -s 6 -c 3 -o gpurun_out/prof_attn63 $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:"norm_|softmax_ce|colsum" -s 40 -c 8 -o gpurun_out/prof_bw63 $B > /dev/null 2>&1
ls -la gpurun_out
