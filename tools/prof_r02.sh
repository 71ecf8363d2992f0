# Round-2 profiling evidence (run under gpurun, 1 GPU): launch list of one eager step of the bench
# workload and --set full captures of the top kernels; raw-page CSVs are kept (small), the .ncu-rep
# files only where small. Summaries go to profiles/r02/.
set -x
mkdir -p gpurun_out
B="python bench.py --steps 1 --warmup 2 --graphs 0 --no-cpu-baseline --no-e2e --emulate 0"
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -s 19000 -c 10000 --csv \
  --log-file gpurun_out/launches_r02.csv $B > gpurun_out/launches_r02.log 2>&1
gzip -f gpurun_out/launches_r02.csv
for k in norm_bwd_pipe_k fa_bwd_dkdv_ts fa_bwd_dq_img softmax_ce_reg_k norm_fwd_pipe_k norm_apply_k gemm_bf16_tc2; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 60 -c 2 \
    -o gpurun_out/prof_$k $B --micro 2 > gpurun_out/prof_$k.log 2>&1
  ncu -i gpurun_out/prof_$k.ncu-rep --page raw --csv > gpurun_out/raw_$k.csv 2>/dev/null
  gzip -f gpurun_out/raw_$k.csv
  rm -f gpurun_out/prof_$k.ncu-rep
done
du -sh gpurun_out
