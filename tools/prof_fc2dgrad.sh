mkdir -p gpurun_out
for sk in 1 4; do
  timeout 600 ncu --set full --clock-control none -k regex:gemm_bf16_tc2 -s $sk -c 1 -o gpurun_out/prof_fc2dg_$sk python tools/gemm_fc2dgrad.py > gpurun_out/prof_fc2dg_$sk.log 2>&1
  ncu -i gpurun_out/prof_fc2dg_$sk.ncu-rep --page raw --csv > gpurun_out/raw_fc2dg_$sk.csv 2>/dev/null
  gzip -f gpurun_out/raw_fc2dg_$sk.csv; rm -f gpurun_out/prof_fc2dg_$sk.ncu-rep
done
