# full GPU suite, default bench line, and ncu --set full of the attention backward kernels (cfg-2 shape)
mkdir -p gpurun_out
timeout 1300 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_s7.log 2>&1; echo "rc=$?" >> gpurun_out/gputest_s7.log
timeout 900 python bench.py > gpurun_out/bench_s7.json 2> gpurun_out/bench_s7.err
for k in fa_bwd_dkdv_n128 fa_bwd_dq_img; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o gpurun_out/prof_$k \
    python tools/attn_one.py > gpurun_out/prof_$k.log 2>&1
  ncu -i gpurun_out/prof_$k.ncu-rep --page raw --csv > gpurun_out/raw_$k.csv 2>/dev/null
  ncu -i gpurun_out/prof_$k.ncu-rep --page details --csv > gpurun_out/details_$k.csv 2>/dev/null
  gzip -f gpurun_out/raw_$k.csv
done
