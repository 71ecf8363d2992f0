# ncu --set full of the attention forward (fa_fwd2_tc, cfg-2 shape) with source correlation
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fa_fwd2_tc -s 1 -c 1 -o gpurun_out/prof_fwd2 \
  python tools/attn_one.py > gpurun_out/prof_fwd2.log 2>&1
ncu -i gpurun_out/prof_fwd2.ncu-rep --page raw --csv > gpurun_out/raw_fwd2.csv 2>/dev/null
ncu -i gpurun_out/prof_fwd2.ncu-rep --page source --csv --print-source sass > gpurun_out/src_fwd2.csv 2>/dev/null
ncu -i gpurun_out/prof_fwd2.ncu-rep --page details --csv > gpurun_out/details_fwd2.csv 2>/dev/null
gzip -f gpurun_out/raw_fwd2.csv gpurun_out/src_fwd2.csv
