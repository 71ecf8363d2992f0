# --set full of one backward layer's GEMMs (fc2 dgrad with GeLU' aux + colsum, wgrads, dgrads)
mkdir -p gpurun_out
B="python bench.py --micro 2 --steps 1 --warmup 3 --graphs 0 --no-cpu-baseline --no-e2e --no-projection"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc2 -s 200 -c 12 -o gpurun_out/prof_gemm90 $B > /dev/null 2>&1
echo rc $?
