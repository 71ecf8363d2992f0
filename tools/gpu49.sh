mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"fa_bwd_dq_pers|fa_bwd_dkdv" -c 2 -o gpurun_out/prof_bwd6 python tools/attn_bwd_exp.py 0 > /dev/null 2>&1
echo rc=$?
