mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q 2>&1 | tail -1
timeout 300 python tools/gemm_step.py 2>&1 | grep "fc2 dgrad\|fc1 fwd"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc2 -s 5 -c 1 -o gpurun_out/prof_fc2dgrad python tools/gemm_step.py > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_bf16_tc2 -s 2 -c 1 -o gpurun_out/prof_fc1fwd python tools/gemm_step.py > /dev/null 2>&1
ls gpurun_out
