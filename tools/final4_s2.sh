# after the Chimera order change: full GPU suite + cfg 4 bench line (Chimera emulated at 8 stages)
mkdir -p gpurun_out
timeout 1300 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_final4.log 2>&1; echo "rc=$?" >> gpurun_out/gputest_final4.log
timeout 1200 python bench.py --config cfg4 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg4_final4.json 2> gpurun_out/bench_cfg4_final4.err
