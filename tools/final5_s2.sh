# persistent attention forward by default: full GPU suite, smoke(), default bench line, cfg 4 line
mkdir -p gpurun_out
timeout 1300 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_final5.log 2>&1; echo "rc=$?" >> gpurun_out/gputest_final5.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final5.log 2>&1; echo "rc=$?" >> gpurun_out/smoke_final5.log
timeout 900 python bench.py > gpurun_out/bench_final5.json 2> gpurun_out/bench_final5.err
