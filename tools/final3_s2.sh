# Round-2 session-2 closing validation at HEAD: full GPU suite, smoke(), default bench line
mkdir -p gpurun_out
timeout 1300 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_final3.log 2>&1; echo "rc=$?" >> gpurun_out/gputest_final3.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final3.log 2>&1; echo "rc=$?" >> gpurun_out/smoke_final3.log
timeout 900 python bench.py > gpurun_out/bench_final3.json 2> gpurun_out/bench_final3.err
timeout 600 python bench.py --impl reference --steps 1 --warmup 0 > gpurun_out/bench_ref_final3.json 2> gpurun_out/bench_ref_final3.err
