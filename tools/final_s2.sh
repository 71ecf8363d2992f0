# Round-2 session-2 validation on one B200: full GPU suite, smoke(), the default bench line, cfg3/4/5 bench
# lines, and the launch list of one eager cfg-2 step (ncu gpu__time_duration, share of step)
mkdir -p gpurun_out
timeout 1300 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_final.log 2>&1; echo "rc=$?" >> gpurun_out/gputest_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1; echo "rc=$?" >> gpurun_out/smoke_final.log
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
bash tools/bench_cfgs.sh
B="python bench.py --steps 1 --warmup 2 --graphs 0 --no-cpu-baseline --no-e2e --emulate 0"
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -s 19000 -c 10000 --csv \
  --log-file gpurun_out/launches_s2.csv $B > gpurun_out/launches_s2.log 2>&1
gzip -f gpurun_out/launches_s2.csv
