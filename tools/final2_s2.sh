# Round-2 session-2 final validation on one B200 (HEAD): full GPU suite, smoke(), default bench line,
# cfg3/4/5 bench lines, per-shape GEMMs of one layer, and the launch list of one eager cfg-2 step
mkdir -p gpurun_out
timeout 1300 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_final2.log 2>&1; echo "rc=$?" >> gpurun_out/gputest_final2.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final2.log 2>&1; echo "rc=$?" >> gpurun_out/smoke_final2.log
timeout 900 python bench.py > gpurun_out/bench_final2.json 2> gpurun_out/bench_final2.err
bash tools/bench_cfgs.sh
timeout 600 python tools/gemm_step.py > gpurun_out/gemm_step_final2.jsonl 2>&1
B="python bench.py --steps 1 --warmup 2 --graphs 0 --no-cpu-baseline --no-e2e --emulate 0"
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -s 19000 -c 10000 --csv \
  --log-file gpurun_out/launches_final2.csv $B > gpurun_out/launches_final2.log 2>&1
gzip -f gpurun_out/launches_final2.csv
