# Extra bench lines (1 GPU): cfg3 (LLaMA2-7B, Interleave emulated at 8 stages), cfg4 (GPT-3 2.7B with
# dh 80 on the padded tcgen05 attention, Chimera emulated at 8 stages), cfg5 per-layer (s 16384).
mkdir -p gpurun_out
timeout 1500 python bench.py --config cfg3 --steps 2 --warmup 3 --no-cpu-baseline --emulate-levels ckpt,mario \
  > gpurun_out/bench_cfg3.json 2> gpurun_out/bench_cfg3.err
timeout 1200 python bench.py --config cfg4 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg4.json \
  2> gpurun_out/bench_cfg4.err
timeout 900 python bench.py --config cfg5 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_cfg5.json \
  2> gpurun_out/bench_cfg5.err
for c in cfg3 cfg4 cfg5; do tail -c 400 gpurun_out/bench_$c.err; done
