# refresh measurements with the final kernels: tuner with measured estimators (cfg 2/3/4, 8 GPUs x 40 GB)
# and the 2- / 4-stage emulated cfg-2 pipelines
mkdir -p gpurun_out
for c in cfg2 cfg3 cfg4; do timeout 900 python tools/tune_measured.py $c 40 > gpurun_out/tune_${c}_s2.json 2> gpurun_out/tune_${c}_s2.err; done
for n in 2 4; do timeout 900 python bench.py --emulate-only --emulate $n --steps 2 --warmup 2 > gpurun_out/emu_cfg2_s${n}_s2.json 2> gpurun_out/emu_cfg2_s${n}_s2.err; done
