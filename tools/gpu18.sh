timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -2
timeout 1500 python bench.py --steps 3 --warmup 3 2>&1 | tail -1 > gpurun_out/bench_latest.json; cat gpurun_out/bench_latest.json | cut -c1-1500
