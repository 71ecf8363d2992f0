mkdir -p gpurun_out
for v in "1 8" "1 32" "0 32"; do set -- $v
  MARIO_PEER_RX=$1 CUDA_DEVICE_MAX_CONNECTIONS=$2 timeout 600 python bench.py --emulate-only --steps 2 > gpurun_out/emu_rx$1_c$2.json 2>gpurun_out/emu_rx$1_c$2.err
  python -c "
import json,sys; d=json.load(open('gpurun_out/emu_rx$1_c$2.json'))['pipeline_emulated']
print('rx=$1 conn=$2', {k:(round(v['ms_per_iter']),round(v['bubble_measured'],3),round(v['bubble_simulated'],3),round(v['makespan_simulated_ms'])) for k,v in d['levels'].items()}, 'mario/ckpt', round(d['mario_vs_ckpt'],3))"
done
