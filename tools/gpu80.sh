timeout 300 python -m pytest tests/test_gpu_norm.py -x -q 2>&1 | tail -1
run() { echo "== $*"; env "$@" timeout 120 python tools/bw_perf.py 2 2>&1 | grep 'norm_bwd' | python -c "
import sys,json
print(' '.join(f\"h{json.loads(l)['h']}={json.loads(l)['us']}\" for l in sys.stdin))"; }
run MARIO_NORM_BWD_V=1
run MARIO_NORM_BWD_V=2
run MARIO_NORM_BWD_V=2 MARIO_NORM_BWD_RING=73728 MARIO_NORM_BWD_SMAX=6
run MARIO_NORM_BWD_V=2 MARIO_NORM_BWD_RING=98304 MARIO_NORM_BWD_SMAX=8
