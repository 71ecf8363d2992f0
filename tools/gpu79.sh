run() { echo "== $*"; env "$@" timeout 120 python tools/bw_perf.py 2 2>&1 | grep '"h": 2048' | grep -v copy | python -c "
import sys,json
print(' '.join(f\"{json.loads(l)['kernel'][:14]}={json.loads(l)['us']}\" for l in sys.stdin))"; }
run X=0
run MARIO_NORM_FWD_RING=49152 MARIO_NORM_FWD_SMAX=12
run MARIO_NORM_FWD_RING=16384 MARIO_NORM_FWD_SMAX=4
run MARIO_NORM_FWD_RING=12288 MARIO_NORM_FWD_SMAX=4
run MARIO_NORM_BWD_RING=98304 MARIO_NORM_BWD_SMAX=8
run MARIO_NORM_BWD_RING=24576 MARIO_NORM_BWD_SMAX=4
run MARIO_NORM_BWD_RING=36864 MARIO_NORM_BWD_SMAX=6
