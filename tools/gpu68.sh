timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q 2>&1 | tail -1
for v in F G; do MARIO_LIB=$PWD/ab/libmario_$v.so timeout 300 python tools/gemm_step.py 2>&1 | tail -16 | python -c "
import sys,json
t=[]
for l in sys.stdin:
    d=json.loads(l); t.append(f\"{d.get('gemm','TOTAL')}={d.get('us_epi', d.get('layer_ms'))}\")
print('$v', ' '.join(t))"; done
bash tools/gpu65.sh
