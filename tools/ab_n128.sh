# dK/dV attention backward: 64-query tiles (fa_bwd_dkdv_ts) vs 128-query tiles (fa_bwd_dkdv_n128,
# POLY 0/2/4): time, error vs float64, bitwise equality of dQKV against the 64-query kernel; then the
# attention tests and the bf16 parity cases with the N128 kernel.
mkdir -p gpurun_out
MARIO_ATTN_DKDV_N128=0 ATTN_AB_SAVE=gpurun_out/dq_n0 timeout 300 python tools/attn_bwd_ab.py 2>/dev/null >> gpurun_out/attn_n128.jsonl
for p in 0 2 4; do MARIO_ATTN_DKDV_N128=1 MARIO_ATTN_BWD_POLY=$p ATTN_AB_SAVE=gpurun_out/dq_n1p$p timeout 300 python tools/attn_bwd_ab.py 2>/dev/null >> gpurun_out/attn_n128.jsonl; done
MARIO_ATTN_DKDV_N128=0 timeout 300 python tools/attn_bwd_ab.py 2>/dev/null >> gpurun_out/attn_n128.jsonl
python - <<'PY' >> gpurun_out/attn_n128.jsonl
import torch, glob
for f in sorted(glob.glob("gpurun_out/dq_n0_*.pt")):
    a = torch.load(f)
    for p in (0, 2, 4):
        b = torch.load(f.replace("n0", f"n1p{p}"))
        print({"file": f, "poly": p, "bitwise_equal": bool(torch.equal(a, b)),
               "max_abs_diff": float((a.float() - b.float()).abs().max())})
PY
rm -f gpurun_out/dq_n*.pt
MARIO_ATTN_DKDV_N128=1 timeout 600 python -m pytest tests/test_gpu_attention.py -x -q > gpurun_out/attn_n128_tests.log 2>&1
echo "rc=$?" >> gpurun_out/attn_n128_tests.log
