# 128-query dK/dV kernel: one CTA per item (PERS=0) vs persistent snake order (PERS=1), against the
# 64-query kernel (N128=0): time, error, bitwise dQKV; attention tests with PERS=1.
mkdir -p gpurun_out
MARIO_ATTN_DKDV_N128=0 ATTN_AB_SAVE=gpurun_out/dq_ref timeout 300 python tools/attn_bwd_ab.py 2>/dev/null >> gpurun_out/attn_pers.jsonl
for p in 0 1 0 1; do MARIO_ATTN_DKDV_PERS=$p ATTN_AB_SAVE=gpurun_out/dq_p$p timeout 300 python tools/attn_bwd_ab.py 2>/dev/null >> gpurun_out/attn_pers.jsonl; done
python - <<'PY' >> gpurun_out/attn_pers.jsonl
import torch, glob
for f in sorted(glob.glob("gpurun_out/dq_ref_*.pt")):
    a = torch.load(f)
    for p in (0, 1):
        b = torch.load(f.replace("dq_ref", f"dq_p{p}"))
        print({"file": f, "pers": p, "bitwise_equal_to_64q": bool(torch.equal(a, b))})
PY
rm -f gpurun_out/dq_*.pt
MARIO_ATTN_DKDV_PERS=1 timeout 600 python -m pytest tests/test_gpu_attention.py -x -q > gpurun_out/attn_pers_tests.log 2>&1
echo "rc=$?" >> gpurun_out/attn_pers_tests.log
timeout 600 python -m pytest tests/test_gpu_attention.py -x -q >> gpurun_out/attn_pers_tests.log 2>&1
echo "rc=$?" >> gpurun_out/attn_pers_tests.log
