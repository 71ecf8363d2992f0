# dK/dV attention backward: tensor-pipe drain between the dV/dK MMAs of tile i and the S/dP MMAs of
# tile i + 2 (INORDER=0) vs relying on tcgen05.mma's issue-order execution (INORDER=1): time, error
# vs float64, and bitwise equality of dQKV between the two.
mkdir -p gpurun_out
for p in 0 1 0 1; do MARIO_ATTN_BWD_INORDER=$p ATTN_AB_SAVE=gpurun_out/dq_io$p timeout 300 python tools/attn_bwd_ab.py 2>/dev/null >> gpurun_out/attn_inorder.jsonl; done
python - <<'PY' >> gpurun_out/attn_inorder.jsonl
import torch, glob
for f in sorted(glob.glob("gpurun_out/dq_io0_*.pt")):
    a, b = torch.load(f), torch.load(f.replace("io0", "io1"))
    print({"file": f, "bitwise_equal": bool(torch.equal(a, b))})
PY
rm -f gpurun_out/dq_io*.pt
MARIO_ATTN_BWD_INORDER=1 timeout 600 python -m pytest tests/test_gpu_attention.py -x -q > gpurun_out/attn_inorder_tests.log 2>&1
echo "rc=$?" >> gpurun_out/attn_inorder_tests.log
