# recomputing dQ kernel: 64-key tiles (fa_bwd_dq_pers) vs 128-key tiles (fa_bwd_dq_n128), through the
# no-workspace C-ABI path (cfg 5 uses it): time and bitwise dQKV; attention tests with the N128 dQ kernel
mkdir -p gpurun_out
cat > /tmp/dq_ab.py <<'PY'
import json, os, sys, torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib
L = _lib.lib()
tag = os.environ.get("MARIO_ATTN_DQ_N128", "0")
for (B, s, nh, dh) in [(4, 2048, 16, 128), (1, 16384, 8, 128), (1, 4096, 32, 128), (2, 2048, 16, 64)]:
    h = nh * dh
    torch.manual_seed(0)
    qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
    O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
    lse = torch.empty(nh, B * s, device="cuda")
    dO = torch.randn(B * s, h, device="cuda").bfloat16()
    dq = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
    scr = torch.empty(nh, B * s, device="cuda")
    assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0
    f = lambda: L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(), scr.data_ptr(), B, s, nh, dh, 1, None)
    for _ in range(3): assert f() == 0
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(10): f()
    e1.record(); torch.cuda.synchronize()
    torch.save(dq.cpu(), f"gpurun_out/dqn_{tag}_{B}_{s}_{nh}_{dh}.pt")
    print(json.dumps({"shape": [B, s, nh, dh], "dq_n128": tag, "bwd_us": round(e0.elapsed_time(e1) / 10 * 1e3, 1)}), flush=True)
PY
for v in 0 1 0 1; do MARIO_ATTN_DQ_N128=$v timeout 300 python /tmp/dq_ab.py >> gpurun_out/dq_n128.jsonl 2>&1; done
python - <<'PY' >> gpurun_out/dq_n128.jsonl
import torch, glob
for f in sorted(glob.glob("gpurun_out/dqn_0_*.pt")):
    a, b = torch.load(f), torch.load(f.replace("dqn_0", "dqn_1"))
    print({"file": f, "bitwise_equal": bool(torch.equal(a, b)), "max_abs": float((a.float() - b.float()).abs().max())})
PY
rm -f gpurun_out/dqn_*.pt
MARIO_ATTN_DQ_N128=1 timeout 600 python -m pytest tests/test_gpu_attention.py -x -q > gpurun_out/dq_n128_tests.log 2>&1
echo "rc=$?" >> gpurun_out/dq_n128_tests.log
