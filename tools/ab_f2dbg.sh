# attention forward with the softmax exponentials replaced by an FMA (MARIO_F2_DBG=1, wrong results):
# how much of the kernel the SFU / softmax arithmetic costs
mkdir -p gpurun_out
cat > /tmp/f2.py <<'PY'
import json, os, sys, torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib
L = _lib.lib()
st = os.environ.get("F2", "3")
for (B, s, nh, dh) in [(4, 2048, 32, 64), (4, 2048, 16, 128)]:
    if st == "5" and dh == 128: continue
    h = nh * dh
    qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
    O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
    lse = torch.empty(nh, B * s, device="cuda")
    L.mario_k_attn_set_variant(3)
    f = lambda: L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None)
    for _ in range(3): assert f() == 0
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(20): f()
    e1.record(); torch.cuda.synchronize()
    print(json.dumps({"stages": st, "shape": [B, s, nh, dh], "us": round(e0.elapsed_time(e1) / 20 * 1e3, 1)}), flush=True)
PY
mkdir -p gpurun_out
for n in 1 0; do
  NVCC_EXTRA="-DMARIO_F2_DBG=$n" python -c "from paper_conf_ppopp_liultj25_b200 import build; build.build()" > gpurun_out/f2dbg_build_$n.log 2>&1
  F2=dbg$n timeout 300 python /tmp/f2.py >> gpurun_out/f2dbg.jsonl 2>&1
done
