"""Time attention fwd/bwd through the C-ABI at the config-2 shape for each kernel variant."""
import sys, json
import torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib, api  # noqa
L = _lib.lib()
for (B, s, nh, dh) in [(4, 2048, 16, 128), (1, 4096, 32, 128), (1, 2048, 32, 64)]:
    h = nh * dh
    qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
    O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
    lse = torch.empty(nh, B * s, device="cuda")
    dO = torch.randn(B * s, h, device="cuda").bfloat16()
    dq = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
    scr = torch.empty(nh, B * s, device="cuda")
    fl_f = 4.0 * B * nh * dh * s * (s + 1) / 2
    for variant in (0, -1):
        L.mario_k_attn_set_variant(variant)
        def fwd(): return L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None)
        def bwd(): return L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(), scr.data_ptr(), B, s, nh, dh, 1, None)
        res = {}
        for name, f, fl in (("fwd", fwd, fl_f), ("bwd", bwd, 2 * fl_f)):
            for _ in range(3): assert f() == 0
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record()
            for _ in range(10): f()
            e1.record(); torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / 10
            res[name] = (round(ms, 3), round(fl / ms / 1e9, 1))
        print(json.dumps({"shape": [B, s, nh, dh], "variant": variant, "fwd_ms_tflops": res["fwd"], "bwd_ms_tflops": res["bwd"]}), flush=True)
