"""Attention forward through the C-ABI at the cfg-2 / cfg-4 shapes for each forward variant (-1 auto, 2 one-Q-tile, 3 two-Q-tile)."""
import json, sys, torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib
L = _lib.lib()
for (B, s, nh, dh) in [(1, 2048, 32, 80), (1, 2048, 32, 128), (4, 2048, 16, 128), (1, 2048, 20, 128)]:
    h = nh * dh
    qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
    O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
    lse = torch.empty(nh, B * s, device="cuda")
    for var in (-1, 2, 3):
        L.mario_k_attn_set_variant(var)
        f = lambda: L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None)
        for _ in range(3): assert f() == 0
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        for _ in range(20): f()
        e1.record(); torch.cuda.synchronize()
        print(json.dumps({"shape": [B, s, nh, dh], "variant": var, "us": round(e0.elapsed_time(e1) / 20 * 1e3, 1)}), flush=True)
    L.mario_k_attn_set_variant(-1)
