import sys, torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib, api
L = _lib.lib()
for (B, s, nh, dh) in [(1, 64, 1, 128), (1, 200, 1, 128), (2, 200, 3, 128), (1, 64, 1, 16)]:
    h = nh * dh
    qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
    O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
    lse = torch.empty(nh, B * s, device="cuda")
    r = L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None)
    torch.cuda.synchronize(); print("fwd", B, s, nh, dh, r, flush=True)
    dO = torch.randn(B * s, h, device="cuda").bfloat16()
    dq = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
    scr = torch.empty(nh, B * s, device="cuda")
    r = L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(), scr.data_ptr(), B, s, nh, dh, 1, None)
    torch.cuda.synchronize(); print("bwd", B, s, nh, dh, r, flush=True)
