"""One fwd + one bwd through the dS-workspace path (dK/dV kernel + dQ from the dS image) at the cfg-2
attention shape (B 4, s 2048, 16 heads, dh 128), for ncu captures of fa_bwd_dkdv_n128 / fa_bwd_dq_img."""
import ctypes
import sys
import torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib
L = _lib.lib()
L.mario_k_attn_bwd_ws_bytes.restype = ctypes.c_size_t
B, s, nh, dh = 4, 2048, 16, 128
h = nh * dh
qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
lse = torch.empty(nh, B * s, device="cuda")
dO = torch.randn(B * s, h, device="cuda").bfloat16()
dq = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
scr = torch.empty(nh, B * s, device="cuda")
wsb = L.mario_k_attn_bwd_ws_bytes(B, s, nh, dh)
ws = torch.empty(wsb, device="cuda", dtype=torch.uint8)
for _ in range(2):
    assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0
    assert L.mario_k_attn_bwd_ws(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(),
                                 scr.data_ptr(), ws.data_ptr(), wsb, B, s, nh, dh, None) == 0
torch.cuda.synchronize()
