"""A/B of the attention backward dK/dV kernels at a given shape (default cfg 2: B 4, s 2048, 16 heads,
dh 128): run in two processes, MARIO_ATTN_DKDV_PERS=0 (fa_bwd_dkdv_ts) and =1 (fa_bwd_dkdv_pers); each
prints the CUDA-event time per call and a hash of dQKV (the two must be bitwise equal).

    MARIO_ATTN_DKDV_PERS=1 python tools/attn_pers_check.py [B s nh dh]
"""
import hashlib
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_liultj25_b200 import _lib, api  # noqa: E402,F401

B, s, nh, dh = (int(x) for x in (sys.argv[1:5] if len(sys.argv) >= 5 else (4, 2048, 16, 128)))
L = _lib.lib()
g = torch.Generator(device="cuda").manual_seed(11)
h = nh * dh
qkv = torch.randn(B * s, 3 * h, device="cuda", generator=g).bfloat16()
dO = torch.randn(B * s, h, device="cuda", generator=g).bfloat16()
O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
lse = torch.empty(nh, B * s, device="cuda")
assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0
scr = torch.empty(nh, B * s, device="cuda")
wsb = L.mario_k_attn_bwd_ws_bytes(B, s, nh, dh)
ws = torch.empty(max(wsb, 1), device="cuda", dtype=torch.uint8)
d = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)


def call():
    if wsb:
        return L.mario_k_attn_bwd_ws(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), d.data_ptr(),
                                     scr.data_ptr(), ws.data_ptr(), wsb, B, s, nh, dh, None)
    return L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), d.data_ptr(),
                              scr.data_ptr(), B, s, nh, dh, 1, None)


for _ in range(3):
    assert call() == 0
torch.cuda.synchronize()
ts = []
for _ in range(10):
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    call()
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
digest = hashlib.sha1(d.cpu().view(torch.int16).numpy().tobytes()).hexdigest()[:16]
ts.sort()
print(f"pers={os.environ.get('MARIO_ATTN_DKDV_PERS', '0')} B={B} s={s} nh={nh} dh={dh} "
      f"us_median={ts[len(ts) // 2] * 1e3:.1f} us_min={ts[0] * 1e3:.1f} dqkv_sha={digest}")
