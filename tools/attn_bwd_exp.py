"""Attention-backward experiments at the cfg-2 shape: dK/dV and dQ kernels timed separately, with
MARIO_ATTN_DBG knobs (1: no softmax math, 2: no S/dP MMAs, 4: no accumulate MMAs)."""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()
B, s, nh, dh = 4, 2048, 16, 128
h = nh * dh
qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
lse = torch.empty(nh, B * s, device="cuda")
dO = torch.randn(B * s, h, device="cuda").bfloat16()
dq = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
scr = torch.empty(nh, B * s, device="cuda")
L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None)
fl = 4.0 * B * nh * dh * s * (s + 1) / 2
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
for only in ("dkdv", "dq", ""):
    for dbg in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "0,1,2,4,6,3,5").split(",")]:
        os.environ["MARIO_ATTN_TC_ONLY"] = only
        if not only:
            del os.environ["MARIO_ATTN_TC_ONLY"]
        os.environ["MARIO_ATTN_DBG"] = str(dbg)
        f = lambda: L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(),
                                       scr.data_ptr(), B, s, nh, dh, 1, None)
        for _ in range(3):
            f()
        torch.cuda.synchronize()
        e0.record()
        for _ in range(10):
            f()
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        print(json.dumps({"kernel": only or "both", "dbg": dbg, "us": round(ms * 1e3, 1),
                          "alg_tflops_full_bwd": round(2 * fl / ms / 1e9, 1)}), flush=True)
        if not only and dbg:
            break
os.environ.pop("MARIO_ATTN_DBG", None)
# dQ from the stored dS image (mario_k_attn_bwd_ws)
wsb = L.mario_k_attn_bwd_ws_bytes(B, s, nh, dh)
ws = torch.empty(wsb, device="cuda", dtype=torch.uint8)
f = lambda: L.mario_k_attn_bwd_ws(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(),
                                  scr.data_ptr(), ws.data_ptr(), wsb, B, s, nh, dh, None)
for only in ("dkdv", ""):
    if only:
        os.environ["MARIO_ATTN_TC_ONLY"] = only
    else:
        os.environ.pop("MARIO_ATTN_TC_ONLY", None)
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    e0.record()
    for _ in range(10):
        f()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    print(json.dumps({"kernel": (only or "both") + "+ds_image", "ws_MB": round(wsb / 1e6, 1), "us": round(ms * 1e3, 1),
                      "alg_tflops_full_bwd": round(2 * fl / ms / 1e9, 1)}), flush=True)
