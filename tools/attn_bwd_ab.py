"""Attention backward (production path: dK/dV kernel + dS image + dQ-from-image) at the bench shapes,
event-timed through the C-ABI, plus its error against float64 torch math on sampled heads. Run once
per setting of a launch-time env knob (e.g. MARIO_ATTN_BWD_POLY=0/1) to A/B it."""
import json
import os
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()
L.mario_k_attn_bwd_ws_bytes.restype = __import__("ctypes").c_size_t
tag = {k: v for k, v in os.environ.items() if k.startswith("MARIO_ATTN")}
for (B, s, nh, dh) in [(4, 2048, 16, 128), (1, 4096, 32, 128), (2, 2048, 32, 128)]:
    h = nh * dh
    torch.manual_seed(0)
    qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
    O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
    lse = torch.empty(nh, B * s, device="cuda")
    dO = torch.randn(B * s, h, device="cuda").bfloat16()
    dq = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
    scr = torch.empty(nh, B * s, device="cuda")
    wsb = L.mario_k_attn_bwd_ws_bytes(B, s, nh, dh)
    ws = torch.empty(max(wsb, 16), device="cuda", dtype=torch.uint8)
    assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0

    def bwd():
        return L.mario_k_attn_bwd_ws(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(),
                                     scr.data_ptr(), ws.data_ptr(), wsb, B, s, nh, dh, None)
    for _ in range(3):
        assert bwd() == 0
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(20):
        bwd()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 20
    fl = 8.0 * B * nh * dh * s * (s + 1) / 2
    # reference on two heads of sample 0 (float64, causal)
    errs = []
    for hd in (0, nh - 1):
        q, k, v = (qkv[:s, j * h + hd * dh: j * h + (hd + 1) * dh].double().requires_grad_() for j in range(3))
        S = (q @ k.T) / dh ** 0.5
        S = S.masked_fill(torch.ones(s, s, device="cuda", dtype=torch.bool).triu(1), float("-inf"))
        o = torch.softmax(S, -1) @ v
        o.backward(dO[:s, hd * dh:(hd + 1) * dh].double())
        for j, t in enumerate((q, k, v)):
            got = dq[:s, j * h + hd * dh: j * h + (hd + 1) * dh].double()
            errs.append(float((got - t.grad).abs().max() / t.grad.abs().max()))
    if os.environ.get("ATTN_AB_SAVE"):
        torch.save(dq.cpu(), f"{os.environ['ATTN_AB_SAVE']}_{B}_{s}_{nh}.pt")
    print(json.dumps({"shape": [B, s, nh, dh], "env": tag, "bwd_us": round(ms * 1e3, 1),
                      "tflops": round(fl / ms / 1e9, 1), "max_rel_err_dq_dk_dv": round(max(errs), 5)}), flush=True)
