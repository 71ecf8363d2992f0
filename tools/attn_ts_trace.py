"""Per-tile clock64 timeline of fa_bwd_dkdv_ts (CTA 0 = key block 0, the longest item) plus CUDA-event
timings of the attention backward at the cfg-2 shape (B 4, s 2048, 16 heads, dh 128), dS image on.

    python tools/attn_ts_trace.py [B s nh dh]
"""
import os
import subprocess
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()
B, s, nh, dh = (int(x) for x in sys.argv[1:5]) if len(sys.argv) > 4 else (4, 2048, 16, 128)
h = nh * dh
g = torch.Generator(device="cuda").manual_seed(0)
qkv = torch.randn(B * s, 3 * h, device="cuda", generator=g).bfloat16()
O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
lse = torch.empty(nh, B * s, device="cuda")
dO = torch.randn(B * s, h, device="cuda", generator=g).bfloat16()
dq = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
scr = torch.empty(nh, B * s, device="cuda")
wsb = L.mario_k_attn_bwd_ws_bytes(B, s, nh, dh)
ws = torch.empty(max(wsb, 1), device="cuda", dtype=torch.uint8)
assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0


def bwd():
    return L.mario_k_attn_bwd_ws(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(),
                                 scr.data_ptr(), ws.data_ptr(), wsb, B, s, nh, dh, None)


def timed(n=30):
    for _ in range(3):
        bwd()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        bwd()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n * 1e3


flops = 8 * B * nh * dh * s * (s + 1) / 2
t = timed()
print(f"attn bwd (dkdv_ts + dq_img) B{B} s{s} nh{nh} dh{dh}: {t:.1f} us, {flops / t / 1e6:.0f} TFLOP/s")
if os.environ.get("MARIO_ATTN_TC_ONLY") is None:
    os.environ["MARIO_ATTN_TC_ONLY"] = "dkdv"
    t2 = timed()
    print(f"  dkdv_ts alone: {t2:.1f} us ({flops * 5 / 8 / t2 / 1e6:.0f} TFLOP/s of its 5/8 share)")
    os.environ["MARIO_ATTN_TRACE"] = "1"
    os.environ["MARIO_ATTN_TRACE_CTAS"] = os.environ.get("CTAS_OUT", "/tmp/ctas.txt")
    bwd()
    torch.cuda.synchronize()
    del os.environ["MARIO_ATTN_TRACE"]
    del os.environ["MARIO_ATTN_TC_ONLY"]
print(subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm", "--format=csv,noheader"], capture_output=True,
                     text=True).stdout.strip())
