"""Microbenchmark of the dK/dV kernel's phases via MARIO_ATTN_DBG (fa_bwd_dkdv_tc: bit 0 skips the
softmax arithmetic, bit 1 the S/dP MMAs, bit 2 the accumulate MMAs, bit 4 the streamed TMA loads) at
the cfg-2 shape, to separate the SS-mode S^T/dP^T MMA rate (M128 N64 K16) from the rest.

    python tools/attn_mma_rate.py [B s nh dh]
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()
B, s, nh, dh = (int(x) for x in sys.argv[1:5]) if len(sys.argv) > 4 else (4, 2048, 16, 128)
h = nh * dh
qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
lse = torch.empty(nh, B * s, device="cuda")
dO = torch.randn(B * s, h, device="cuda").bfloat16()
dq = torch.empty(B * s, 3 * h, device="cuda", dtype=torch.bfloat16)
scr = torch.empty(nh, B * s, device="cuda")
assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0
os.environ["MARIO_ATTN_TC_ONLY"] = "dkdv"
ntile = B * nh * sum(s // 64 - 2 * j for j in range(s // 128))
sms = torch.cuda.get_device_properties(0).multi_processor_count


def timed(dbg, n=20):
    os.environ["MARIO_ATTN_DBG"] = str(dbg)
    f = lambda: L.mario_k_attn_bwd(qkv.data_ptr(), O.data_ptr(), dO.data_ptr(), lse.data_ptr(), dq.data_ptr(),  # noqa
                                   scr.data_ptr(), B, s, nh, dh, 1, None)
    for _ in range(3):
        f()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        f()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n * 1e3


for dbg, what in [(0, "ts (production)"), (1 << 30, "tc, all phases"), (1, "no softmax"), (5, "S/dP MMAs + loads"),
                  (21, "S/dP MMAs only"), (3, "acc MMAs + loads"), (19, "acc MMAs only"), (7, "loads only"),
                  (23, "empty pipeline"), (32, "1 tile per CTA"), (55, "1 empty tile per CTA"),
                  (55 | 128, "+ no K/V load")]:
    us = timed(dbg)
    clk = us * 1e-6 * 1.965e9 * sms / ntile
    print(f"dbg {dbg:>10} {what:22s} {us:8.1f} us  {clk:7.0f} SM-clk per 64-query tile (at 1965 MHz)")
