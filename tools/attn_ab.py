"""A/B the attention forward variants (-1 two-Q-tile tcgen05, 2 one-Q-tile tcgen05, 0 mma.sync) on
the cfg-2 shape and others: time + max |diff| of O and lse against the mma.sync kernel."""
import sys, json
import torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib
L = _lib.lib()
for (B, s, nh, dh) in [(4, 2048, 16, 128), (1, 4096, 32, 128), (1, 2048, 32, 64), (2, 1000, 4, 128), (1, 300, 2, 64)]:
    h = nh * dh
    g = torch.Generator(device="cuda").manual_seed(s + dh)
    qkv = (torch.randn(B * s, 3 * h, device="cuda", generator=g) * 2).bfloat16()
    fl = 4.0 * B * nh * dh * s * (s + 1) / 2
    res = {}
    for v in (0, 2, -1):
        L.mario_k_attn_set_variant(v)
        O = torch.full((B * s, h), float("nan"), device="cuda", dtype=torch.bfloat16)
        lse = torch.full((nh, B * s), float("nan"), device="cuda")
        f = lambda: L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None)
        assert f() == 0
        torch.cuda.synchronize()
        res[v] = (O.float().clone(), lse.clone())
        for _ in range(3): f()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        torch.cuda.synchronize(); e0.record()
        for _ in range(10): f()
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 10
        dO = (res[v][0] - res[0][0]).abs().max().item()
        dl = (res[v][1] - res[0][1]).abs().max().item()
        print(json.dumps({"shape": [B, s, nh, dh], "variant": v, "ms": round(ms, 4), "tflops": round(fl / ms / 1e9, 1),
                          "max_dO_vs_mma": dO, "max_dlse_vs_mma": dl, "nan": bool(torch.isnan(res[v][0]).any())}), flush=True)
L.mario_k_attn_set_variant(-1)
