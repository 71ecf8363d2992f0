"""Norm forward A/B at bench shapes (T = 8192 rows; h = 2048 / 4096 / 5120): variant 2 (row-pipelined,
cp.async.bulk ring) vs 3 (warp per row, v2). Cold = inputs rotate over > 126 MB (HBM reads), warm =
one buffer (L2-resident, as in a step where the norm reads the GEMM output just written). Also checks
the two variants against a float64 torch LayerNorm / RMSNorm of the same bf16 input."""
import json
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)


def timeit(f, nbuf, it=64):
    for i in range(4):
        f(i % nbuf)
    torch.cuda.synchronize()
    e0.record()
    for i in range(it):
        f(i % nbuf)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it


T = 8192
for h in (2048, 4096, 5120):
    nb = max(2, int(400e6 // (T * h * 2 * 2)))
    xs = [(torch.randn(T, h, device="cuda") * 2 + 0.5).bfloat16() for _ in range(nb)]
    ys = [torch.empty(T, h, device="cuda", dtype=torch.bfloat16) for _ in range(nb)]
    g = torch.randn(h, device="cuda") * 0.2 + 1
    b = torch.randn(h, device="cuda") * 0.1
    stats = torch.empty(T, 2, device="cuda")
    for rms in (0, 1):
        x64 = xs[0].double()
        if rms:
            ref = x64 * torch.rsqrt((x64 * x64).mean(1, keepdim=True) + 1e-5) * g.double()
        else:
            mu = x64.mean(1, keepdim=True)
            ref = (x64 - mu) * torch.rsqrt(((x64 - mu) ** 2).mean(1, keepdim=True) + 1e-5) * g.double() + b.double()
        outs = {}
        for var in (2, 3):
            L.mario_k_norm_set_variant(var)
            f = lambda i: L.mario_k_norm_fwd(xs[i].data_ptr(), g.data_ptr(), b.data_ptr(), ys[i].data_ptr(),
                                             stats.data_ptr(), T, h, 1e-5, rms, 1, None)
            cold = timeit(f, nb)
            warm = timeit(f, 1)
            f(0)
            torch.cuda.synchronize()
            outs[var] = ys[0].clone()
            err = float(((ys[0].double() - ref).abs().max() / ref.abs().max()))
            print(json.dumps({"h": h, "rms": rms, "variant": var, "cold_us": round(cold * 1e3, 2),
                              "warm_us": round(warm * 1e3, 2), "cold_GBps": round(2 * T * h * 2 / cold / 1e6),
                              "max_rel_err_vs_f64": err}))
        d = (outs[2].float() - outs[3].float()).abs()
        print(json.dumps({"h": h, "rms": rms, "v2_vs_v3_max_abs": float(d.max()),
                          "frac_differ": float((d > 0).float().mean())}))
    L.mario_k_norm_set_variant(2)
    ms = timeit(lambda i: ys[i].copy_(xs[i]), nb)
    print(json.dumps({"h": h, "kernel": "torch copy (ref)", "us": round(ms * 1e3, 2),
                      "GBps": round(2 * T * h * 2 / ms / 1e6)}))
    del xs, ys
