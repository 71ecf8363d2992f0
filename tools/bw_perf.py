"""Bandwidth kernels at bench shapes (T = 8192 rows; h = 2048 / 4096 / 5120): achieved GB/s of
algorithmic bytes for the norm variants (2 = row-pipelined, 1 = block-per-row-tile, 0 = warp-per-row)
and the softmax-CE at V = 50304. Inputs rotate over enough buffers (> 126 MB L2) that every launch
reads from HBM, as inside a training step."""
import json
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)


def timeit(f, nbuf, it=48):
    for i in range(3):
        f(i % nbuf)
    torch.cuda.synchronize()
    e0.record()
    for i in range(it):
        f(i % nbuf)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it


T = 8192
variants = [int(v) for v in sys.argv[1].split(",")] if len(sys.argv) > 1 else [2, 1, 0]
for h in (2048, 4096, 5120):
    nb = max(2, int(400e6 // (T * h * 2 * 3)))
    xs = [torch.randn(T, h, device="cuda").bfloat16() for _ in range(nb)]
    dys = [torch.randn(T, h, device="cuda").bfloat16() for _ in range(nb)]
    rs = [torch.randn(T, h, device="cuda").bfloat16() for _ in range(nb)]
    ys = [torch.empty(T, h, device="cuda", dtype=torch.bfloat16) for _ in range(nb)]
    g = torch.randn(h, device="cuda")
    b = torch.randn(h, device="cuda")
    stats = torch.empty(T, 2, device="cuda")
    dg = torch.zeros(h, device="cuda")
    db = torch.zeros(h, device="cuda")
    ds = torch.zeros(h, device="cuda")
    part = torch.empty(3 * h * 148 * 8, device="cuda")
    for var in variants:
        L.mario_k_norm_set_variant(var)
        ms = timeit(lambda i: L.mario_k_norm_fwd(xs[i].data_ptr(), g.data_ptr(), b.data_ptr(), ys[i].data_ptr(),
                                                 stats.data_ptr(), T, h, 1e-5, 0, 1, None), nb)
        print(json.dumps({"h": h, "variant": var, "kernel": "layernorm_fwd", "us": round(ms * 1e3, 2),
                          "GBps": round(2 * T * h * 2 / ms / 1e6)}))
        ms = timeit(lambda i: L.mario_k_norm_fwd(xs[i].data_ptr(), g.data_ptr(), b.data_ptr(), ys[i].data_ptr(),
                                                 stats.data_ptr(), T, h, 1e-5, 1, 1, None), nb)
        print(json.dumps({"h": h, "variant": var, "kernel": "rmsnorm_fwd", "us": round(ms * 1e3, 2),
                          "GBps": round(2 * T * h * 2 / ms / 1e6)}))
        ms = timeit(lambda i: L.mario_k_norm_bwd(dys[i].data_ptr(), xs[i].data_ptr(), stats.data_ptr(), g.data_ptr(),
                                                 rs[i].data_ptr(), ys[i].data_ptr(), dg.data_ptr(), db.data_ptr(),
                                                 ds.data_ptr(), part.data_ptr(), part.numel(), T, h, 0, 1, None), nb)
        print(json.dumps({"h": h, "variant": var, "kernel": "norm_bwd+dres+dg,db,dsum", "us": round(ms * 1e3, 2),
                          "GBps": round(4 * T * h * 2 / ms / 1e6)}))
    L.mario_k_norm_set_variant(2)
    ms = timeit(lambda i: ys[i].copy_(xs[i]), nb)
    print(json.dumps({"h": h, "kernel": "torch copy (ref)", "us": round(ms * 1e3, 2),
                      "GBps": round(2 * T * h * 2 / ms / 1e6)}))
    del xs, dys, rs, ys

V = 50304
rows = 8192
logits = [torch.randn(rows, V, device="cuda") * 3 for _ in range(2)]
tok = torch.randint(0, V, (4, 2049), device="cuda", dtype=torch.int32)
dl = torch.empty(rows, V, device="cuda", dtype=torch.bfloat16)
rl = torch.empty(rows, device="cuda")
ms = timeit(lambda i: L.mario_k_softmax_ce(logits[i].data_ptr(), tok.data_ptr(), 2049, 2048, rows, V, 1.0 / rows,
                                           dl.data_ptr(), rl.data_ptr(), 1, None), 2, it=10)
print(json.dumps({"kernel": "softmax_ce V=50304", "us": round(ms * 1e3, 1), "GBps": round(rows * V * 6 / ms / 1e6)}))
