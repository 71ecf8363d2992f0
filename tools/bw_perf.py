"""Bandwidth kernels at cfg-2 shapes (T = 8192 rows, h = 2048): achieved GB/s of algorithmic bytes,
for both norm variants (1 = block-per-row-tile, 0 = warp-per-row + separate column sums)."""
import sys, json
import torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib
L = _lib.lib()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
def timeit(f, it=50):
    for _ in range(3): f()
    torch.cuda.synchronize(); e0.record()
    for _ in range(it): f()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it
T = 8192
for h in (2048, 4096, 5120):
    x = torch.randn(T, h, device="cuda").bfloat16(); y = torch.empty_like(x); dy = torch.randn_like(x); dx = torch.empty_like(x)
    g = torch.randn(h, device="cuda"); b = torch.randn(h, device="cuda"); stats = torch.empty(T, 2, device="cuda")
    dg = torch.zeros(h, device="cuda"); db = torch.zeros(h, device="cuda"); ds = torch.zeros(h, device="cuda")
    part = torch.empty(3 * h * 148 * 8, device="cuda")
    for var in (1, 0):
        L.mario_k_norm_set_variant(var)
        ms = timeit(lambda: L.mario_k_norm_fwd(x.data_ptr(), g.data_ptr(), b.data_ptr(), y.data_ptr(), stats.data_ptr(), T, h, 1e-5, 0, 1, None))
        print(json.dumps({"h": h, "variant": var, "kernel": "layernorm_fwd", "us": ms * 1e3, "GBps": 2 * T * h * 2 / ms / 1e6}))
        ms = timeit(lambda: L.mario_k_norm_bwd(dy.data_ptr(), x.data_ptr(), stats.data_ptr(), g.data_ptr(), x.data_ptr(), dx.data_ptr(), None, None, None, None, 0, T, h, 0, 1, None))
        print(json.dumps({"h": h, "variant": var, "kernel": "norm_bwd_dx", "us": ms * 1e3, "GBps": 4 * T * h * 2 / ms / 1e6}))
        ms = timeit(lambda: L.mario_k_norm_bwd(dy.data_ptr(), x.data_ptr(), stats.data_ptr(), g.data_ptr(), x.data_ptr(), dx.data_ptr(), dg.data_ptr(), db.data_ptr(), ds.data_ptr(), part.data_ptr(), part.numel(), T, h, 0, 1, None))
        print(json.dumps({"h": h, "variant": var, "kernel": "norm_bwd+dg,db,dsum", "us": ms * 1e3, "GBps": 4 * T * h * 2 / ms / 1e6}))
    L.mario_k_norm_set_variant(1)
ms = timeit(lambda: y.copy_(x))
print(json.dumps({"kernel": "torch copy (ref)", "us": ms * 1e3, "GBps": 2 * T * h * 2 / ms / 1e6}))
