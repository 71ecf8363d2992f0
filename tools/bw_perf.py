"""Bandwidth kernels at cfg-2 shapes: achieved GB/s vs the measured HBM copy peak."""
import sys, json
import torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib
L = _lib.lib()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
def timeit(f, it=20):
    for _ in range(3): f()
    torch.cuda.synchronize(); e0.record()
    for _ in range(it): f()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it
T, h = 8192, 2048
x = torch.randn(T, h, device="cuda").bfloat16(); y = torch.empty_like(x); dy = torch.randn_like(x); dx = torch.empty_like(x)
g = torch.randn(h, device="cuda"); b = torch.randn(h, device="cuda"); stats = torch.empty(T, 2, device="cuda")
dg = torch.zeros(h, device="cuda"); db = torch.zeros(h, device="cuda"); part = torch.empty(2 * 128 * h, device="cuda")
ms = timeit(lambda: L.mario_k_norm_fwd(x.data_ptr(), g.data_ptr(), b.data_ptr(), y.data_ptr(), stats.data_ptr(), T, h, 1e-5, 0, 1, None))
print(json.dumps({"kernel": "layernorm_fwd", "ms": ms, "GBps": 2 * T * h * 2 / ms / 1e6}))
ms = timeit(lambda: L.mario_k_norm_bwd(dy.data_ptr(), x.data_ptr(), stats.data_ptr(), g.data_ptr(), x.data_ptr(), dx.data_ptr(), None, None, None, T, h, 0, 1, None))
print(json.dumps({"kernel": "norm_bwd_dx", "ms": ms, "GBps": 4 * T * h * 2 / ms / 1e6}))
ms = timeit(lambda: L.mario_k_norm_bwd(dy.data_ptr(), x.data_ptr(), stats.data_ptr(), g.data_ptr(), x.data_ptr(), dx.data_ptr(), dg.data_ptr(), db.data_ptr(), part.data_ptr(), T, h, 0, 1, None))
print(json.dumps({"kernel": "norm_bwd_dx+colsum", "ms": ms, "GBps": 6 * T * h * 2 / ms / 1e6}))
ms = timeit(lambda: y.copy_(x))
print(json.dumps({"kernel": "torch copy (ref)", "ms": ms, "GBps": 2 * T * h * 2 / ms / 1e6}))
