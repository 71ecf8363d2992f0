"""fc2 dgrad at cfg 2 (dZ[T,f] = dH[T,h] W2[h,f] * gelu'(Z), T 8192, h 2048, f 8192) through the C-ABI,
without (stored activation set, the default) and with (lean set) the recomputed G = gelu(Z) second
output, for ncu captures: launch 0-2 without G, 3-5 with G. Algorithmic bytes: dH + W2 + Z in, dZ out
(+ G out) = 335 MB (469 MB)."""
import sys
import torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib
L = _lib.lib()
T, h, f = 8192, 2048, 8192
dH = torch.randn(T, h, device="cuda").bfloat16()
W2 = (torch.randn(h, f, device="cuda") * 0.02).bfloat16()
Z = torch.randn(T, f, device="cuda").bfloat16()
dZ = torch.empty(T, f, device="cuda", dtype=torch.bfloat16)
G = torch.empty(T, f, device="cuda", dtype=torch.bfloat16)
st = torch.cuda.current_stream().cuda_stream
for with_g in (False, True):
    for _ in range(3):
        rc = L.mario_k_gemm_bf16(dH.data_ptr(), h, 0, W2.data_ptr(), f, 1, T, f, h, dZ.data_ptr(), f, 0, 0.0, None,
                                 None, f, G.data_ptr() if with_g else None, Z.data_ptr(), f, st)
        assert rc == 0, rc
torch.cuda.synchronize()
