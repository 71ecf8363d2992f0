"""Library attention on the same causal shapes (context for our kernels' roofline): torch SDPA
with the cuDNN and flash backends, forward and forward+backward. Same FLOP convention as
attn_perf.py (fwd = 4 B nh dh s(s+1)/2, bwd = 2x fwd)."""
import json
import torch
from torch.nn.attention import sdpa_kernel, SDPBackend
for (B, s, nh, dh) in [(4, 2048, 16, 128), (1, 4096, 32, 128), (1, 2048, 32, 64)]:
    q, k, v = (torch.randn(B, nh, s, dh, device="cuda", dtype=torch.bfloat16, requires_grad=True) for _ in range(3))
    do = torch.randn(B, nh, s, dh, device="cuda", dtype=torch.bfloat16)
    fl_f = 4.0 * B * nh * dh * s * (s + 1) / 2
    for be in (SDPBackend.CUDNN_ATTENTION, SDPBackend.FLASH_ATTENTION):
        try:
            with sdpa_kernel([be]):
                def fwd():
                    with torch.no_grad():
                        return torch.nn.functional.scaled_dot_product_attention(q, k, v, is_causal=True)
                def fb():
                    o = torch.nn.functional.scaled_dot_product_attention(q, k, v, is_causal=True)
                    o.backward(do)
                res = {}
                for name, f in (("fwd", fwd), ("fwd+bwd", fb)):
                    for _ in range(3): f()
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
                    e0.record()
                    for _ in range(10): f()
                    e1.record(); torch.cuda.synchronize()
                    res[name] = e0.elapsed_time(e1) / 10
                bwd = res["fwd+bwd"] - res["fwd"]
                print(json.dumps({"shape": [B, s, nh, dh], "backend": str(be), "fwd_ms": round(res["fwd"], 3),
                                  "fwd_tflops": round(fl_f / res["fwd"] / 1e9, 1), "bwd_ms": round(bwd, 3),
                                  "bwd_tflops": round(2 * fl_f / bwd / 1e9, 1)}), flush=True)
        except Exception as e:  # backend unavailable for this shape
            print(json.dumps({"shape": [B, s, nh, dh], "backend": str(be), "error": str(e)[:200]}), flush=True)
