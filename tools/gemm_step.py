"""The twelve GEMMs of one GPT-3 1.3B layer (cfg 2: T = 8192 tokens, h = 2048, f = 8192) with the
executor's epilogues (bias, residual, GeLU second output, GeLU' aux, fp32 += wgrad), in step order,
each timed with CUDA events. Activations rotate over 3 micro-batch sets (> L2) as in a real step.
Prints per-call TFLOP/s next to the same shape without epilogue and cuBLAS."""
import json
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()
import os  # noqa: E402
# the default stored activation set keeps G = gelu(Z) from the forward, so the fc2 dgrad epilogue has
# no G output; MARIO_STORE_ACT=0 (lean set) times it with the recomputed G as a second output
LEAN = os.environ.get("MARIO_STORE_ACT", "1") == "0"
if os.environ.get("STREAMK"):
    L.mario_k_gemm_set_streamk(int(os.environ["STREAMK"]))
if os.environ.get("VARIANT"):
    L.mario_k_gemm_set_variant(int(os.environ["VARIANT"]))
T, h, f = 8192, 2048, 8192
bf = torch.bfloat16
dev = "cuda"
V = 50304
Wh = torch.randn(V, h, device=dev).to(bf) * 0.02
dWh = torch.zeros(V, h, device=dev)
W = {"qkv": torch.randn(3 * h, h, device=dev).to(bf) * 0.02, "proj": torch.randn(h, h, device=dev).to(bf) * 0.02,
     "fc1": torch.randn(f, h, device=dev).to(bf) * 0.02, "fc2": torch.randn(h, f, device=dev).to(bf) * 0.02}
bias = {k: torch.randn(v.shape[0], device=dev) * 0.02 for k, v in W.items()}
dW = {k: torch.zeros(v.shape, device=dev) for k, v in W.items()}
NS = 3


def act():
    r = lambda *s: torch.randn(*s, device=dev).to(bf)
    return {"A": r(T, h), "QKV": r(T, 3 * h), "O": r(T, h), "Hin": r(T, h), "H1": r(T, h), "A2": r(T, h),
            "Z": r(T, f), "G": r(T, f), "Hout": r(T, h), "dH": r(T, h), "dZ": r(T, f), "dA": r(T, h),
            "dH1": r(T, h), "dO": r(T, h), "dQKV": r(T, 3 * h),
            "Hf": r(T, h), "logits": torch.empty(T, V, device=dev), "dlog": r(T, V)}


sets = [act() for _ in range(NS)]
st = torch.cuda.current_stream().cuda_stream
P = lambda t: t.data_ptr() if t is not None else None


def gemm(A, lda, amn, B, ldb, bmn, M, N, K, D, ldd, f32, beta, b=None, res=None, d2=None, aux=None):
    rc = L.mario_k_gemm_bf16(P(A), lda, amn, P(B), ldb, bmn, M, N, K, P(D), ldd, f32, beta, P(b), P(res), ldd,
                             P(d2), P(aux), ldd, st)
    assert rc == 0, rc


def calls(a, epi=True):
    e = epi
    return [
        ("qkv fwd", 2 * T * 3 * h * h, lambda: gemm(a["A"], h, 0, W["qkv"], h, 0, T, 3 * h, h, a["QKV"], 3 * h, 0, 0.,
                                                    bias["qkv"] if e else None)),
        ("proj fwd", 2 * T * h * h, lambda: gemm(a["O"], h, 0, W["proj"], h, 0, T, h, h, a["H1"], h, 0, 0.,
                                                 bias["proj"] if e else None, a["Hin"] if e else None)),
        ("fc1 fwd", 2 * T * f * h, lambda: gemm(a["A2"], h, 0, W["fc1"], h, 0, T, f, h, a["Z"], f, 0, 0.,
                                                bias["fc1"] if e else None, None, a["G"] if e else None)),
        ("fc2 fwd", 2 * T * h * f, lambda: gemm(a["G"], f, 0, W["fc2"], f, 0, T, h, f, a["Hout"], h, 0, 0.,
                                                bias["fc2"] if e else None, a["H1"] if e else None)),
        ("fc2 wgrad", 2 * T * h * f, lambda: gemm(a["dH"], h, 1, a["G"], f, 1, h, f, T, dW["fc2"], f, 1,
                                                  1. if e else 0.)),
        ("fc2 dgrad", 2 * T * h * f, lambda: gemm(a["dH"], h, 0, W["fc2"], f, 1, T, f, h, a["dZ"], f, 0, 0.,
                                                  d2=a["G"] if (e and LEAN) else None, aux=a["Z"] if e else None)),
        ("fc1 wgrad", 2 * T * h * f, lambda: gemm(a["dZ"], f, 1, a["A2"], h, 1, f, h, T, dW["fc1"], h, 1,
                                                  1. if e else 0.)),
        ("fc1 dgrad", 2 * T * h * f, lambda: gemm(a["dZ"], f, 0, W["fc1"], h, 1, T, h, f, a["dA"], h, 0, 0.)),
        ("proj wgrad", 2 * T * h * h, lambda: gemm(a["dH1"], h, 1, a["O"], h, 1, h, h, T, dW["proj"], h, 1,
                                                   1. if e else 0.)),
        ("proj dgrad", 2 * T * h * h, lambda: gemm(a["dH1"], h, 0, W["proj"], h, 1, T, h, h, a["dO"], h, 0, 0.)),
        ("qkv wgrad", 2 * T * 3 * h * h, lambda: gemm(a["dQKV"], 3 * h, 1, a["A"], h, 1, 3 * h, h, T, dW["qkv"], h, 1,
                                                      1. if e else 0.)),
        ("qkv dgrad", 2 * T * 3 * h * h, lambda: gemm(a["dQKV"], 3 * h, 0, W["qkv"], h, 1, T, h, 3 * h, a["dA"], h,
                                                      0, 0.)),
        ("head fwd", 2 * T * V * h, lambda: gemm(a["Hf"], h, 0, Wh, h, 0, T, V, h, a["logits"], V, 1, 0.)),
        ("head wgrad", 2 * T * V * h, lambda: gemm(a["dlog"], V, 1, a["Hf"], h, 1, V, h, T, dWh, h, 1,
                                                   1. if e else 0.)),
        ("head dgrad", 2 * T * V * h, lambda: gemm(a["dlog"], V, 0, Wh, h, 1, T, h, V, a["dA"], h, 0, 0.)),
    ]


def run(epi, iters=6):
    ev = []
    for it in range(iters):
        for name, fl, fn in calls(sets[it % NS], epi):
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record()
            fn()
            e1.record()
            ev.append((it, name, fl, e0, e1))
    torch.cuda.synchronize()
    out = {}
    for it, name, fl, e0, e1 in ev:
        if it < 2:
            continue
        out.setdefault(name, []).append((fl, e0.elapsed_time(e1)))
    return {k: (sum(x[0] for x in v) / sum(x[1] for x in v) / 1e9, sum(x[1] for x in v) / len(v)) for k, v in out.items()}


def cublas(iters=6):
    """The same (M, N, K) as plain cuBLAS bf16 GEMMs (torch.mm, bf16 out), for context."""
    shapes = {"qkv fwd": (T, 3 * h, h), "proj fwd": (T, h, h), "fc1 fwd": (T, f, h), "fc2 fwd": (T, h, f),
              "fc2 wgrad": (h, f, T), "fc2 dgrad": (T, f, h), "fc1 wgrad": (f, h, T), "fc1 dgrad": (T, h, f),
              "proj wgrad": (h, h, T), "proj dgrad": (T, h, h), "qkv wgrad": (3 * h, h, T), "qkv dgrad": (T, h, 3 * h),
              "head fwd": (T, V, h), "head wgrad": (V, h, T), "head dgrad": (T, h, V)}
    out = {}
    for name, (M, N, K) in shapes.items():
        a = [torch.randn(M, K, device=dev).to(bf) for _ in range(NS)]
        b = [torch.randn(K, N, device=dev).to(bf) for _ in range(NS)]
        ts = []
        for it in range(iters):
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record()
            torch.mm(a[it % NS], b[it % NS])
            e1.record()
            ts.append((e0, e1))
        torch.cuda.synchronize()
        ms = sum(e0.elapsed_time(e1) for e0, e1 in ts[2:]) / (iters - 2)
        out[name] = 2.0 * M * N * K / ms / 1e9
        del a, b
    return out


with_epi = run(True)
no_epi = run(False)
cub = cublas()
tot_fl = tot_ms = 0.0
for name, fl, _ in calls(sets[0]):
    tf, ms = with_epi[name]
    tot_fl += fl
    tot_ms += ms
    print(json.dumps({"gemm": name, "tflops_epi": round(tf, 1), "us_epi": round(ms * 1e3, 1),
                      "tflops_noepi": round(no_epi[name][0], 1), "tflops_cublas": round(cub[name], 1)}))
print(json.dumps({"layer_total_tflops": round(tot_fl / tot_ms / 1e9, 1), "layer_ms": round(tot_ms, 3)}))
