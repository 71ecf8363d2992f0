"""Time the tcgen05 GEMM variants on config-2 shapes vs torch.matmul (cuBLAS) with CUDA events.
Variants are interleaved per shape so clock/power drift affects them alike."""
import sys, json
import torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib

L = _lib.lib()
shapes = [("qkv", 8192, 6144, 2048), ("proj", 8192, 2048, 2048), ("fc1", 8192, 8192, 2048),
          ("fc2", 8192, 2048, 8192), ("head", 8192, 50304, 2048)]
VARIANTS = [int(v) for v in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["-1", "0", "2", "3"])]
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
def timeit(f, it=10):
    for _ in range(3): f()
    torch.cuda.synchronize(); e0.record()
    for _ in range(it): f()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it
for name, M, N, K in shapes:
    for mode in ("fwd", "dgrad", "wgrad"):
        if mode == "fwd":
            A = torch.randn(M, K, device="cuda").bfloat16(); B = torch.randn(N, K, device="cuda").bfloat16()
            am, bm, lda, ldb, m, n, k = 0, 0, K, K, M, N, K
        elif mode == "dgrad":
            A = torch.randn(M, N, device="cuda").bfloat16(); B = torch.randn(N, K, device="cuda").bfloat16()
            am, bm, lda, ldb, m, n, k = 0, 1, N, K, M, K, N
        else:
            A = torch.randn(M, N, device="cuda").bfloat16(); B = torch.randn(M, K, device="cuda").bfloat16()
            am, bm, lda, ldb, m, n, k = 1, 1, N, K, N, K, M
        out_f32 = 1 if mode == "wgrad" else 0
        D = torch.zeros(m, n, device="cuda", dtype=torch.float32 if out_f32 else torch.bfloat16)
        st = torch.cuda.current_stream().cuda_stream
        run = lambda: L.mario_k_gemm_bf16(A.data_ptr(), lda, am, B.data_ptr(), ldb, bm, m, n, k, D.data_ptr(), n,
                                          out_f32, 1.0 if out_f32 else 0.0, None, None, 0, None, None, 0, st)
        ref = (lambda: A @ B.t()) if mode == "fwd" else (lambda: A @ B) if mode == "dgrad" else (lambda: A.t() @ B)
        fl = 2.0 * M * N * K
        row = {"name": name, "mode": mode, "M": m, "N": n, "K": k, "cublas": round(fl / timeit(ref) / 1e9, 1)}
        for v in VARIANTS:
            L.mario_k_gemm_set_variant(v)
            row[f"v{v}"] = round(fl / timeit(run) / 1e9, 1)
        L.mario_k_gemm_set_variant(-1)
        print(json.dumps(row), flush=True)
