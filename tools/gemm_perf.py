"""Time the tcgen05 GEMM on config-2/5 shapes vs torch.matmul (cuBLAS) with CUDA events."""
import sys, json
import torch
sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib

L = _lib.lib()
shapes = [("qkv", 8192, 6144, 2048), ("proj", 8192, 2048, 2048), ("fc1", 8192, 8192, 2048),
          ("fc2", 8192, 2048, 8192), ("head", 8192, 50304, 2048), ("sq8k", 8192, 8192, 8192)]
res = []
VARIANTS = [int(v) for v in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["0", "1"])]
for variant in VARIANTS:
  L.mario_k_gemm_set_variant(variant)
  for name, M, N, K in shapes:
    for mode in ("fwd", "dgrad", "wgrad"):
        if mode == "fwd":
            A = torch.randn(M, K, device="cuda").bfloat16(); B = torch.randn(N, K, device="cuda").bfloat16()
            am, bm, lda, ldb, m, n, k = 0, 0, K, K, M, N, K
        elif mode == "dgrad":   # dX[M,K] = dY[M,N] W[N,K]
            A = torch.randn(M, N, device="cuda").bfloat16(); B = torch.randn(N, K, device="cuda").bfloat16()
            am, bm, lda, ldb, m, n, k = 0, 1, N, K, M, K, N
        else:                   # dW[N,K] = dY^T X
            A = torch.randn(M, N, device="cuda").bfloat16(); B = torch.randn(M, K, device="cuda").bfloat16()
            am, bm, lda, ldb, m, n, k = 1, 1, N, K, N, K, M
        out_f32 = 1 if mode == "wgrad" else 0
        D = torch.zeros(m, n, device="cuda", dtype=torch.float32 if out_f32 else torch.bfloat16)
        def run():
            return L.mario_k_gemm_bf16(A.data_ptr(), lda, am, B.data_ptr(), ldb, bm, m, n, k, D.data_ptr(), n,
                                       out_f32, 1.0 if out_f32 else 0.0, None, None, 0, None, None, 0,
                                       torch.cuda.current_stream().cuda_stream)
        for _ in range(3): assert run() == 0
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        it = 10
        e0.record()
        for _ in range(it): run()
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / it
        # cuBLAS reference for the same product
        if mode == "fwd": f = lambda: A @ B.t()
        elif mode == "dgrad": f = lambda: A @ B
        else: f = lambda: A.t() @ B
        for _ in range(3): f()
        torch.cuda.synchronize(); e0.record()
        for _ in range(it): f()
        e1.record(); torch.cuda.synchronize()
        ms_ref = e0.elapsed_time(e1) / it
        tf = 2.0 * M * N * K / ms / 1e9
        res.append(dict(variant=variant, name=name, mode=mode, M=m, N=n, K=k, ms=round(ms, 4), tflops=round(tf, 1),
                        cublas_tflops=round(2.0 * M * N * K / ms_ref / 1e9, 1)))
        print(json.dumps(res[-1]), flush=True)
