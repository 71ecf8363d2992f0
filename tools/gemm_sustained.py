"""Sustained (power-capped) GEMM throughput, apples to apples with MEASURED_PEAKS.json's
bf16_tflops_sustained: 8192^3 bf16 back to back for ~4 s each, torch.matmul (cuBLAS) and the tcgen05
kernel (mario_k_gemm_bf16), alternating twice; SM clock sampled by NVML during each run. Also the
cfg-2 layer GEMM mix (tools/gemm_step.py shapes, no epilogues) for 4 s."""
import json
import sys
import threading
import time

import torch

sys.path.insert(0, ".")
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()


class Clock:
    def __init__(self):
        import pynvml
        pynvml.nvmlInit()
        self.nv = pynvml
        self.h = pynvml.nvmlDeviceGetHandleByIndex(0)
        self.samples = []
        self.run = False

    def start(self):
        self.samples = []
        self.run = True
        self.t = threading.Thread(target=self._loop, daemon=True)
        self.t.start()

    def _loop(self):
        while self.run:
            self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            time.sleep(0.05)

    def stop(self):
        self.run = False
        self.t.join()
        s = sorted(self.samples)
        return s[len(s) // 2] if s else None


clk = Clock()
M, N, K = (int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "8192,8192,8192").split(","))
A = torch.randn(M, K, device="cuda").bfloat16()
B = torch.randn(N, K, device="cuda").bfloat16()
D = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
st = torch.cuda.current_stream().cuda_stream


def ours():
    L.mario_k_gemm_bf16(A.data_ptr(), K, 0, B.data_ptr(), K, 0, M, N, K, D.data_ptr(), N, 0, 0.0, None, None, N, None,
                        None, N, st)


def cublas():
    torch.matmul(A, B.t(), out=D)


def sustained(fn, fl, secs=4.0):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    clk.start()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    n = 0
    t0 = time.time()
    e0.record()
    while time.time() - t0 < secs:
        for _ in range(10):
            fn()
        n += 10
        torch.cuda.synchronize()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    return round(fl * n / (ms / 1e3) / 1e12, 1), clk.stop()


fl = 2.0 * M * N * K
for rnd in range(int(sys.argv[1]) if len(sys.argv) > 1 else 2):
    for name, fn in (("cublas", cublas), ("ours", ours)):
        tf, mhz = sustained(fn, fl)
        print(json.dumps({"round": rnd, "gemm": name, "shape": [M, N, K], "sustained_tflops": tf, "sm_mhz_median": mhz}),
              flush=True)
