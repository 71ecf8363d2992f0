"""Probe: full-width bf16 parity for two more BASELINE widths (GPT-3 1.3B under Interleave v = 2,
LLaMA2-13B widths at s 1024), worst per-tensor errors vs the fp32 oracle (timings included)."""
import sys
import time

import numpy as np

sys.path.insert(0, ".")
import synth
from oracle import model as om
from tests.test_gpu_parity import check, rounded, run_plan

CASES = [
    ("gpt3-1.3b-interleave", synth.with_(synth.GPT3_1P3B, n_layers=4, micro_batch=1), "interleave", 2, 2, 2),
    ("llama2-13b-s1024", synth.with_(synth.LLAMA2_13B, n_layers=2, micro_batch=1, seq_len=1024), "1f1b", 2, 2, 1),
]
for name, cfg, scheme, S, N, v in CASES:
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, N)
    t0 = time.time()
    loss, grads, _ = run_plan(cfg, S, N, scheme, "mario", "bf16", params, toks, chunks=v)
    t1 = time.time()
    l_o, g_o = om.step(cfg, rounded(params), toks, N, np.float32)
    t2 = time.time()
    wi, wl = check(loss, grads, l_o, g_o, 1.0, norm="l2", inf_guard=1.0)
    print(f"[{name}] loss {loss:.6f} vs {l_o:.6f}; worst inf {wi}; worst l2 {wl}; gpu {t1 - t0:.1f}s oracle {t2 - t1:.1f}s",
          flush=True)
