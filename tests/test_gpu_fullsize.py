"""BASELINE.json configs[1] at FULL size, in the launch configuration bench.py times (GPT-3 1.3B:
24 layers, h 2048, mbs 4, s 2048, V 50304, bf16, one GPU, the bench's device-side A20 perf init).
No oracle finishes this size, so properties that hold at any size pin it (SURVEY §8(c) c1
"several results are correct", c4 forward pin (7) and the CE invariant):
  1. base / ckpt / mario plans give bitwise-identical loss and gradients, and a repeat is bitwise equal;
  2. initial loss = ln V + sigma_z^2 / 2 (Hf rows have unit variance at gamma 1, beta 0, so a logit
     of vocab entry v has variance ||wte_v||^2; sigma_z^2 = their mean), within 0.02;
  3. sum_v dwte[v] = sum_p dwpe[p]: the head term dlogits^T Hf sums to 0 over v (softmax rows minus
     one-hot sum to 0), leaving sum over tokens of dH0 on both sides (rounding of the bf16 dlogits
     bounds the residual)."""
import math
import os
import sys

import numpy as np
import pytest
import torch

import synth
from paper_conf_ppopp_liultj25_b200 import api

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from bench import init_weights_device  # noqa: E402

pytestmark = pytest.mark.gpu
N = 4


def _run(level, w0, tok, ctx):
    cfg = synth.GPT3_1P3B
    plan = api.Plan(cfg, 1, N, "1f1b", level, dtype="bf16")
    w, g, ws = api.alloc_for(plan, 0)
    w.copy_(w0)
    loss = ctx.run_iter(plan, w, tok, g, ws)
    torch.cuda.synchronize()
    out = (loss, g.clone())
    if level == "mario":
        loss2 = ctx.run_iter(plan, w, tok, g, ws)
        torch.cuda.synchronize()
        assert loss2 == loss and torch.equal(g, out[1]), "repeat not bitwise equal"
    del w, g, ws
    torch.cuda.empty_cache()
    return out, plan


def test_bench_config_full_size_properties():
    torch.cuda.set_device(0)
    cfg = synth.GPT3_1P3B
    assert (cfg.n_layers, cfg.hidden, cfg.micro_batch, cfg.seq_len, cfg.vocab) == (24, 2048, 4, 2048, 50304)
    ctx = api.default_context()
    plan0 = api.Plan(cfg, 1, N, "1f1b", "mario", dtype="bf16")
    w0 = init_weights_device(plan0, 0, torch)
    tok = torch.from_numpy(synth.make_tokens(cfg, N)).cuda()
    res = {}
    for level in ("mario", "base", "ckpt"):
        res[level], plan = _run(level, w0, tok, ctx)
    lm, gm = res["mario"]
    for level in ("base", "ckpt"):
        l, g = res[level]
        assert l == lm and torch.equal(g, gm), level
    offs = {name: (off, cnt) for name, off, cnt in plan.rank_params(0)}
    V, h, s = cfg.vocab, cfg.hidden, cfg.seq_len
    o, c = offs["wte"]
    wte = w0[o:o + c].view(V, h).double()
    sigma2 = float((wte * wte).sum(1).mean())
    expect = math.log(V) + sigma2 / 2
    print(f"[full size] loss {lm:.6f}, ln V + sigma_z^2/2 = {expect:.6f} (sigma_z^2 {sigma2:.4f})")
    assert abs(lm - expect) < 0.02
    dwte = gm[o:o + c].view(V, h).double().sum(0)
    o2, c2 = offs["wpe"]
    dwpe = gm[o2:o2 + c2].view(s, h).double().sum(0)
    rel = float((dwte - dwpe).norm() / dwpe.norm())
    print(f"[full size] ||sum_v dwte - sum_p dwpe|| / ||sum_p dwpe|| = {rel:.3e}")
    assert rel < 0.05
