"""8-stage plans (north_star: "a Mario-scheduled 8-stage iteration whose gradients match the CPU
oracle") through mario_run_iter, every rank's list executed on this GPU in loopback.

* fp32 (<= 1e-4, A19 inf-norm) on tiny models with L = 8 * v layers: 1F1B S = 8, N = 16;
  Interleave S = 8, v = 2, N = 16; Chimera S = 8, N = 8 and 16; at base / ckpt / mario.
* Mario and ckpt are bitwise equal to base at S = 8 (P:133 checkpointing replays the forward,
  P:99 synchronous flush; passes 1-4 never reorder BW per (device, part)).
* bf16 at GPT-3 1.3B width with one layer per stage (SURVEY §8(d) d5 parity shape, N reduced to 8).
"""
import numpy as np
import pytest
import torch

import synth
from oracle import model as om
from paper_conf_ppopp_liultj25_b200 import api

from .test_gpu_parity import check, rounded, run_plan

pytestmark = pytest.mark.gpu

TINY8 = synth.with_(synth.TINY_GPT, n_layers=8)
TINY16 = synth.with_(synth.TINY_GPT, n_layers=16)
TINY8_L = synth.with_(synth.tiny_llama(), n_layers=8)

CASES = [
    ("1f1b-gpt", TINY8, "1f1b", 16, 1),
    ("1f1b-llama", TINY8_L, "1f1b", 16, 1),
    ("interleave-gpt", TINY16, "interleave", 16, 2),
    ("chimera-gpt-n8", TINY8, "chimera", 8, 1),
    ("chimera-gpt-n16", TINY8, "chimera", 16, 1),
]


@pytest.mark.parametrize("name,cfg,scheme,N,v", CASES, ids=[c[0] for c in CASES])
def test_s8_fp32_parity_all_levels(name, cfg, scheme, N, v):
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, N)
    l_o, g_o = om.step(cfg, params, toks, N, np.float32)
    flat = {}
    for level in ("base", "ckpt", "mario"):
        loss, grads, flat[level] = run_plan(cfg, 8, N, scheme, level, "f32", params, toks, chunks=v)
        check(loss, grads, l_o, g_o, 1e-4)
    assert np.array_equal(flat["base"], flat["ckpt"]), "ckpt differs from base"
    assert np.array_equal(flat["base"], flat["mario"]), "mario differs from base"


@pytest.mark.parametrize("scheme,cfg,N,v", [("1f1b", TINY8, 16, 1), ("interleave", TINY16, 16, 2),
                                            ("chimera", TINY8, 16, 1)], ids=["1f1b", "interleave", "chimera"])
def test_s8_bf16_mario_bitwise_base(scheme, cfg, N, v):
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, N)
    outs = [run_plan(cfg, 8, N, scheme, lvl, "bf16", params, toks, chunks=v) for lvl in ("base", "mario")]
    assert outs[0][0] == outs[1][0]
    assert np.array_equal(outs[0][2], outs[1][2])
    l_o, g_o = om.step(cfg, rounded(params), toks, N, np.float32)
    check(outs[1][0], outs[1][1], l_o, g_o, 2e-2)


@pytest.mark.slow
def test_s8_bf16_cfg2_width():
    """GPT-3 1.3B width (h 2048, 16 heads, s 2048, V 50304), L = 8 (one layer per stage), S = 8,
    N = 8, mbs 1, Mario 1F1B: the CTA-pair GEMM and the tcgen05 attention with the dS image run at
    the shapes bench.py times; held to north_star's 2e-2 per-tensor inf-norm bound (A19)."""
    cfg = synth.with_(synth.GPT3_1P3B, n_layers=8, micro_batch=1)
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 8)
    loss, grads, flat = run_plan(cfg, 8, 8, "1f1b", "mario", "bf16", params, toks)
    base = run_plan(cfg, 8, 8, "1f1b", "base", "bf16", params, toks)[2]
    assert np.array_equal(flat, base)
    l_o, g_o = om.step(cfg, rounded(params), toks, 8, np.float32)
    wi, wl = check(loss, grads, l_o, g_o, 2e-2)
    print(f"[s8 cfg2-width] loss {loss:.6f} vs {l_o:.6f}; worst inf-rel {wi}; worst l2-rel {wl}")
