"""GPU parity: mario_run_iter (C-ABI, hand-written sm_100a kernels) vs the CPU oracle on the
same seeded synthetic inputs. Tolerances (north_star / DESIGN.md A19): per-tensor max relative
error ||g - o||_inf / ||o||_inf <= 1e-4 in fp32 mode and <= 2e-2 in bf16 mode; same for the loss.
Multi-stage plans run in loopback (all ranks in one process, one GPU)."""
import numpy as np
import pytest
import torch

import synth
from oracle import model as om
from paper_conf_ppopp_liultj25_b200 import api

pytestmark = pytest.mark.gpu

_CTX = {}


def ctx():
    if "c" not in _CTX:
        torch.cuda.set_device(0)
        _CTX["c"] = api.Context(0, 1, 0)
    return _CTX["c"]


def run_plan(cfg, S, N, scheme, level, dtype, params, toks, chunks=1):
    plan = api.Plan(cfg, S, N, scheme, level, chunks=chunks, dtype=dtype)
    rank = -1 if S > 1 else 0
    w, g, ws = api.alloc_for(plan, rank)
    w.copy_(torch.from_numpy(api.pack_params(plan, params, rank)))
    loss = ctx().run_iter(plan, w, toks, g, ws)
    torch.cuda.synchronize()
    return loss, api.unpack_params(plan, g.cpu().numpy(), rank), g.cpu().numpy()


def rounded(params):
    """A6 reading: in bf16 mode the GPU rounds the matrix weights RNE to bf16; vectors stay fp32."""
    return {k: (synth.round_to_bf16(v) if v.ndim == 2 else v) for k, v in params.items()}


def check(loss, grads, l_o, g_o, tol):
    assert abs(loss - l_o) <= tol * abs(l_o), (loss, l_o)
    worst = (None, 0.0)
    for k, v in g_o.items():
        err = float(np.abs(grads[k] - v).max() / max(np.abs(v).max(), 1e-30))
        if err > worst[1]:
            worst = (k, err)
    assert worst[1] <= tol, worst


TINY_L = synth.tiny_llama()


@pytest.mark.parametrize("cfg", [synth.TINY_GPT, TINY_L], ids=["gpt", "llama"])
@pytest.mark.parametrize("S,level", [(1, "mario"), (2, "base"), (2, "ckpt"), (2, "mario"), (4, "mario")])
def test_fp32_parity_1f1b(cfg, S, level):
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 4)
    loss, grads, _ = run_plan(cfg, S, 4, "1f1b", level, "f32", params, toks)
    l_o, g_o = om.step(cfg, params, toks, 4, np.float32)
    check(loss, grads, l_o, g_o, 1e-4)


@pytest.mark.parametrize("scheme,S,N,v", [("interleave", 2, 4, 2), ("chimera", 2, 4, 1), ("chimera", 4, 4, 1)])
def test_fp32_parity_other_schemes(scheme, S, N, v):
    cfg = synth.TINY_GPT
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, N)
    loss, grads, _ = run_plan(cfg, S, N, scheme, "mario", "f32", params, toks, chunks=v)
    l_o, g_o = om.step(cfg, params, toks, N, np.float32)
    check(loss, grads, l_o, g_o, 1e-4)


@pytest.mark.parametrize("cfg", [synth.TINY_GPT, TINY_L], ids=["gpt", "llama"])
def test_bf16_parity(cfg):
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 4)
    loss, grads, _ = run_plan(cfg, 2, 4, "1f1b", "mario", "bf16", params, toks)
    l_o, g_o = om.step(cfg, rounded(params), toks, 4, np.float32)
    check(loss, grads, l_o, g_o, 2e-2)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_mario_bitwise_equals_base(dtype):
    """Rescheduling + checkpointing must not change a single bit."""
    cfg = synth.TINY_GPT
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 8)
    outs = [run_plan(cfg, 4, 8, "1f1b", lvl, dtype, params, toks)[2] for lvl in ("base", "ckpt", "mario")]
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])


def test_ragged_multi_tile_bf16():
    """Sizes spanning several GEMM tiles with a ragged tail (T = 2*100 tokens, h = 192, V = 1000)."""
    cfg = synth.ModelCfg("gpt", 2, 192, 3, 768, 1000, 100, 2, True)
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 2)
    loss, grads, _ = run_plan(cfg, 2, 2, "1f1b", "mario", "bf16", params, toks)
    l_o, g_o = om.step(cfg, rounded(params), toks, 2, np.float32)
    check(loss, grads, l_o, g_o, 2e-2)


def test_deterministic_repeat():
    cfg = synth.tiny_llama()
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 4)
    a = run_plan(cfg, 2, 4, "1f1b", "mario", "bf16", params, toks)[2]
    b = run_plan(cfg, 2, 4, "1f1b", "mario", "bf16", params, toks)[2]
    assert np.array_equal(a, b)
