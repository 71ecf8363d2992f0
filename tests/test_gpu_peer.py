"""Peer transport (mario_init_emulated): S pipeline ranks in one process on one GPU, each on its own
streams and optionally its own green-context SM partition, running the multi-process code path of
the executor (per-rank lists, slot-reuse guards, blocking receives, pair gradient reductions) with
activations / gradients exchanged through peer memory and device-side flags (P:216 blocking
receive, P:222 buffered send).

* bitwise equal to the loopback executor (same kernels; tile results do not depend on the grid
  size and the column reductions partition rows by the device's full SM count);
* fp32 parity with the oracle at S = 8 (1F1B, Interleave v = 2, Chimera) and all levels;
* the ranks really run concurrently (per-rank CUDA-event timelines overlap).
"""
import numpy as np
import pytest
import torch

import synth
from oracle import model as om
from paper_conf_ppopp_liultj25_b200 import api

from .test_gpu_parity import check, rounded

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(600, method="thread")]

TINY8 = synth.with_(synth.TINY_GPT, n_layers=8)
TINY16 = synth.with_(synth.TINY_GPT, n_layers=16)


def run_loopback(cfg, S, N, scheme, level, dtype, params, toks, v=1):
    ctx = api.default_context()
    plan = api.Plan(cfg, S, N, scheme, level, chunks=v, dtype=dtype)
    w, g, ws = api.alloc_for(plan, -1)
    w.copy_(torch.from_numpy(api.pack_params(plan, params, -1)))
    loss = ctx.run_iter(plan, w, toks, g, ws)
    torch.cuda.synchronize()
    return loss, g.cpu().numpy()


class Emu:
    """An emulated context for the duration of a block (the default context is closed first)."""

    def __init__(self, S, sms=0):
        self.S, self.sms = S, sms

    def __enter__(self):
        api.close_default_context()
        self.ctx = api.Context.emulated(self.S, 0, self.sms)
        return self.ctx

    def __exit__(self, *a):
        torch.cuda.synchronize()
        self.ctx.close()


def run_peer(ctx, cfg, S, N, scheme, level, dtype, params, toks, v=1, repeat=1):
    plan = api.Plan(cfg, S, N, scheme, level, chunks=v, dtype=dtype)
    w, g, ws = api.alloc_for(plan, -2)
    w.copy_(torch.from_numpy(api.pack_params(plan, params, -2)))
    outs = []
    for _ in range(repeat):
        loss = ctx.run_iter(plan, w, toks, g, ws)
        torch.cuda.synchronize()
        outs.append((loss, g.cpu().numpy().copy()))
    return plan, outs


CASES = [("1f1b", TINY8, 2, 4, 1), ("1f1b", TINY8, 4, 8, 1), ("1f1b", TINY8, 8, 16, 1),
         ("interleave", TINY16, 8, 16, 2), ("chimera", TINY8, 8, 16, 1), ("chimera", TINY8, 4, 8, 1)]


@pytest.mark.parametrize("sms", [0, 16], ids=["shared-sms", "green-16"])
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("scheme,cfg,S,N,v", CASES, ids=[f"{c[0]}-S{c[2]}" for c in CASES])
def test_peer_bitwise_equals_loopback(scheme, cfg, S, N, v, dtype, sms):
    if sms and S * sms > torch.cuda.get_device_properties(0).multi_processor_count:
        pytest.skip("not enough SMs for the partitions")
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, N)
    ref = {lvl: run_loopback(cfg, S, N, scheme, lvl, dtype, params, toks, v) for lvl in ("base", "mario")}
    with Emu(S, sms) as ctx:
        if sms:
            assert ctx.sms_per_rank >= sms
        for lvl in ("base", "ckpt", "mario"):
            _, outs = run_peer(ctx, cfg, S, N, scheme, lvl, dtype, params, toks, v, repeat=2)
            r = ref["base" if lvl == "base" else "mario"] if lvl != "ckpt" else ref["base"]
            for loss, g in outs:                 # every call: identical bits (flags reset per call)
                assert loss == r[0], (lvl, loss, r[0])
                assert np.array_equal(g, r[1]), lvl


@pytest.mark.parametrize("scheme,cfg,N,v", [("1f1b", TINY8, 16, 1), ("interleave", TINY16, 16, 2),
                                            ("chimera", TINY8, 16, 1)], ids=["1f1b", "interleave", "chimera"])
def test_peer_s8_fp32_oracle_parity(scheme, cfg, N, v):
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, N)
    l_o, g_o = om.step(cfg, params, toks, N, np.float32)
    with Emu(8, 16) as ctx:
        for lvl in ("base", "ckpt", "mario"):
            plan, outs = run_peer(ctx, cfg, 8, N, scheme, lvl, "f32", params, toks, v)
            grads = api.unpack_params(plan, outs[0][1], -2)
            check(outs[0][0], grads, l_o, g_o, 1e-4)


def test_peer_graph_replay_bitwise():
    cfg = synth.with_(synth.tiny_llama(), n_layers=8)
    params = synth.make_weights(cfg)
    toks = [synth.make_tokens(cfg, 8, iteration=i) for i in range(4)]
    with Emu(4, 32) as ctx:
        plan = api.Plan(cfg, 4, 8, "1f1b", "mario", dtype="bf16")
        w, g, ws = api.alloc_for(plan, -2)
        w.copy_(torch.from_numpy(api.pack_params(plan, params, -2)))
        eager = []
        for t in toks:
            l = ctx.run_iter(plan, w, t, g, ws)
            eager.append((l, g.cpu().numpy().copy()))
        ctx.set_graphs(True)
        try:
            for i, t in enumerate(toks):
                l = ctx.run_iter(plan, w, t, g, ws)
                assert l == eager[i][0]
                assert np.array_equal(g.cpu().numpy(), eager[i][1]), i
        finally:
            ctx.set_graphs(False)


def test_peer_ranks_run_concurrently():
    """Per-rank event timelines of an emulated 4-stage 1F1B iteration overlap in time: while one
    rank computes, another does too (a loopback iteration never overlaps)."""
    cfg = synth.with_(synth.GPT3_1P3B, n_layers=4, micro_batch=1, seq_len=1024, hidden=1024, n_heads=8,
                      ffn_hidden=4096, vocab=8192)
    params = synth.make_weights(cfg, parity=False)
    toks = synth.make_tokens(cfg, 8)
    with Emu(4, 32) as ctx:
        plan, _ = run_peer(ctx, cfg, 4, 8, "1f1b", "mario", "bf16", params, toks)
        ctx.set_timing(True)
        run_peer(ctx, cfg, 4, 8, "1f1b", "mario", "bf16", params, toks)
        ctx.set_timing(False)
        tl = [ctx.last_timeline(d) for d in range(4)]
    iv = [(a, b, d) for d in range(4) for a, b in zip(*tl[d])]
    overlap = 0.0
    for i, (a0, b0, d0) in enumerate(iv):
        for a1, b1, d1 in iv[i + 1:]:
            if d1 != d0:
                overlap += max(0.0, min(b0, b1) - max(a0, a1))
    busy = sum(b - a for a, b, _ in iv)
    assert overlap > 0.2 * busy, (overlap, busy)


def test_profile_then_simulate_matches_measured():
    """P:242-252 in the library: time an emulated 4-stage iteration, read the per-virtual-stage costs
    back (mario_last_costs), re-plan with them and compare the simulator's makespan and bubble with
    the measured per-rank timelines (the emulated pipeline: real concurrency, real p2p)."""
    cfg = synth.with_(synth.GPT3_1P3B, n_layers=4, micro_batch=1, seq_len=1024, hidden=1024, n_heads=8,
                      ffn_hidden=4096, vocab=8192)
    params = synth.make_weights(cfg, parity=False)
    toks = synth.make_tokens(cfg, 8)
    with Emu(4, 32) as ctx:
        plan, _ = run_peer(ctx, cfg, 4, 8, "1f1b", "mario", "bf16", params, toks)
        ctx.set_timing(True)
        run_peer(ctx, cfg, 4, 8, "1f1b", "mario", "bf16", params, toks)
        ctx.set_timing(False)
        tl = [ctx.last_timeline(d) for d in range(4)]
        costs = ctx.last_costs(plan)
    assert all(x > 0 for x in costs["fw_ms"] + costs["bw_ms"])
    measured = max(max(b) for _, b in tl)
    sim = api.Plan(cfg, 4, 8, "1f1b", "mario", dtype="bf16", costs=costs).simulate()
    assert abs(sim.makespan_ms - measured) <= 0.15 * measured, (sim.makespan_ms, measured)


@pytest.mark.slow
def test_peer_cfg2_width_bitwise_equals_loopback():
    """Real message sizes and the production kernels on SM partitions: GPT-3 1.3B width (h 2048,
    s 2048, V 50304), 4 layers over 4 ranks of 32 SMs, N = 8, Mario 1F1B, bf16: bitwise the
    loopback result (8 MB activation / gradient messages through the peer transport)."""
    cfg = synth.with_(synth.GPT3_1P3B, n_layers=4, micro_batch=1)
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 8)
    ref = run_loopback(cfg, 4, 8, "1f1b", "mario", "bf16", params, toks)
    with Emu(4, 32) as ctx:
        _, outs = run_peer(ctx, cfg, 4, 8, "1f1b", "mario", "bf16", params, toks, repeat=2)
    for loss, g in outs:
        assert loss == ref[0]
        assert np.array_equal(g, ref[1])


def test_peer_training_loop_bitwise_equals_loopback():
    """Five iterations of run_iter + mario_adamw_step on the emulated 4-stage pipeline (SM partitions,
    CUDA-graph replay from the second call) follow the loopback executor bit for bit: weights, losses
    and grads, while the weights change under the captured graph every iteration."""
    cfg = synth.with_(synth.tiny_llama(), n_layers=4)
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 8)

    def loop(ctx, rank):
        plan = api.Plan(cfg, 4, 8, "1f1b", "mario", dtype="bf16")
        w, g, ws = api.alloc_for(plan, rank)
        w.copy_(torch.from_numpy(api.pack_params(plan, params, rank)))
        m_, v_ = torch.zeros_like(w), torch.zeros_like(w)
        ctx.set_graphs(True)
        losses = []
        try:
            for it in range(1, 6):
                losses.append(ctx.run_iter(plan, w, toks, g, ws))
                api.adamw_step(w, g, m_, v_, it, lr=3e-3)
        finally:
            ctx.set_graphs(False)
        torch.cuda.synchronize()
        return losses, w.cpu().numpy(), g.cpu().numpy()

    ref = loop(api.default_context(), -1)
    with Emu(4, 32) as ctx:
        got = loop(ctx, -2)
    assert got[0] == ref[0]
    assert np.array_equal(got[1], ref[1]) and np.array_equal(got[2], ref[2])
    assert ref[0][-1] < ref[0][0]
