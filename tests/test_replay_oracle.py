"""Pin (SURVEY §8(c) c4 "Pipelining (2)"): executing a plan's per-device lists on the CPU with the
paper's FW / CFW / RC / BW semantics (oracle/replay.py) gives the plain definition's loss and
gradients (oracle/model.py step) — checkpointing only replays the forward and the pipeline
flushes. Every parameter whose contributions arrive in micro-batch order is BITWISE equal
(one copy per parameter, same numpy ops on the same inputs); a tied GPT wte (an input copy on
stage 0 and a head copy on the last stage, reading A8) and Chimera's two replicas differ only
by the association of the final copy sum. Negative cases: lists that break the semantics raise."""
import numpy as np
import pytest

import synth
from oracle import model as om
from oracle import replay as orp
from oracle import schedule as osch

TINY4 = synth.TINY_GPT                                   # L 4
TINY4_L = synth.tiny_llama()


def lists_for(scheme, S, N, v, level):
    pipe = osch.Pipe(scheme, S, N, v)
    return pipe, osch.transform(pipe, level)


def multi_copy(cfg, pipe):
    names = {}
    parts = 2 if pipe.scheme == osch.X_CHIMERA else pipe.v
    for d in range(pipe.S):
        for p in range(parts):
            for n in orp.stage_param_names(cfg, pipe, pipe.vstage(d, p)):
                names[n] = names.get(n, 0) + 1
    return {n for n, c in names.items() if c > 1}


@pytest.mark.parametrize("cfg", [TINY4, TINY4_L], ids=["gpt", "llama"])
@pytest.mark.parametrize("scheme,S,N,v", [("1f1b", 2, 4, 1), ("1f1b", 4, 8, 1), ("interleave", 2, 4, 2)])
@pytest.mark.parametrize("level", ["base", "ckpt", "mario"])
def test_replay_bitwise_plain_accumulation(cfg, scheme, S, N, v, level):
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, N)
    pipe, lists = lists_for(scheme, S, N, v, level)
    loss, grads, _ = orp.replay(cfg, params, toks, pipe, lists, np.float32)
    l_o, g_o = om.step(cfg, params, toks, N, np.float32)
    assert loss == l_o
    tied = multi_copy(cfg, pipe)
    assert tied == ({"wte"} if cfg.family == "gpt" else set())
    for k, v_ in g_o.items():
        if k in tied:
            assert np.abs(grads[k] - v_).max() <= 1e-6 * np.abs(v_).max(), k
        else:
            assert np.array_equal(grads[k], v_), k


@pytest.mark.parametrize("S,N", [(2, 4), (4, 4), (4, 8)])
@pytest.mark.parametrize("level", ["base", "ckpt", "mario"])
def test_replay_chimera_replica_sum(S, N, level):
    """Chimera: two replicas per parameter (down stage d on worker d, up stage on D-1-d);
    fp64 so the replica-sum association is the only difference (<= 1e-12 relative)."""
    cfg = TINY4
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, N)
    pipe, lists = lists_for("chimera", S, N, 1, level)
    loss, grads, copies = orp.replay(cfg, params, toks, pipe, lists, np.float64)
    l_o, g_o = om.step(cfg, params, toks, N, np.float64)
    assert abs(loss - l_o) <= 1e-13 * abs(l_o)
    for k, v_ in g_o.items():
        assert np.abs(grads[k] - v_).max() <= 1e-12 * np.abs(v_).max(), k
    # each replica saw exactly its own pipeline's micro-batches: both are nonzero
    assert all(np.abs(c["h0.qkv.w"]).max() > 0 for (d, p), c in copies.items() if "h0.qkv.w" in c)


def test_replay_mario_equals_base_bitwise_s8():
    """S = 8, N = 16, L = 8: every Mario level replays to the base plan's grads bit for bit."""
    cfg = synth.with_(TINY4, n_layers=8, seq_len=8, vocab=64, hidden=32, n_heads=2, ffn_hidden=64)
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 16)
    ref = None
    for level in ("base", "ckpt", "mario"):
        pipe, lists = lists_for("1f1b", 8, 16, 1, level)
        loss, grads, _ = orp.replay(cfg, params, toks, pipe, lists, np.float32)
        if ref is None:
            ref = (loss, grads)
        else:
            assert loss == ref[0]
            assert all(np.array_equal(grads[k], ref[1][k]) for k in grads)


def test_replay_rejects_broken_semantics():
    cfg = TINY4
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 4)
    pipe, lists = lists_for("1f1b", 2, 4, 1, "mario")
    # drop one RC: its BW has no activations
    bad = [list(L) for L in lists]
    i = next(j for j, x in enumerate(bad[0]) if x[0] == osch.RC)
    del bad[0][i]
    with pytest.raises(AssertionError):
        orp.replay(cfg, params, toks, pipe, bad, np.float32)
    # RC after its BW
    bad = [list(L) for L in lists]
    i = next(j for j, x in enumerate(bad[0]) if x[0] == osch.RC)
    rc = bad[0].pop(i)
    j = bad[0].index((osch.BW, rc[1], rc[2]))
    bad[0].insert(j + 1, rc)
    with pytest.raises(AssertionError):
        orp.replay(cfg, params, toks, pipe, bad, np.float32)
    # a receive that can never be satisfied (its send removed) deadlocks
    bad = [list(L) for L in lists]
    bad[0] = [x for x in bad[0] if not (x[0] == osch.SA and x[1] == 1)]
    with pytest.raises((RuntimeError, AssertionError)):
        orp.replay(cfg, params, toks, pipe, bad, np.float32)


def test_replay_prepose_negative_case_deadlocks():
    """SURVEY c4 Planner (5): preposing CFW_2, CFW_3 on device 2 alone at S = N = 4 creates a cycle
    (the simulator returns None, tests/test_schedule_oracle.py); executing those lists stalls."""
    pipe = osch.Pipe("1f1b", 4, 4)
    L = osch.pass3_remove_redundancy(osch.pass2_overlap_recompute(osch.pass1_apply_checkpoint(
        osch.build_base(pipe))))
    bad = ((osch.RA, 2, 0), (osch.CFW, 2, 0), (osch.RA, 3, 0), (osch.CFW, 3, 0))
    d2 = [x for x in L[2] if x not in bad]
    i = d2.index((osch.SA, 1, 0)) + 1
    d2[i:i] = list(bad)
    L[2] = d2
    assert osch.simulate(pipe, L, osch.UnitCosts()) is None
    cfg = synth.with_(TINY4, seq_len=8)
    with pytest.raises(RuntimeError):
        orp.replay(cfg, synth.make_weights(cfg), synth.make_tokens(cfg, 4), pipe, L, np.float32)
