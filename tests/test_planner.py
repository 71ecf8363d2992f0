"""The C++ planner behind the C-ABI (mario_plan) must emit exactly the schedule oracle's
lists (oracle/schedule.py) and reproduce its simulated makespans; plus ABI checks. CPU only:
the planner is host code, no GPU is touched."""
import os

import numpy as np
import pytest

import synth
from oracle import schedule as osch
from paper_conf_ppopp_liultj25_b200 import _lib
from paper_conf_ppopp_liultj25_b200 import api
from paper_conf_ppopp_liultj25_b200.api import MarioError, Plan

TINY = synth.TINY_GPT
OP_SCHEME = {"1f1b": osch.V_1F1B, "interleave": osch.W_INTERLEAVE, "chimera": osch.X_CHIMERA}


def unit_costs(K, F=1.0, B=2.0, R=1.0, comm=0.0):
    return {"fw_ms": [F] * K, "bw_ms": [B] * K, "rc_ms": [R] * K, "p2p_alpha_ms": comm, "p2p_GBps": 0.0,
            "act_bytes": [1.0] * K, "ckpt_bytes": [0.0] * K, "work_bytes": [0.0] * K, "static_bytes": 0.0}


def model_for(L):
    return synth.with_(TINY, n_layers=L)


CASES = [("1f1b", 4, 4, 1), ("1f1b", 2, 4, 1), ("1f1b", 4, 8, 1), ("1f1b", 8, 8, 1), ("1f1b", 3, 5, 1),
         ("interleave", 4, 4, 2), ("interleave", 4, 8, 2), ("interleave", 2, 4, 2), ("chimera", 4, 4, 1),
         ("chimera", 4, 8, 1), ("chimera", 2, 4, 1)]


@pytest.mark.parametrize("level", ["base", "ckpt", "mario"])
@pytest.mark.parametrize("scheme,S,N,v", CASES)
def test_lists_match_oracle(scheme, S, N, v, level):
    K = S * v
    pipe = osch.Pipe(OP_SCHEME[scheme], S, N, v)
    F = 1.0 / v
    c = osch.UnitCosts(F=F, B=2 * F, R=F)
    want = osch.transform(pipe, level, c)
    plan = Plan(model_for(K * 2 if scheme != "chimera" else S * 2), S, N, scheme, level, chunks=v, dtype="f32",
                costs=unit_costs(K, F, 2 * F, F))
    assert plan.lists() == want
    assert plan.simulate().makespan_ms == osch.simulate(pipe, want, c).makespan
    for d in range(S):
        a, b = plan.timeline(d)
        r = osch.simulate(pipe, want, c)
        comp = [x for x in want[d] if x[0] in osch.COMPUTE]
        assert a == [r.start[(d,) + x] for x in comp]


@pytest.mark.parametrize("budget", [1, 2, 3, 5, 100])
@pytest.mark.parametrize("scheme,S,N,v", CASES)
def test_budget_level_matches_oracle(scheme, S, N, v, budget):
    """MARIO_LEVEL_BUDGET (f2, reading A28): same lists and tail k as oracle pass5_budget."""
    K = S * v
    pipe = osch.Pipe(OP_SCHEME[scheme], S, N, v)
    F = 1.0 / v
    c = osch.UnitCosts(F=F, B=2 * F, R=F)
    want, k = osch.pass5_budget(pipe, c, osch.MemUnits(), budget)
    try:
        plan = Plan(model_for(K * 2 if scheme != "chimera" else S * 2), S, N, scheme, "mario_budget", chunks=v,
                    dtype="f32", costs=unit_costs(K, F, 2 * F, F), mem_budget=budget)
    except MarioError as e:   # nothing fits: EBUDGET, and the oracle's lists exceed the budget too
        assert e.code == -2
        assert max(osch.memory_walk(pipe, want, osch.MemUnits()).peak) > budget
        return
    assert plan.lists() == want
    assert plan.unckpt_tail == k
    assert plan.simulate().makespan_ms == osch.simulate(pipe, want, c).makespan
    assert "unckpt_tail=%d" % k in plan.serialize()


def test_budget_level_needs_a_budget():
    with pytest.raises(MarioError) as e:
        Plan(model_for(4), 4, 4, "1f1b", "mario_budget", dtype="f32", costs=unit_costs(4))
    assert e.value.code == -1


def test_fig2_through_abi():
    totals = []
    for level in ("base", "ckpt", "mario"):
        p = Plan(model_for(4), 4, 4, "1f1b", level, dtype="f32", costs=unit_costs(4))
        totals.append(p.simulate().makespan_ms)
    assert totals == [21.0, 28.0, 22.0]


def test_memory_counts_match_oracle():
    for scheme, S, N, v in [("1f1b", 8, 16, 1), ("interleave", 4, 8, 2), ("chimera", 4, 8, 1)]:
        pipe = osch.Pipe(OP_SCHEME[scheme], S, N, v)
        for level in ("base", "mario"):
            want = osch.memory_walk(pipe, osch.transform(pipe, level, osch.UnitCosts(F=1 / v, B=2 / v, R=1 / v)),
                                    osch.MemUnits())
            p = Plan(model_for(S * v * (2 if scheme == "chimera" else 1)), S, N, scheme, level, chunks=v,
                     dtype="f32", costs=unit_costs(S * v, 1 / v, 2 / v, 1 / v))
            assert p.simulate().max_live_act == want.max_live_act


def test_budget_matches_oracle_and_ebudget():
    pipe = osch.Pipe(osch.V_1F1B, 4, 4)
    mem = osch.MemUnits(act=10.0, ckpt=1.0, work=0.0)
    c = osch.UnitCosts()
    l3 = osch.pass3_remove_redundancy(osch.pass2_overlap_recompute(osch.pass1_apply_checkpoint(osch.build_base(pipe))))
    budget = max(osch.memory_walk(pipe, l3, mem).peak)
    want = osch.pass4_prepose_forward(pipe, l3, c, mem=mem, budget=budget)
    costs = unit_costs(4)
    costs.update(act_bytes=[10.0] * 4, ckpt_bytes=[1.0] * 4)
    p = Plan(model_for(4), 4, 4, "1f1b", "mario", dtype="f32", costs=costs, mem_budget=int(budget))
    assert p.lists() == want
    with pytest.raises(MarioError) as e:
        Plan(model_for(4), 4, 4, "1f1b", "base", dtype="f32", costs=costs, mem_budget=int(budget) - 1)
    assert e.value.code == -2


def test_serialization_deterministic_and_golden():
    p1 = Plan(model_for(4), 4, 4, "1f1b", "mario", dtype="f32", costs=unit_costs(4))
    p2 = Plan(model_for(4), 4, 4, "1f1b", "mario", dtype="f32", costs=unit_costs(4))
    s = p1.serialize()
    assert s == p2.serialize()
    gold = open(os.path.join(os.path.dirname(__file__), "golden", "plan_fig2_mario.txt")).read()
    assert s == gold


@pytest.mark.parametrize("bad", [dict(stages=3, N=4, L=4),            # L % S != 0
                                 dict(stages=4, N=6, L=8, scheme="interleave", v=2),   # N % S
                                 dict(stages=3, N=6, L=6, scheme="chimera")])          # odd S
def test_einval(bad):
    with pytest.raises(MarioError) as e:
        Plan(model_for(bad["L"]), bad["stages"], bad["N"], bad.get("scheme", "1f1b"), "mario",
             chunks=bad.get("v", 1), dtype="f32")
    assert e.value.code == -1


def test_param_names_match_synth():
    for cfg in (TINY, synth.tiny_llama(), synth.with_(TINY, tie_embeddings=False)):
        p = Plan(cfg, 2, 4, "1f1b", "mario", dtype="f32")
        assert p.param_names() == [n for n, _ in synth.param_shapes(cfg)]


def test_rank_params_cover_model():
    cfg = TINY
    shapes = dict(synth.param_shapes(cfg))
    for scheme, S, v in [("1f1b", 2, 1), ("interleave", 2, 2), ("chimera", 2, 1), ("1f1b", 1, 1)]:
        p = Plan(cfg, S, 2 * S if scheme != "1f1b" else 4, scheme, "mario", chunks=v, dtype="f32")
        seen = {}
        for r in range(S):
            for name, off, cnt in p.rank_params(r):
                assert cnt == int(np.prod(shapes[name]))
                assert off % 64 == 0
                seen[name] = seen.get(name, 0) + 1
        assert set(seen) == set(shapes)
        if scheme == "chimera":
            assert all(v == 2 for k, v in seen.items() if k != "wte") and seen["wte"] == 4
        elif S > 1:
            assert seen["wte"] == 2 and all(v == 1 for k, v in seen.items() if k != "wte")


def test_library_exports_every_declared_symbol():
    """include/*.h declarations are all exported by libmario.so (no compute calls)."""
    import re
    root = os.path.dirname(os.path.dirname(__file__))
    lib = _lib.lib()
    names = []
    for h in ("mario.h", "mario_kernels.h"):
        txt = open(os.path.join(root, "include", h)).read()
        txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
        names += re.findall(r"\b(mario_[a-z0-9_]+)\s*\(", txt)
    assert len(set(names)) > 15
    for n in set(names):
        assert hasattr(lib, n), n


def test_cfg5_memory_cap_base_infeasible_mario_fits():
    """BASELINE.json configs[4]: LLaMA2-13B, s = 16384, 8 stages, 40 GB per GPU (the paper's
    A100-40G): plain 1F1B exceeds the cap on device 0 (Table 1: D x M_theta), full-checkpoint
    1F1B and Mario fit (M_theta per device), and Mario's simulated makespan beats ckpt."""
    cfg = synth.LLAMA2_13B
    cap = 40 * 10 ** 9
    with pytest.raises(MarioError) as e:
        Plan(cfg, 8, 16, "1f1b", "base", dtype="bf16", mem_budget=cap)
    assert e.value.code == -2
    ck = Plan(cfg, 8, 16, "1f1b", "ckpt", dtype="bf16", mem_budget=cap).simulate()
    ma = Plan(cfg, 8, 16, "1f1b", "mario", dtype="bf16", mem_budget=cap).simulate()
    assert max(ma.peak_bytes) <= cap and max(ck.peak_bytes) <= cap
    assert ma.makespan_ms < ck.makespan_ms
    assert ma.max_live_act == [1] * 8
    base = Plan(cfg, 8, 16, "1f1b", "base", dtype="bf16").simulate()
    assert base.max_live_act == [8, 7, 6, 5, 4, 3, 2, 1]            # Table 1
    assert max(base.peak_bytes) / min(base.peak_bytes) > 2.0          # imbalanced
    assert max(ma.peak_bytes) / min(ma.peak_bytes) < 1.25            # balanced (SURVEY d3 bar)


def test_chrome_trace_of_fig2():
    """P:256 visualization: one box per compute instruction, simulated start/finish."""
    import json
    p = Plan(model_for(4), 4, 4, "1f1b", "mario", dtype="f32", costs=unit_costs(4))
    tr = api.chrome_trace(p)
    boxes = [e for e in tr["traceEvents"] if e.get("ph") == "X"]
    assert len(boxes) == sum(1 for d in range(4) for x in p.instrs(d) if x[0] in ("FW", "CFW", "RC", "BW"))
    assert max(e["ts"] + e["dur"] for e in boxes) == 22.0 * 1e3   # Fig. 2 step 4: 22t
    json.dumps(tr)


def test_max_seq_len_boundary_and_order():
    """§6.5 analogue: PP 8, mbs 1, N = 2 x stages, 40 GB cap (the paper's
    A100-40G). The returned s fits and s + 64 does not; freeing activation memory (Mario) admits a
    longer sequence than base 1F1B and no shorter one than naive full checkpointing."""
    cfg = synth.with_(synth.GPT3_1P3B, micro_batch=1)
    cap = 40 * 10 ** 9
    got = {lvl: api.max_seq_len(cfg, 8, 16, lvl, cap) for lvl in ("base", "ckpt", "mario", "mario_budget")}
    for lvl, s in got.items():
        assert s >= 1024 and (s - 1024) % 64 == 0
        Plan(synth.with_(cfg, seq_len=s), 8, 16, "1f1b", lvl, mem_budget=cap)
        with pytest.raises(MarioError):
            Plan(synth.with_(cfg, seq_len=s + 64), 8, 16, "1f1b", lvl, mem_budget=cap)
    assert got["mario"] > 1.3 * got["base"]
    assert got["mario"] >= got["ckpt"] and got["mario_budget"] >= got["mario"]
    assert api.max_seq_len(cfg, 8, 16, "base", 10 ** 6) == 0


def test_store_act_default_and_lean_fallback(monkeypatch):
    """Activation sets keep the norm outputs A, A2 (+2 [T, h] per layer) unless the budget needs
    the lean set: a budget between the lean and the stored peak plans the lean set instead of
    failing; MARIO_STORE_ACT forces either."""
    cfg = synth.with_(synth.GPT3_1P3B, n_layers=8, micro_batch=1)
    full = Plan(cfg, 4, 8, "1f1b", "mario")
    assert full.store_act
    monkeypatch.setenv("MARIO_STORE_ACT", "0")
    lean = Plan(cfg, 4, 8, "1f1b", "mario")
    assert not lean.store_act
    monkeypatch.delenv("MARIO_STORE_ACT")
    p_full, p_lean = max(full.simulate().peak_bytes), max(lean.simulate().peak_bytes)
    assert p_full > p_lean   # + A, A2 per stored layer, - the lean transients (Arec, CFW A/A2)
    mid = Plan(cfg, 4, 8, "1f1b", "mario", mem_budget=(p_full + p_lean) // 2)
    assert not mid.store_act and max(mid.simulate().peak_bytes) <= (p_full + p_lean) // 2
    assert mid.lists() == lean.lists()
    with pytest.raises(MarioError) as e:
        Plan(cfg, 4, 8, "1f1b", "mario", mem_budget=p_lean // 2)
    assert e.value.code == -2
