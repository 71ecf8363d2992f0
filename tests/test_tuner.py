"""mario_tune: the schedule tuner of PAPER.md §5.3 / Eq. 1. CPU only."""
import math

import pytest

import synth
from paper_conf_ppopp_liultj25_b200 import api


def test_every_row_matches_a_directly_built_plan():
    cfg = synth.with_(synth.GPT3_1P3B, n_layers=8)
    rows, best = api.tune(cfg, 4, 32)
    assert best >= 0 and len(rows) > 8
    for r in rows[:12]:
        c = synth.with_(cfg, micro_batch=r["micro_batch"])
        K = r["pp"] * r["chunks"]
        lps = c.n_layers // K
        # analytic costs as the tuner derives them (FLOPs at 1 PFLOP/s; RC = FW)
        p0 = api.Plan(c, r["pp"], r["microbatches"], r["scheme"], r["level"], chunks=r["chunks"])
        assert p0.simulate().makespan_ms == pytest.approx(r["makespan_ms"], rel=1e-12)
        assert max(p0.simulate().peak_bytes) == r["peak_bytes"]


def test_oom_configs_score_zero_and_cfg5_picks_mario():
    """F = 0 when the estimated peak exceeds device memory. LLaMA2-13B at s = 16384 with the
    paper's 40 GB devices: every no-checkpoint configuration is infeasible; the tuner picks Mario."""
    rows, best = api.tune(synth.LLAMA2_13B, 8, 16, mem_budget=40 * 10 ** 9)
    for r in rows:
        assert (r["samples_per_s"] == 0.0) == (not r["feasible"])
        if r["level"] == "base":
            assert not r["feasible"]
    assert best >= 0 and rows[best]["level"] in ("mario", "mario_budget") and rows[best]["feasible"]


def test_lmbs_freed_memory_buys_a_larger_microbatch():
    """The paper's lmbs: Mario frees activation memory, so under the same budget it
    can run a larger micro-batch, which a larger-is-more-efficient cost table (as profiled on a
    GPU) rewards. Per-layer costs: t(mbs) = mbs * t1 * (1 - 0.12 log2 mbs)."""
    cfg = synth.GPT3_1P3B
    mbs = [1, 2, 4, 8]
    t1 = 0.35
    eff = [1 - 0.12 * math.log2(m) for m in mbs]
    costs = {"mbs": mbs, "layer_fw_ms": [m * t1 * e for m, e in zip(mbs, eff)],
             "layer_bw_ms": [2 * m * t1 * e for m, e in zip(mbs, eff)],
             "head_fw_ms": [m * 1.2 * e for m, e in zip(mbs, eff)],
             "head_bw_ms": [2 * m * 1.2 * e for m, e in zip(mbs, eff)], "p2p_alpha_ms": 0.02, "p2p_GBps": 770.0}
    rows_free, b_free = api.tune(cfg, 8, 128, costs=costs)
    budget = 20 * 10 ** 9
    rows, best = api.tune(cfg, 8, 128, mem_budget=budget, costs=costs)
    assert best >= 0
    win = rows[best]
    # the best feasible base configuration uses a smaller micro-batch than the winner
    feas_base = [r for r in rows if r["level"] == "base" and r["feasible"]]
    assert win["level"] in ("mario", "mario_budget")
    assert not feas_base or max(r["micro_batch"] for r in feas_base) < win["micro_batch"] or \
        max(r["samples_per_s"] for r in feas_base) < win["samples_per_s"]
    assert win["peak_bytes"] <= budget


def test_tune_rejects_bad_arguments():
    with pytest.raises(api.MarioError):
        api.tune(synth.TINY_GPT, 0, 8)


def test_budget_level_in_grid_never_worse_than_mario():
    """With a budget, MARIO_LEVEL_BUDGET (reading A28) joins the grid; per grid point it is never
    slower than plain Mario (k = 0 is one of its candidates) and always within the budget."""
    budget = 20 * 10 ** 9
    rows, best = api.tune(synth.GPT3_1P3B, 8, 128, mem_budget=budget)
    key = lambda r: (r["scheme"], r["pp"], r["chunks"], r["dp"], r["micro_batch"])
    mario = {key(r): r for r in rows if r["level"] == "mario"}
    n = 0
    for r in rows:
        if r["level"] != "mario_budget" or not r["feasible"]:
            continue
        n += 1
        assert r["peak_bytes"] <= budget
        m = mario[key(r)]
        if m["feasible"]:
            assert r["makespan_ms"] <= m["makespan_ms"] + 1e-9
    assert n > 0
    _, b0 = api.tune(synth.GPT3_1P3B, 8, 128)
    assert all(r["level"] != "mario_budget" for r in api.tune(synth.GPT3_1P3B, 8, 128)[0])


@pytest.mark.gpu
def test_profile_costs_measured_estimators_drive_the_tuner():
    """P:242 profile step inside the library (api.profile_costs): measured per-layer / head costs per
    micro-batch size, then mario_tune (Eq. 1) on them. Costs are positive, a micro-batch 4x larger
    costs more per layer, and the tuner finds a feasible configuration under 40 GB."""
    cfg = synth.with_(synth.GPT3_1P3B, seq_len=1024)
    costs = api.profile_costs(cfg, (1, 4))
    assert costs["mbs"] == [1, 4]
    for k in ("layer_fw_ms", "layer_bw_ms"):
        assert all(v > 0 for v in costs[k]), costs
        assert costs[k][1] > costs[k][0], costs
    assert all(v >= 0 for v in costs["head_fw_ms"] + costs["head_bw_ms"])
    rows, best = api.tune(cfg, 8, 64, mem_budget=40 * 10 ** 9, costs=costs)
    assert best >= 0 and rows[best]["feasible"] and rows[best]["micro_batch"] in (1, 4)
