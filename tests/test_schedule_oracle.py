"""Pins for oracle/schedule.py: the paper's Fig. 2 totals, closed forms derived from the
schedule definitions, Table 1's in-flight bounds, the deadlock negative case and
structural invariants (SURVEY §8(c) c4 'Planner / simulator')."""
import os

import pytest

from oracle.schedule import (BASE, CKPT, MARIO, MARIO_BUDGET, BW, CFW, FW, RA, RC, RG, SA, SG, V_1F1B,
                             W_INTERLEAVE, X_CHIMERA, MemUnits, Pipe, UnitCosts, build_base,
                             check_structure, find_inst, memory_walk, pass1_apply_checkpoint,
                             pass2_overlap_recompute, pass3_remove_redundancy,
                             pass4_prepose_forward, pass5_budget, simulate, transform)

from oracle import schedule as S

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _fig2_gold():
    out = {}
    for line in open(os.path.join(GOLD, "fig2_totals.txt")):
        line = line.split("#")[0].split()
        if line:
            out[line[0]] = float(line[1])
    return out


def test_fig2_totals_match_paper():
    """21t -> 28t -> 25t -> 23t -> 22t (4 stages, 4 micro-batches, B=2F, RC=F)."""
    g = _fig2_gold()
    pipe, c = Pipe(V_1F1B, 4, 4), UnitCosts(F=1, B=2, R=1, comm=0)
    l0 = build_base(pipe)
    l1 = pass1_apply_checkpoint(l0)
    l2 = pass2_overlap_recompute(l1)
    l3 = pass3_remove_redundancy(l2)
    l4 = pass4_prepose_forward(pipe, l3, c)
    got = [simulate(pipe, L, c).makespan for L in (l0, l1, l2, l3, l4)]
    assert got == [g["base"], g["step1_ckpt"], g["step2"], g["step3"], g["step4"]]
    for L in (l0, l1, l2, l3, l4):
        check_structure(pipe, L)


@pytest.mark.parametrize("S,N", [(2, 4), (4, 4), (4, 8), (8, 8), (8, 32), (3, 5)])
def test_1f1b_closed_forms(S, N):
    """base (N+S-1)(F+B); CKPT (N+S-1)(F+B+R); MARIO (S-2)(F+B) + N(F+B+R)."""
    pipe, c = Pipe(V_1F1B, S, N), UnitCosts()
    base = simulate(pipe, transform(pipe, BASE), c).makespan
    ckpt = simulate(pipe, transform(pipe, CKPT), c).makespan
    mario = simulate(pipe, transform(pipe, MARIO, c), c).makespan
    assert base == (N + S - 1) * 3
    assert ckpt == (N + S - 1) * 4
    assert mario == (S - 2) * 3 + N * 4


@pytest.mark.parametrize("S,N", [(4, 4), (4, 8), (8, 8), (8, 16)])
def test_interleave_closed_form(S, N):
    """Interleave with v chunks, per-chunk F=1/v, B=2/v: makespan (N*v + S - 1)(F+B)/v."""
    v = 2
    pipe, c = Pipe(W_INTERLEAVE, S, N, v), UnitCosts(F=0.5, B=1.0, R=0.5)
    assert simulate(pipe, transform(pipe, BASE), c).makespan == (N * v + S - 1) * 1.5


def test_mario_between_base_and_ckpt_all_schemes():
    for pipe, c in [(Pipe(V_1F1B, 4, 8), UnitCosts()),
                    (Pipe(W_INTERLEAVE, 4, 8, 2), UnitCosts(F=0.5, B=1, R=0.5)),
                    (Pipe(X_CHIMERA, 4, 8), UnitCosts())]:
        b = simulate(pipe, transform(pipe, BASE), c).makespan
        k = simulate(pipe, transform(pipe, CKPT), c).makespan
        mm = transform(pipe, MARIO, c)
        check_structure(pipe, mm)
        m = simulate(pipe, mm, c).makespan
        assert b <= m < k, (pipe, b, m, k)


@pytest.mark.parametrize("S,N", [(4, 4), (4, 8), (8, 32)])
def test_table1_1f1b_inflight(S, N):
    """Table 1: 1F1B holds [1, D] activation sets; device d holds S-d. Mario: 1."""
    pipe = Pipe(V_1F1B, S, N)
    live = memory_walk(pipe, transform(pipe, BASE), MemUnits()).max_live_act
    assert live == [min(S - d, N) for d in range(S)]
    live_m = memory_walk(pipe, transform(pipe, MARIO), MemUnits()).max_live_act
    assert live_m == [1] * S


@pytest.mark.parametrize("S", [4, 8])
def test_table1_interleave_inflight(S):
    """Table 1 with reading A18: Megatron order gives 3S-1 chunk activations on
    device 0 down to S+1 on the last device (N > S). Mario: 1 chunk activation (M_theta/2)."""
    pipe = Pipe(W_INTERLEAVE, S, 2 * S, 2)
    live = memory_walk(pipe, transform(pipe, BASE), MemUnits()).max_live_act
    assert live == [2 * (S - 1 - d) + S + 1 for d in range(S)]
    assert live[0] == 3 * S - 1 and live[-1] == S + 1


@pytest.mark.parametrize("D", [4, 8])
def test_table1_chimera_inflight(D):
    """Table 1: Chimera holds [(D/2+1), D] activation sets per worker; 2 weight replicas."""
    pipe = Pipe(X_CHIMERA, D, 2 * D)
    live = memory_walk(pipe, transform(pipe, BASE), MemUnits()).max_live_act
    assert min(live) == D // 2 + 1 and max(live) == D
    check_structure(pipe, transform(pipe, BASE))


def test_prepose_on_stage2_alone_deadlocks():
    """Negative case [derived]: preposing CFW_2, CFW_3 on device 2 only (S=N=4) creates a
    dependency cycle, which the simulator must report (returns None)."""
    pipe, c = Pipe(V_1F1B, 4, 4), UnitCosts()
    L = pass3_remove_redundancy(pass2_overlap_recompute(pass1_apply_checkpoint(build_base(pipe))))
    d2 = [x for x in L[2] if x not in ((RA, 2, 0), (CFW, 2, 0), (RA, 3, 0), (CFW, 3, 0))]
    i = d2.index((SA, 1, 0)) + 1
    d2[i:i] = [(RA, 2, 0), (CFW, 2, 0), (RA, 3, 0), (CFW, 3, 0)]
    L[2] = d2
    assert simulate(pipe, L, c) is None


def test_algorithm1_matches_vstage_geometry():
    """find_prev/next (Alg. 1) must land on the owner of virtual stage k-1 / k+1."""
    for pipe in (Pipe(V_1F1B, 4, 4), Pipe(W_INTERLEAVE, 4, 4, 2), Pipe(X_CHIMERA, 4, 4)):
        for m in range(pipe.N):
            pl = pipe.part_of_micro(m)
            for k in range(pipe.K):
                d, p = pipe.device_part(k, pl)
                nx = find_inst(pipe, d, m, p, FW, nxt=True)
                pv = find_inst(pipe, d, m, p, FW, nxt=False)
                if k + 1 < pipe.K:
                    assert (nx[0], nx[2]) == pipe.device_part(k + 1, pl)
                else:
                    assert nx is None
                if k > 0:
                    assert (pv[0], pv[2]) == pipe.device_part(k - 1, pl)
                else:
                    assert pv is None
                # BW runs the opposite direction
                assert find_inst(pipe, d, m, p, BW, nxt=True) == (None if k == 0 else (pv[0], m, pv[2], BW))


def test_passes_keep_bw_order_and_rc_before_rg():
    pipe = Pipe(V_1F1B, 8, 16)
    base = transform(pipe, BASE)
    mm = transform(pipe, MARIO)
    for d in range(8):
        assert [x for x in base[d] if x[0] == BW] == [x for x in mm[d] if x[0] == BW]
        for op, m, p in mm[d]:
            if op == RC and (RG, m, p) in mm[d]:
                assert mm[d].index((RC, m, p)) < mm[d].index((RG, m, p))


def test_budget_blocks_prepose():
    """With a budget of one checkpoint beyond base-ckpt usage, pass 4 cannot prepose."""
    pipe, c = Pipe(V_1F1B, 4, 4), UnitCosts()
    mem = MemUnits(act=10.0, ckpt=1.0, work=0.0)
    l3 = pass3_remove_redundancy(pass2_overlap_recompute(pass1_apply_checkpoint(build_base(pipe))))
    peak3 = max(memory_walk(pipe, l3, mem).peak)
    l4 = pass4_prepose_forward(pipe, l3, c, mem=mem, budget=peak3)
    assert max(memory_walk(pipe, l4, mem).peak) <= peak3
    assert simulate(pipe, l4, c).makespan >= 22


# ------------------------------------------------ budget-driven partial checkpointing (f2, A28)
def _tail_makespan(S, N, k):
    """[derived] 1F1B, F = 1, B = 2, RC = 1: Mario's closed form (S-2)(F+B) + N(F+B+R) for k <= 1;
    each further un-checkpointed tail device takes one RC off the critical path (3 units, SURVEY d4:
    146 -> 143 -> ... -> 128 at S = 8, N = 32), never below base (N+S-1)(F+B); k = S is base."""
    mario_t, base_t = (S - 2) * 3 + N * 4, (N + S - 1) * 3
    if k <= 1:
        return mario_t
    return base_t if k == S else max(base_t, mario_t - 3 * (k - 1))


@pytest.mark.parametrize("S,N", [(4, 8), (4, 16), (6, 12), (8, 16)])
def test_budget_tail_1f1b_closed_form(S, N):
    """A tail device d keeps its base in-flight count S - d (Table 1), so a budget of b activation
    sets admits tails k <= b; the level picks the fastest, ties to the smaller k."""
    pipe, c, mem = Pipe(V_1F1B, S, N), UnitCosts(), MemUnits()
    for b in range(1, S + 1):
        L, k = pass5_budget(pipe, c, mem, b)
        check_structure(pipe, L)
        ks = [0] + list(range(2, min(b, S) + 1))
        want_t = min(_tail_makespan(S, N, j) for j in ks)
        want_k = min(j for j in ks if _tail_makespan(S, N, j) == want_t)
        assert (k, simulate(pipe, L, c).makespan) == (want_k, want_t)
        peaks = memory_walk(pipe, L, mem).peak
        assert peaks == [float(S - d) if d >= S - k else 1.0 for d in range(S)]
        if k == S:
            assert L == build_base(pipe)


def test_budget_tail_survey_sequence():
    """SURVEY d4 [derived]: S = 8, N = 32, budgets of 2 .. 7 activation sets."""
    pipe, c, mem = Pipe(V_1F1B, 8, 32), UnitCosts(), MemUnits()
    got = [simulate(pipe, pass5_budget(pipe, c, mem, b)[0], c).makespan for b in (2, 4, 7)]
    assert got == [143, 137, 128]


def test_budget_tail_picks_fastest_not_largest():
    """Chimera S = 4, N = 8: un-checkpointing only the last device lengthens the schedule
    (38 > 36), so with room for it the rule still keeps k = 0 (smallest makespan, ties to k);
    with room for three un-checkpointed tails it reaches the base makespan (32)."""
    pipe, c, mem = Pipe(X_CHIMERA, 4, 8), UnitCosts(), MemUnits()
    L0 = transform(pipe, MARIO, c)
    L, k = pass5_budget(pipe, c, mem, 3)
    assert k == 0 and L == L0
    L, k = pass5_budget(pipe, c, mem, 4)
    assert k in (3, 4) and simulate(pipe, L, c).makespan == simulate(pipe, build_base(pipe), c).makespan == 32


def test_budget_level_keeps_invariants_all_schemes():
    c, mem = UnitCosts(F=0.5, B=1.0, R=0.5), MemUnits()
    for pipe in (Pipe(V_1F1B, 4, 8), Pipe(W_INTERLEAVE, 4, 8, 2), Pipe(X_CHIMERA, 4, 8)):
        for b in (1, 2, 4, 6, 12):
            L = transform(pipe, MARIO_BUDGET, c, mem, b)
            check_structure(pipe, L)
            assert simulate(pipe, L, c) is not None
            # never slower than the paper's passes when those fit
            assert simulate(pipe, L, c).makespan <= simulate(pipe, transform(pipe, MARIO, c, mem, b), c).makespan


@pytest.mark.parametrize("D", [4, 6, 8, 16])
def test_chimera_unit_closed_form(D):
    """Chimera's own bubble count ([23], the scheme PAPER.md P:61 cites): one basic unit of N = D
    micro-batches on D workers, forward and backward of equal cost, finishes in 2N + D - 2 slots
    (each worker is busy 2N and idles D - 2), against 2N + 2(D - 1) for 1F1B. Built and simulated at
    F = B = 1 (the production order is the same greedy at F = 1, B = 2)."""
    pipe = S.Pipe(S.X_CHIMERA, D, D)
    lists = S.build_chimera(pipe, F=1.0, B=1.0)
    S.check_structure(pipe, lists)
    r = S.simulate(pipe, lists, S.UnitCosts(F=1.0, B=1.0))
    assert r.makespan == 2 * D + D - 2
    one = S.simulate(S.Pipe(S.V_1F1B, D, D), S.build_1f1b(S.Pipe(S.V_1F1B, D, D)), S.UnitCosts(F=1.0, B=1.0))
    assert one.makespan == 2 * D + 2 * (D - 1)
