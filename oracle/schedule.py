"""ORACLE (test infrastructure only) — Mario's pipeline-schedule transformations and simulator.

Written step by step in the paper's order and notation, independent of the C++ planner
(`paper_conf_ppopp_liultj25_b200/csrc/plan/`), which must emit byte-identical lists.

- IR (Table 3): per-device ordered list of instructions
  (op, micro_id m, part_id p). Ops: FW, CFW, RC, BW, SA, RA, SG, RG.
- Base schemes: 1F1B "V" (Megatron order), Interleave "W" (Megatron
  interleaved order, reading A9), Chimera "X" (bidirectional, reading A10 — the order is
  defined outside PAPER.md; pinned by Chimera's basic-unit bubble count D - 2 at F = B).
- Passes (§5.1): pass 1 apply-checkpoint, pass 2 overlap-recompute,
  pass 3 remove-redundancy, pass 4 prepose-forward with the SA rule;
  applied iteratively. Readings A14-A17 fix the details the paper leaves open.
- Virtual pipeline + Algorithm 1 find_prev/next (garbled; readings A9/A11).
- DP timeline: start(I) = max(finish of horizontal predecessor (list order),
  finish of vertical predecessor (+ p2p time)); sends are buffered (per-channel FIFO) and
  a send is posted when the compute preceding it in its list has finished (reading A12).
- Memory walk (reading A13): list-order accounting of live checkpoints and
  activation sets.

Pins: tests/test_schedule_oracle.py — Fig. 2 totals 21/28/25/23/22, closed
forms, Table 1 in-flight bounds, structural invariants.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Tuple

FW, CFW, RC, BW, SA, RA, SG, RG = "FW", "CFW", "RC", "BW", "SA", "RA", "SG", "RG"
COMPUTE = (FW, CFW, RC, BW)
RECV = (RA, RG)
SEND = (SA, SG)

V_1F1B, W_INTERLEAVE, X_CHIMERA = "1f1b", "interleave", "chimera"
BASE, CKPT, MARIO = "base", "ckpt", "mario"
MARIO_BUDGET = "mario_budget"   # extension (reading A28)

Instr = Tuple[str, int, int]  # (op, micro, part)


@dataclass
class Pipe:
    """Geometry of the virtual pipeline."""
    scheme: str
    S: int          # devices (= pipeline stages per pipeline)
    N: int          # micro-batches
    v: int = 1      # Interleave chunks per device

    @property
    def K(self) -> int:
        """Number of virtual stages of one pipeline."""
        return self.S * self.v if self.scheme == W_INTERLEAVE else self.S

    def part_of_micro(self, m: int) -> int:
        """Chimera: micro-batches of each basic unit of D go first D/2 down (p=0), then up (p=1)."""
        if self.scheme != X_CHIMERA:
            return 0
        return 0 if (m % self.S) < self.S // 2 else 1

    def vstage(self, d: int, p: int) -> int:
        if self.scheme == V_1F1B:
            return d
        if self.scheme == W_INTERLEAVE:
            return p * self.S + d
        return d if p == 0 else self.S - 1 - d

    def device_part(self, k: int, pipeline: int = 0) -> Tuple[int, int]:
        if self.scheme == V_1F1B:
            return k, 0
        if self.scheme == W_INTERLEAVE:
            return k % self.S, k // self.S
        return (k, 0) if pipeline == 0 else (self.S - 1 - k, 1)


def find_inst(pipe: Pipe, d: int, m: int, p: int, t: str, nxt: bool) -> Optional[Tuple[int, int, int, str]]:
    """Algorithm 1: FIND_[PREV|NEXT]_INST(d, m, p, t).
    step = -1 for find_prev, +1 for find_next in the logical direction of FW; the
    direction is opposite for BW (reading A11). Returns (d_o, m_o, p_o, t_o) or
    None when the target lies outside the virtual pipeline."""
    step = 1 if nxt else -1
    if t == BW:
        step = -step
    d_o, m_o, p_o, t_o = d, m, p, t
    if pipe.scheme == V_1F1B:
        d_o = d + step
        if not 0 <= d_o < pipe.S:
            return None
    elif pipe.scheme == X_CHIMERA:
        d_o = d + step if p == 0 else d - step
        if not 0 <= d_o < pipe.S:
            return None
    else:  # Interleave: modular wrap with part_id change (reading A9: p_o = p + step)
        d_o = (d + step + pipe.S) % pipe.S
        if d_o != d + step:
            p_o = p + step
        if not 0 <= p_o < pipe.v:
            return None
    return d_o, m_o, p_o, t_o


# ----------------------------------------------------------------------- base schedules
def _fw_group(pipe, d, m, p):
    k = pipe.vstage(d, p)
    g = []
    if k > 0:
        g.append((RA, m, p))
    g.append((FW, m, p))
    if k < pipe.K - 1:
        g.append((SA, m, p))
    return g


def _bw_group(pipe, d, m, p):
    k = pipe.vstage(d, p)
    g = []
    if k < pipe.K - 1:
        g.append((RG, m, p))
    g.append((BW, m, p))
    if k > 0:
        g.append((SG, m, p))
    return g


def build_1f1b(pipe: Pipe) -> List[List[Instr]]:
    """1F1B (Megatron-DeepSpeed order): warm-up S-d-1 forwards, steady 1F1B, cool-down."""
    S, N = pipe.S, pipe.N
    lists = []
    for d in range(S):
        warm = min(S - d - 1, N)
        L: List[Instr] = []
        for i in range(warm):
            L += _fw_group(pipe, d, i, 0)
        for i in range(N - warm):
            L += _fw_group(pipe, d, warm + i, 0)
            L += _bw_group(pipe, d, i, 0)
        for i in range(N - warm, N):
            L += _bw_group(pipe, d, i, 0)
        lists.append(L)
    return lists


def build_interleave(pipe: Pipe) -> List[List[Instr]]:
    """Interleave (Megatron-LM schedules.py order; reading A9)."""
    S, N, v = pipe.S, pipe.N, pipe.v
    total = N * v

    def chunk(k, forward):
        c = (k % (S * v)) // S
        return c if forward else v - 1 - c

    def micro(k):
        return (k // (S * v)) * S + k % S

    lists = []
    for d in range(S):
        if N == S:
            warm = total
        else:
            warm = min((S - d - 1) * 2 + (v - 1) * S, total)
        L: List[Instr] = []
        for k in range(warm):
            L += _fw_group(pipe, d, micro(k), chunk(k, True))
        for i in range(total - warm):
            kf = warm + i
            L += _fw_group(pipe, d, micro(kf), chunk(kf, True))
            L += _bw_group(pipe, d, micro(i), chunk(i, False))
        for kb in range(total - warm, total):
            L += _bw_group(pipe, d, micro(kb), chunk(kb, False))
        lists.append(L)
    return lists


def build_chimera(pipe: Pipe, F: float = 1.0, B: float = 2.0) -> List[List[Instr]]:
    """Chimera (reading A10): one basic unit of D micro-batches (first D/2 on the down
    pipeline p=0, last D/2 on the up pipeline p=1) is ordered by a greedy list schedule
    at unit costs F=1, B=2: whenever a worker is idle it runs the ready instruction with
    priority BW before FW, then the deeper virtual stage (higher k) first, ties by micro id.
    Units are concatenated for N > D. Pinned against Chimera's own closed form ([23], cited at
    P:61 / Table 1): built and simulated at F = B the basic unit takes 2N + D - 2 (D - 2
    bubbles per worker) for N = D (tests/test_schedule_oracle.py::test_chimera_unit_closed_form)."""
    D, N = pipe.S, pipe.N
    unit = Pipe(X_CHIMERA, D, D)
    # tasks per worker
    fin: Dict[Tuple[str, int, int], float] = {}
    order: List[List[Tuple[str, int, int]]] = [[] for _ in range(D)]
    # each (op, m, k) is owned by device device_part(k, pipeline)
    def owner(m, k):
        return unit.device_part(k, unit.part_of_micro(m))[0]

    busy_until = [0.0] * D
    t = 0.0
    remaining = {(op, m, k) for m in range(D) for k in range(D) for op in (FW, BW)}
    while remaining:
        progressed = False
        for d in range(D):
            if busy_until[d] > t + 1e-12:
                continue
            ready = []
            for (op, m, k) in remaining:
                if owner(m, k) != d:
                    continue
                if op == FW:
                    dep = None if k == 0 else (FW, m, k - 1)
                else:
                    dep = (FW, m, k) if k == D - 1 else (BW, m, k + 1)
                    if (FW, m, k) not in fin or fin[(FW, m, k)] > t + 1e-12:
                        continue
                if dep is not None and (dep not in fin or fin[dep] > t + 1e-12):
                    continue
                ready.append((0 if op == BW else 1, -k, m, op))
            if not ready:
                continue
            ready.sort()
            _, nk, m, op = ready[0]
            k = -nk
            remaining.discard((op, m, k))
            dur = F if op == FW else B
            fin[(op, m, k)] = t + dur
            busy_until[d] = t + dur
            order[d].append((op, m, unit.part_of_micro(m)))
            progressed = True
        # advance time to the next event
        future = [f for f in list(busy_until) + list(fin.values()) if f > t + 1e-12]
        if not future:
            if not progressed and remaining:
                raise RuntimeError("chimera greedy stalled")
            continue
        t = min(future)
    lists = []
    for d in range(D):
        L: List[Instr] = []
        for u in range(N // D):
            for op, m, p in order[d]:
                mm = u * D + m
                if op == FW:
                    L += _fw_group(pipe, d, mm, p)
                else:
                    L += _bw_group(pipe, d, mm, p)
        lists.append(L)
    return lists


def build_base(pipe: Pipe) -> List[List[Instr]]:
    if pipe.scheme == V_1F1B:
        return build_1f1b(pipe)
    if pipe.scheme == W_INTERLEAVE:
        return build_interleave(pipe)
    return build_chimera(pipe)


# ------------------------------------------------------------------------------ passes
def pass1_apply_checkpoint(lists, keep=()):
    """every FW_i -> CFW_i; RC_i inserted right before BW_i (after RG_i: the naive
    placement of Fig. 2 step 1, reading A14). Devices in `keep` stay un-checkpointed in their
    base order (the budget-driven extension, reading A28; empty for the paper's passes)."""
    out = []
    for d, L in enumerate(lists):
        if d in keep:
            out.append(list(L))
            continue
        N = []
        for (op, m, p) in L:
            if op == FW:
                N.append((CFW, m, p))
            elif op == BW:
                N.append((RC, m, p))
                N.append((BW, m, p))
            else:
                N.append((op, m, p))
        out.append(N)
    return out


def pass2_overlap_recompute(lists):
    """RC_i placed immediately before RG_i (reading A15)."""
    out = []
    for L in lists:
        N = [x for x in L if x[0] != RC]
        rcs = [x for x in L if x[0] == RC]
        for (op, m, p) in rcs:
            anchor = N.index((RG, m, p)) if (RG, m, p) in N else N.index((BW, m, p))
            N.insert(anchor, (RC, m, p))
        out.append(N)
    return out


def pass3_remove_redundancy(lists):
    """when CFW_i and BW_i are adjacent (ignoring comm instructions and RC_i itself,
    reading A16) the checkpoint is redundant: CFW_i -> FW_i and RC_i is dropped."""
    out = []
    for L in lists:
        N = list(L)
        for (op, m, p) in L:
            if op != CFW:
                continue
            i, j = N.index((CFW, m, p)), N.index((BW, m, p))
            between = [x for x in N[i + 1:j] if x[0] in COMPUTE and x != (RC, m, p)]
            if not between:
                N[i] = (FW, m, p)
                N.remove((RC, m, p))
        out.append(N)
    return out


def _group_starts(L):
    """Indices where a new group (leading receives + one compute + trailing sends) may
    be inserted: before a compute or a receive that is not preceded by a receive."""
    out = []
    for j, x in enumerate(L):
        if x[0] in COMPUTE or x[0] in RECV:
            if j > 0 and L[j - 1][0] in RECV:
                continue
            out.append(j)
    out.append(len(L))
    return out


def pass4_prepose_forward(pipe, lists, costs, mem=None, budget=None, max_rounds=8):
    """prepose each CFW_i (with its RA_i) into the earliest bubble after the
    previous forward on its device, devices in ascending order, micro-batches in list
    order (reading A17). A move is accepted at the earliest position that keeps the graph
    acyclic, does not raise the simulated makespan and keeps the peak within the budget.
    SA rule: the sender's SA_i moves up to its CFW_i only when the receiver's
    CFW_i is preposed; otherwise it stays in place and the output is buffered.
    Applied iteratively to a fixpoint."""
    lists = [list(L) for L in lists]
    preposed = set()
    cur = simulate(pipe, lists, costs)
    assert cur is not None, "input lists deadlock"
    best = cur.makespan
    for _ in range(max_rounds):
        changed = False
        for d in range(pipe.S):
            for x in [y for y in lists[d] if y[0] == CFW]:
                _, m, p = x
                L = lists[d]
                i = L.index(x)
                # previous forward on this device
                prev_f = max([j for j in range(i) if L[j][0] in (FW, CFW)], default=-1)
                lo = prev_f + 1
                # start of this CFW's group (its RA)
                gstart = i - 1 if i > 0 and L[i - 1] == (RA, m, p) else i
                cands = [j for j in _group_starts(L) if lo <= j < gstart]
                for j in cands:
                    trial = [list(T) for T in lists]
                    grp = L[gstart:i + 1]
                    rest = L[:gstart] + L[i + 1:]
                    trial[d] = rest[:j] + grp + rest[j:]   # j < gstart: index unchanged
                    # SA rule: the sender's SA_m follows its CFW_m if that CFW was preposed
                    prv = find_inst(pipe, d, m, p, FW, nxt=False)
                    if prv is not None:
                        sd, _, sp, _ = prv
                        if (sd, CFW, m, sp) in preposed:
                            SL = trial[sd]
                            SL.remove((SA, m, sp))
                            SL.insert(SL.index((CFW, m, sp)) + 1, (SA, m, sp))
                    r = simulate(pipe, trial, costs)
                    if r is None or r.makespan > best + 1e-9:
                        continue
                    if budget is not None and mem is not None:
                        if max(memory_walk(pipe, trial, mem).peak) > budget:
                            continue
                    lists = trial
                    best = r.makespan
                    preposed.add((d, CFW, m, p))
                    changed = True
                    break
        if not changed:
            break
    return lists


def transform(pipe: Pipe, level: str, costs=None, mem=None, budget=None, keep=()):
    """BASE: base lists. CKPT: pass 1 only (naive full-checkpoint, A14). MARIO: passes 1-4.
    MARIO_BUDGET: passes 1-4 with the tail devices chosen by pass5_budget left un-checkpointed.
    `keep`: devices passes 1-4 leave in their base order (used by pass5_budget)."""
    if level == MARIO_BUDGET:
        return pass5_budget(pipe, costs or UnitCosts(), mem, budget)[0]
    lists = build_base(pipe)
    if level == BASE:
        return lists
    lists = pass1_apply_checkpoint(lists, keep)
    if level == CKPT:
        return lists
    lists = pass2_overlap_recompute(lists)
    lists = pass3_remove_redundancy(lists)
    costs = costs or UnitCosts()
    return pass4_prepose_forward(pipe, lists, costs, mem, budget)


def pass5_budget(pipe: Pipe, costs, mem, budget):
    """Budget-driven partial checkpointing (reading A28): Pass 3 un-checkpoints
    a stage only when CFW_i and BW_i are adjacent; with memory to spare (mem_budget)
    the tail devices d >= S - k can keep their full activations in their 1F1B order (device d then
    holds its base in-flight count of activation sets, Table 1) while devices < S - k go through
    passes 1-4. For k = 0 .. S: lists_k = transform(MARIO, keep = tail k); feasible iff the peak
    of every device is within the budget; pick the smallest makespan, ties to the smaller k.
    Returns (lists, k)."""
    assert mem is not None and budget is not None, "MARIO_BUDGET needs mem and budget"
    best = None
    for k in range(pipe.S + 1):
        keep = set(range(pipe.S - k, pipe.S))
        L = transform(pipe, MARIO, costs, mem, budget, keep=keep)
        if max(memory_walk(pipe, L, mem).peak) > budget:
            continue
        r = simulate(pipe, L, costs)
        if r is None:
            continue
        if best is None or r.makespan < best[0] - 1e-9:
            best = (r.makespan, L, k)
    if best is None:   # nothing fits: the paper's passes (the caller reports EBUDGET)
        return transform(pipe, MARIO, costs, mem, budget), 0
    return best[1], best[2]


# ---------------------------------------------------------------------------- simulator
@dataclass
class UnitCosts:
    """Per-virtual-stage costs. Defaults: F = t = 1, B = 2t, RC = F, comm 0."""
    F: float = 1.0
    B: float = 2.0
    R: float = 1.0
    comm: float = 0.0
    per_stage: Optional[Dict[int, Tuple[float, float, float]]] = None

    def fw(self, k):
        return self.per_stage[k][0] if self.per_stage and k in self.per_stage else self.F

    def bw(self, k):
        return self.per_stage[k][1] if self.per_stage and k in self.per_stage else self.B

    def rc(self, k):
        return self.per_stage[k][2] if self.per_stage and k in self.per_stage else self.R


@dataclass
class SimResult:
    makespan: float
    start: Dict[Tuple[int, str, int, int], float]
    finish: Dict[Tuple[int, str, int, int], float]
    busy: List[float]


def simulate(pipe: Pipe, lists, costs: UnitCosts) -> Optional[SimResult]:
    """Dynamic-programming timeline, reading A12.

    Each device walks its list in order. Compute instructions (FW/CFW/RC/BW) run serially
    (horizontal dependency). A receive RA_m/RG_m BLOCKS the device's stream until the data
    has arrived — "if RC_i is placed after RG_i, it must wait for RG_i to finish".
    A send SA_m/SG_m is buffered (does not block): it is posted when everything before it
    in its list has completed, and its data arrives `comm` later at the receiver found by
    Algorithm 1 (vertical dependency). Returns None on a dependency cycle (deadlock)."""
    S = pipe.S
    finish: Dict = {}
    start: Dict = {}
    post: Dict = {}
    ptr = [0] * S
    dev_t = [0.0] * S
    busy = [0.0] * S
    total = sum(len(L) for L in lists)
    n_done = 0
    while n_done < total:
        progressed = False
        for d in range(S):
            L = lists[d]
            while ptr[d] < len(L):
                op, m, p = L[ptr[d]]
                k = pipe.vstage(d, p)
                if op in SEND:
                    post[(d, op, m, p)] = dev_t[d]
                elif op in RECV:
                    src = find_inst(pipe, d, m, p, FW if op == RA else BW, nxt=False)
                    key = (src[0], SA if op == RA else SG, m, src[2])
                    if key not in post:
                        break
                    dev_t[d] = max(dev_t[d], post[key] + costs.comm)
                else:
                    dur = costs.fw(k) if op in (FW, CFW) else costs.rc(k) if op == RC else costs.bw(k)
                    start[(d, op, m, p)] = dev_t[d]
                    finish[(d, op, m, p)] = dev_t[d] + dur
                    dev_t[d] += dur
                    busy[d] += dur
                ptr[d] += 1
                n_done += 1
                progressed = True
        if not progressed:
            return None
    return SimResult(max(finish.values()), start, finish, busy)


# ------------------------------------------------------------------------------- memory
@dataclass
class MemUnits:
    """Per-virtual-stage byte counts (reading A13). Defaults count units: one activation
    set = 1, checkpoints = 0 (so peak == max live activation sets, Table 1)."""
    act: float = 1.0
    ckpt: float = 0.0
    work: float = 0.0


@dataclass
class MemResult:
    peak: List[float]
    max_live_act: List[int]
    max_live_ckpt: List[int]


def memory_walk(pipe: Pipe, lists, mem: MemUnits) -> MemResult:
    """static + dynamic; a CFW's dynamic memory is transient; an FW's activation
    set lives until its BW; RC materialises the set again until BW."""
    peaks, acts, ckpts = [], [], []
    for d, L in enumerate(lists):
        cur = 0.0
        peak = 0.0
        live_act = live_ck = 0
        ma = mc = 0
        for op, m, p in L:
            if op == FW:
                live_ck += 1
                live_act += 1
                cur += mem.act + mem.ckpt
                peak = max(peak, cur)
            elif op == CFW:
                live_ck += 1
                cur += mem.ckpt
                peak = max(peak, cur + mem.work)
            elif op == RC:
                live_act += 1
                cur += mem.act
                peak = max(peak, cur)
            elif op == BW:
                live_act -= 1
                live_ck -= 1
                cur -= mem.act + mem.ckpt
            ma, mc = max(ma, live_act), max(mc, live_ck)
        peaks.append(peak)
        acts.append(ma)
        ckpts.append(mc)
    return MemResult(peaks, acts, ckpts)


# ------------------------------------------------------------------------- invariants
def check_structure(pipe: Pipe, lists) -> None:
    """Structural invariants; raises AssertionError."""
    seen = {}
    for d, L in enumerate(lists):
        for x in L:
            assert x not in seen.get(d, set()), ("duplicate", d, x)
            seen.setdefault(d, set()).add(x)
    for m in range(pipe.N):
        pl = pipe.part_of_micro(m)
        for k in range(pipe.K):
            d, p = pipe.device_part(k, pl)
            L = lists[d]
            f = [x for x in L if x[1] == m and x[2] == p and x[0] in (FW, CFW)]
            b = [x for x in L if x[1] == m and x[2] == p and x[0] == BW]
            assert len(f) == 1 and len(b) == 1, (d, m, p, f, b)
            rc = (RC, m, p) in L
            assert rc == (f[0][0] == CFW), (d, m, p)
            if rc:
                assert L.index(f[0]) < L.index((RC, m, p)) < L.index(b[0])
    # channel pairing: SA/RA and SG/RG 1:1 per channel in equal order
    for d, L in enumerate(lists):
        for op, m, p in L:
            if op == SA:
                nx = find_inst(pipe, d, m, p, FW, nxt=True)
                assert nx is not None and (RA, m, nx[2]) in lists[nx[0]]
            if op == SG:
                nx = find_inst(pipe, d, m, p, BW, nxt=True)
                assert nx is not None and (RG, m, nx[2]) in lists[nx[0]]
