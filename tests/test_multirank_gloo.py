"""N > 1 host logic on CPU (gloo, world_size 2 and 4): every rank executes its communication
program from mario_plan_comm_ops exactly as the executor issues it (blocking receive at the RA/RG
position, buffered send after the instruction the program names) with gloo p2p standing in for the
per-channel NCCL communicators (one tag per channel = one FIFO). Checks: every receive gets the
message of the micro-batch/stage it expects (FIFO order is right, also after pass 4), no deadlock,
and the collective splits / pair all-reduces are issued in the same order on all ranks."""
import datetime
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth
from paper_conf_ppopp_liultj25_b200 import api

CASES = [("1f1b", 2, 4, 1, "mario"), ("1f1b", 4, 8, 1, "mario"), ("1f1b", 4, 8, 1, "base"),
         ("interleave", 2, 4, 2, "mario"), ("interleave", 4, 8, 2, "mario"), ("chimera", 4, 8, 1, "mario"),
         ("chimera", 2, 4, 1, "ckpt")]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _plan(scheme, S, N, v, level):
    K = S * v
    cfg = synth.with_(synth.TINY_GPT, n_layers=2 * K)
    return api.Plan(cfg, S, N, scheme, level, chunks=v, dtype="f32")


def _worker(rank, world, port, case, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world, timeout=datetime.timedelta(seconds=60))
        plan = _plan(*case)
        ops = plan.comm_ops(rank)
        instrs = plan.instrs(rank)
        collectives = [(k, a, b, c, cnt) for (k, a, b, c, m, p, li, cnt) in ops if k in (0, 1, 4, 5)]
        handles = []
        n_recv = 0
        for (k, a, b, c, m, p, li, cnt) in ops:
            tag = 1 + 2 * (a * world + b) + c
            if k == 2:   # send: payload = (micro, sender vstage)
                ks = [x for x in plan.instrs(rank) if x[1] == m and x[2] == p][0][3]
                handles.append(dist.isend(torch.tensor([m, ks], dtype=torch.int64), dst=b, tag=tag))
            elif k == 3:  # blocking receive at the RA/RG position
                buf = torch.zeros(2, dtype=torch.int64)
                dist.recv(buf, src=a, tag=tag)
                op, mm, pp, kr = instrs[li][0], instrs[li][1], instrs[li][2], instrs[li][3]
                assert op in ("RA", "RG") and mm == m and pp == p
                assert int(buf[0]) == m, (rank, "got micro", int(buf[0]), "expected", m)
                assert int(buf[1]) == (kr - 1 if op == "RA" else kr + 1)
                n_recv += 1
            elif k == 5:
                t = torch.ones(cnt, dtype=torch.float64)
                dist.all_reduce(t)
                assert float(t[0]) == world
        for h in handles:
            h.wait()
        gathered = [None] * world
        dist.all_gather_object(gathered, collectives)
        splits = [[x for x in g if x[0] in (0, 1, 5)] for g in gathered]
        assert all(s == splits[0] for s in splits), "collective split order differs across ranks"
        for r in range(world):   # pair all-reduces: both members issue the same sequence
            for r2 in range(world):
                a = [x for x in gathered[r] if x[0] == 4 and {x[2], x[3]} == {r, r2}]
                b = [x for x in gathered[r2] if x[0] == 4 and {x[2], x[3]} == {r, r2}]
                if r != r2:
                    assert a == b
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, "ok", n_recv))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, f"fail: {e!r}", 0))


@pytest.mark.parametrize("case", CASES, ids=["-".join(map(str, c)) for c in CASES])
def test_comm_program_gloo(case):
    world = case[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(r[1] == "ok" for r in res), res
    assert sum(r[2] for r in res) > 0


def test_pass4_can_reorder_sends_and_program_restores_fifo():
    """Document why the program reorders: in some Mario plan a sender's SA order differs from the
    receiver's RA order on a channel; the program's send order always equals the RA order."""
    for case in CASES:
        plan = _plan(*case)
        S = case[1]
        for r in range(S):
            sends = {}
            for (k, a, b, c, m, p, li, cnt) in plan.comm_ops(r):
                if k == 2:
                    sends.setdefault((b, c), []).append(m)
            for (b, c), ms in sends.items():
                recv = [x[1] for x in plan.instrs(b) if x[0] == ("RA" if c == 0 else "RG") and x[4] == r]
                assert ms == recv


# ------------------------------------------------------------- PP x DP (f3, reading A29)
DP_CASES = [("1f1b", 2, 4, 1, "mario"), ("chimera", 2, 4, 1, "mario"), ("interleave", 2, 4, 2, "mario"),
            ("1f1b", 1, 4, 1, "mario")]


def _worker_dp(rank, world, dp, port, case, q):
    """World rank = replica * S + stage executes mario_plan_comm_ops_dp exactly like the executor:
    p2p stays inside the replica, splits are issued by every rank in the same order, kind 7
    averages over the stage's replicas."""
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world, timeout=datetime.timedelta(seconds=60))
        plan = _plan(*case)
        S = case[1]
        stage, rep, off = rank % S, rank // S, (rank // S) * S
        ops = plan.comm_ops_dp(rank, dp)
        instrs = plan.instrs(stage)
        assert [o for o in ops if o[0] not in (6, 7)] == [
            (k, a + off if k in (0, 1, 2, 3) else a, b + off if k in (0, 1, 2, 3, 4) else b,
             c + off if k == 4 else c, m, p, li, cnt) for (k, a, b, c, m, p, li, cnt) in plan.comm_ops(stage)]
        seq, handles, groups, n_recv, got_avg = [], [], {}, 0, None
        for (k, a, b, c, m, p, li, cnt) in ops:
            tag = 1 + 2 * (a * world + b) + c
            if k in (0, 1):
                assert rank in range(off, off + S) and a in range(off, off + S) and b in range(off, off + S)
                seq.append((k, a - off, b - off, c))
            elif k == 6:
                assert (a, b, c) == (stage, rep, dp)
                for st in range(S):   # every rank creates every stage's group, same order
                    groups[st] = dist.new_group([st + r * S for r in range(dp)])
                seq.append((6, dp))
            elif k == 2:
                ks = [x for x in instrs if x[1] == m and x[2] == p][0][3]
                handles.append(dist.isend(torch.tensor([m, ks, rep], dtype=torch.int64), dst=b, tag=tag))
            elif k == 3:
                buf = torch.zeros(3, dtype=torch.int64)
                dist.recv(buf, src=a, tag=tag)
                op, mm, kr = instrs[li][0], instrs[li][1], instrs[li][3]
                assert mm == m and int(buf[0]) == m and int(buf[2]) == rep
                assert int(buf[1]) == (kr - 1 if op == "RA" else kr + 1)
                n_recv += 1
            elif k == 7:
                assert cnt == plan.rank_layout(stage)[0] and (a, b, c) == (stage, rep, dp)
                t = torch.tensor([float(rep)], dtype=torch.float64)
                dist.all_reduce(t, group=groups[stage])
                got_avg = float(t[0]) / dp
            elif k == 5:
                assert got_avg is not None or dp == 1, "gradient AR must precede the loss all-reduce"
                t = torch.ones(cnt, dtype=torch.float64)
                dist.all_reduce(t)
                assert float(t[0]) == world
                seq.append((5, cnt))
        for h in handles:
            h.wait()
        assert got_avg == (dp - 1) / 2
        gathered = [None] * world
        dist.all_gather_object(gathered, seq)
        assert all(g == gathered[0] for g in gathered), "split / collective order differs across ranks"
        dist.barrier()
        dist.destroy_process_group()
        q.put((rank, "ok", n_recv))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, f"fail: {e!r}", 0))


@pytest.mark.parametrize("case", DP_CASES, ids=["-".join(map(str, c)) for c in DP_CASES])
def test_pp_x_dp_comm_program_gloo(case):
    dp = 2
    world = case[1] * dp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_dp, args=(r, world, dp, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(r[1] == "ok" for r in res), res
    assert case[1] == 1 or sum(r[2] for r in res) > 0


def test_comm_ops_dp_rejects_bad_rank():
    plan = _plan("1f1b", 2, 4, 1, "mario")
    with pytest.raises(api.MarioError):
        plan.comm_ops_dp(4, 2)
    assert plan.comm_ops_dp(1, 1) == plan.comm_ops(1)
