"""Multi-process peer transport (mario_init_peer): one OS process per pipeline rank, all on cuda:0,
exchanging activations and gradients through CUDA IPC mappings of each other's workspace (the
executor's multi-process code path: every rank walks only its own list; receives wait on the
sender's flag, copy out of its send slot and raise "consumed"; send slots are reused after
"consumed"; tied / replica gradient copies are summed by a reduce-scatter + all-gather over the
mapped grads; an end-of-iteration barrier). The grads of every rank must equal the loopback
executor's bit for bit, on two consecutive iterations (epoch-valued flags)."""
import multiprocessing as mp
import os
import socket
import tempfile

import numpy as np
import pytest
import torch

import synth
from paper_conf_ppopp_liultj25_b200 import api

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(600, method="thread")]

CASES = {
    "1f1b-s2": (synth.with_(synth.TINY_GPT, n_layers=4), "1f1b", 2, 4, 1, "mario", "f32"),
    "1f1b-s4-bf16": (synth.with_(synth.tiny_llama(), n_layers=4), "1f1b", 4, 8, 1, "mario", "bf16"),
    "interleave-s2": (synth.with_(synth.TINY_GPT, n_layers=4), "interleave", 2, 4, 2, "mario", "f32"),
    "chimera-s4": (synth.with_(synth.TINY_GPT, n_layers=4), "chimera", 4, 8, 1, "mario", "bf16"),
    "1f1b-s4-ckpt": (synth.with_(synth.TINY_GPT, n_layers=4), "1f1b", 4, 8, 1, "ckpt", "f32"),
}


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, name, out_dir):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    cfg, scheme, S, N, v, level, dtype = CASES[name]
    plan = api.Plan(cfg, S, N, scheme, level, chunks=v, dtype=dtype)
    ctx = api.Context.peer(rank, world, 0)
    try:
        pc, wsb = plan.rank_layout(rank)
        w = torch.from_numpy(api.pack_params(plan, synth.make_weights(cfg), rank)).cuda()
        g = torch.zeros(pc, dtype=torch.float32, device="cuda")
        ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
        ctx.bind(ws, g)
        for it in range(2):
            loss = ctx.run_iter(plan, w, synth.make_tokens(cfg, N, iteration=it), g, ws)
            torch.cuda.synchronize()
            np.save(os.path.join(out_dir, f"g{rank}_{it}.npy"), g.cpu().numpy())
            np.save(os.path.join(out_dir, f"l{rank}_{it}.npy"), np.array([loss], np.float32))
    finally:
        ctx.close()
        dist.destroy_process_group()


@pytest.mark.parametrize("name", sorted(CASES))
def test_peer_ipc_processes_bitwise_equal_loopback(name):
    cfg, scheme, S, N, v, level, dtype = CASES[name]
    params = synth.make_weights(cfg)
    with tempfile.TemporaryDirectory() as out_dir:
        ctxm = mp.get_context("spawn")
        port = _free_port()
        procs = [ctxm.Process(target=_worker, args=(r, S, port, name, out_dir)) for r in range(S)]
        for p in procs:
            p.start()
        for p in procs:
            p.join(timeout=400)
        alive = [p for p in procs if p.is_alive()]
        for p in alive:
            p.kill()
        assert not alive, "a peer rank hung"
        assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]
        plan = api.Plan(cfg, S, N, scheme, level, chunks=v, dtype=dtype)
        ctx = api.default_context()
        w, g, ws = api.alloc_for(plan, -1)
        w.copy_(torch.from_numpy(api.pack_params(plan, params, -1)))
        for it in range(2):
            loss = ctx.run_iter(plan, w, synth.make_tokens(cfg, N, iteration=it), g, ws)
            ref = g.cpu().numpy()
            base = 0
            for r in range(S):
                n = plan.rank_layout(r)[0]
                got = np.load(os.path.join(out_dir, f"g{r}_{it}.npy"))
                assert np.array_equal(got, ref[base:base + n]), (r, it)
                assert float(np.load(os.path.join(out_dir, f"l{r}_{it}.npy"))[0]) == np.float32(loss), (r, it)
                base += n
