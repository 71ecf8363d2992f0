"""ORACLE (test infrastructure only) — CPU replay of a plan's per-device instruction lists.

SURVEY §8(c) c4 "Pipelining (2)": execute every device's list (Table 3 IR) with the
instruction semantics the paper gives, on the CPU, with the layer maths of `oracle.model`:

- FW_i: forward of micro-batch i through the device's virtual stage; keeps every
  activation its BW needs.
- CFW_i (§3 "stage-level checkpointing"): the same forward, but only the stage input (the
  checkpoint) is kept; the activations are dropped.
- RC_i: replays the forward of micro-batch i from the kept checkpoint and
  materialises the activations again; it records no loss (the loss belongs to the CFW/FW).
- BW_i: backward from the received output gradient (or the loss on the last virtual stage);
  accumulates the parameter gradients of the device's copy and frees the activations.
- SA/RA, SG/RG: activations / gradients cross a virtual-stage boundary; a receive
  waits until the matching send was posted (blocking receive); sends are buffered.

Devices advance round-robin; a receive whose message was not posted yet stalls its device.
No progress in a whole sweep = a cycle (the paper's deadlock) -> RuntimeError.
Using an instruction out of its semantics (BW without activations, RC without checkpoint,
RC after FW, a missing message) raises AssertionError.

Gradients accumulate per parameter COPY: device d's part p holds the parameters of virtual
stage vstage(d, p) (embedding on virtual stage 0, final norm + head on the last; a tied GPT
head keeps its own `wte` copy on the last stage, reading A8; Chimera keeps a down and an up
replica). Copies are summed at the end in (device, part) order (reading A7). Since FW, CFW
and RC run the same `oracle.model` functions on the same inputs, the replay reproduces
`oracle.model.step` exactly whenever a parameter's contributions arrive in the same micro-batch
order (tests/test_replay_oracle.py).
"""
from __future__ import annotations

from typing import Dict, List, Tuple

import numpy as np

from . import model as om
from .schedule import BW, CFW, FW, RA, RC, RG, SA, SG, X_CHIMERA, Pipe


def stage_param_names(cfg, pipe: Pipe, k: int) -> List[str]:
    """Parameters held by virtual stage k (reading A8): its layers (even split), the embedding on
    virtual stage 0, the final norm + head on the last (GPT tied: its own wte copy)."""
    K = pipe.K
    assert cfg.n_layers % K == 0, "L % (S*v) != 0"
    lps = cfg.n_layers // K
    names = []
    if k == 0:
        names += ["wte", "wpe"] if cfg.family == "gpt" else ["emb"]
    from synth import layer_param_shapes   # names only (no method arithmetic)
    for l in range(k * lps, (k + 1) * lps):
        names += [n for n, _ in layer_param_shapes(cfg, l)]
    if k == K - 1:
        if cfg.family == "gpt":
            names += ["lnf.g", "lnf.b"]
            names += ["wte"] if cfg.tie_embeddings else ["head.w"]
        else:
            names += ["nf.g", "out.w"]
    return list(dict.fromkeys(names))


def replay(cfg, params: Dict[str, np.ndarray], tokens: np.ndarray, pipe: Pipe, lists, dtype=np.float32
           ) -> Tuple[float, Dict[str, np.ndarray], Dict[Tuple[int, int], Dict[str, np.ndarray]]]:
    """Execute `lists` (per device: [(op, micro, part)]). Returns (loss, grads summed over copies,
    per-copy grads {(device, part): {name: grad}})."""
    P = {k: np.asarray(v).astype(dtype) for k, v in params.items()}
    mbs, s, K, N = cfg.micro_batch, cfg.seq_len, pipe.K, pipe.N
    assert tokens.shape == (N * mbs, s + 1)
    lps = cfg.n_layers // K
    n_tok = N * mbs * s
    rope = om.rope_tables(s, cfg.head_dim, cfg.rope_base, dtype) if cfg.family == "llama" else None
    hname = "wte" if (cfg.family == "gpt" and cfg.tie_embeddings) else ("head.w" if cfg.family == "gpt" else "out.w")
    ename = "wte" if cfg.family == "gpt" else "emb"

    parts = 2 if pipe.scheme == X_CHIMERA else pipe.v
    G = {(d, p): {n: np.zeros_like(P[n]) for n in stage_param_names(cfg, pipe, pipe.vstage(d, p))}
         for d in range(pipe.S) for p in range(parts)}
    mailbox: Dict[Tuple[str, int, int], np.ndarray] = {}   # (kind, micro, receiving vstage) -> tensor
    ckpt: Dict[Tuple[int, int, int], np.ndarray] = {}      # (d, m, p) -> stage input
    acts: Dict[Tuple[int, int, int], dict] = {}            # (d, m, p) -> what BW needs
    out: Dict[Tuple[int, int, int], np.ndarray] = {}       # (d, m, p) -> stage output awaiting SA
    dinp: Dict[Tuple[int, int, int], np.ndarray] = {}      # (d, m, p) -> input gradient awaiting SG
    recv_act: Dict[Tuple[int, int, int], np.ndarray] = {}  # (d, m, p) -> received activation
    recv_grad: Dict[Tuple[int, int, int], np.ndarray] = {}
    loss_sum: Dict[int, float] = {}

    def xy(m):
        blk = tokens[m * mbs:(m + 1) * mbs]
        return blk[:, :s], blk[:, 1:]

    def forward(d, m, p, k, H_in, keep):
        """Stage forward of virtual stage k; returns (output or None on the last stage, caches)."""
        x, y = xy(m)
        H = om.embed_fwd(cfg, P, x) if k == 0 else H_in
        caches = []
        for l in range(k * lps, (k + 1) * lps):
            H, c = om.layer_fwd(cfg, P, l, H, rope)
            caches.append(c)
        st = {"caches": caches} if keep else None
        if k == K - 1:
            Hf, ncache, logits = om.head_fwd(cfg, P, H)
            tok_loss, probs = om.cross_entropy(logits, y)
            if keep:
                st.update(Hf=Hf, ncache=ncache, probs=probs, y=y)
            return None, st, tok_loss.sum(dtype=np.float64)
        return H, st, None

    def backward(d, m, p, k, dout):
        st = acts.pop((d, m, p))
        Gc = G[(d, p)]
        if k == K - 1:
            probs, y = st["probs"], st["y"]
            onehot = np.zeros_like(probs)
            np.put_along_axis(onehot, y[..., None], 1.0, axis=-1)
            dlogits = (probs - onehot) / n_tok
            Gc[hname] += om._wgrad(dlogits, st["Hf"])
            dHf = np.matmul(dlogits, om.head_weight(cfg, P))
            if cfg.family == "gpt":
                dH, dg, db = om.layernorm_bwd(dHf, st["ncache"], P["lnf.g"])
                Gc["lnf.g"] += dg
                Gc["lnf.b"] += db
            else:
                dH, dg = om.rmsnorm_bwd(dHf, st["ncache"], P["nf.g"])
                Gc["nf.g"] += dg
        else:
            dH = dout
        for i, l in reversed(list(enumerate(range(k * lps, (k + 1) * lps)))):
            dH = om.layer_bwd(cfg, P, l, dH, st["caches"][i], rope, Gc)
        if k == 0:
            x, _ = xy(m)
            np.add.at(Gc[ename], x.reshape(-1), dH.reshape(-1, cfg.hidden))
            if cfg.family == "gpt":
                Gc["wpe"][:s] += dH.sum(axis=0)
            return None
        return dH

    ptr = [0] * pipe.S
    total = sum(len(L) for L in lists)
    done = 0
    while done < total:
        progressed = False
        for d in range(pipe.S):
            L = lists[d]
            while ptr[d] < len(L):
                op, m, p = L[ptr[d]]
                k = pipe.vstage(d, p)
                key = (d, m, p)
                if op == RA:
                    if ("act", m, k) not in mailbox:
                        break
                    recv_act[key] = mailbox.pop(("act", m, k))
                elif op == RG:
                    if ("grad", m, k) not in mailbox:
                        break
                    recv_grad[key] = mailbox.pop(("grad", m, k))
                elif op in (FW, CFW):
                    assert key not in ckpt and key not in acts, ("forward twice", d, op, m, p)
                    H_in = None if k == 0 else recv_act.pop(key)
                    o, st, ls = forward(d, m, p, k, H_in, keep=op == FW)
                    ckpt[key] = H_in          # stage-level checkpoint (None on stage 0: the tokens)
                    if op == FW:
                        acts[key] = st
                    if ls is not None:
                        assert m not in loss_sum
                        loss_sum[m] = float(ls)
                    if o is not None:
                        out[key] = o
                elif op == RC:
                    assert key in ckpt and key not in acts, ("RC without checkpoint / after FW", d, m, p)
                    _, st, _ = forward(d, m, p, k, ckpt[key], keep=True)
                    acts[key] = st
                elif op == BW:
                    assert key in acts, ("BW without activations", d, m, p)
                    dout = None if k == K - 1 else recv_grad.pop(key)
                    dx = backward(d, m, p, k, dout)
                    del ckpt[key]
                    if dx is not None:
                        dinp[key] = dx
                elif op == SA:
                    mailbox[("act", m, k + 1)] = out.pop(key)
                elif op == SG:
                    mailbox[("grad", m, k - 1)] = dinp.pop(key)
                else:
                    raise AssertionError(f"unknown op {op}")
                ptr[d] += 1
                done += 1
                progressed = True
        if not progressed:
            raise RuntimeError("replay deadlock: no device can progress (cycle in the lists)")
    assert not (ckpt or acts or out or dinp or recv_act or recv_grad or mailbox), "state left after the flush"
    assert sorted(loss_sum) == list(range(N)), "loss not produced for every micro-batch"
    total_loss = 0.0
    for m in range(N):                       # reading A21: micro-batch order, fp64
        total_loss += loss_sum[m]
    summed: Dict[str, np.ndarray] = {}
    for (d, p) in sorted(G):
        for n, g in G[(d, p)].items():
            summed[n] = g.copy() if n not in summed else summed[n] + g
    return total_loss / n_tok, summed, G
