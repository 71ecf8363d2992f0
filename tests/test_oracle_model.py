"""Pins for oracle/model.py against things other than itself:
finite differences, an independent torch-fp64 autograd implementation, closed forms,
invariants. Runs on CPU (-m "not gpu")."""
import math

import numpy as np
import pytest
import torch
import torch.nn.functional as F

import synth
from oracle import model as om

FD_GPT = synth.ModelCfg("gpt", 2, 8, 2, 32, 16, 5, 2, True)
FD_LLAMA = synth.ModelCfg("llama", 2, 8, 2, 12, 16, 5, 2, False)


def _rel(a, b):
    return float(np.max(np.abs(a - b)) / max(np.max(np.abs(b)), 1e-300))


# ---------------------------------------------------------------- finite differences
@pytest.mark.parametrize("cfg", [FD_GPT, FD_LLAMA], ids=["gpt", "llama"])
def test_central_fd_every_entry(cfg):
    """Central FD in fp64, every parameter entry, rel err <= 1e-6 (c4 Backward (1))."""
    P = synth.make_weights(cfg, seed=7, dtype=np.float64)
    toks = synth.make_tokens(cfg, n_micro=2, seed=11)
    loss, G = om.step(cfg, P, toks, 2, np.float64)
    eps = 1e-5
    for name, w in P.items():
        fd = np.zeros_like(w)
        flat = w.reshape(-1)
        for i in range(flat.size):
            old = flat[i]
            flat[i] = old + eps
            lp, _ = _loss_only(cfg, P, toks)
            flat[i] = old - eps
            lm, _ = _loss_only(cfg, P, toks)
            flat[i] = old
            fd.reshape(-1)[i] = (lp - lm) / (2 * eps)
        err = np.max(np.abs(fd - G[name])) / max(np.max(np.abs(G[name])), 1e-12)
        assert err < 1e-6, (name, err)


def _loss_only(cfg, P, toks):
    return om.step(cfg, P, toks, 2, np.float64)


# ------------------------------------------------------- independent torch fp64 model
def torch_step(cfg, P, toks, n_micro):
    """Independent implementation with torch.nn.functional + autograd (test-only)."""
    T = {k: torch.tensor(v, dtype=torch.float64, requires_grad=True) for k, v in P.items()}
    tt = torch.tensor(toks, dtype=torch.long)
    x, y = tt[:, :-1], tt[:, 1:]
    h, nh, dh, s = cfg.hidden, cfg.n_heads, cfg.head_dim, cfg.seq_len
    if cfg.family == "gpt":
        H = T["wte"][x] + T["wpe"][:s][None]
    else:
        H = T["emb"][x]
        pos = torch.arange(s, dtype=torch.float64)[:, None]
        inv = cfg.rope_base ** (-torch.arange(0, dh, 2, dtype=torch.float64) / dh)
        ang = pos * inv[None]
        cos, sin = torch.cos(ang), torch.sin(ang)

        def rope(t):
            t1, t2 = t[..., : dh // 2], t[..., dh // 2:]
            return torch.cat([t1 * cos - t2 * sin, t2 * cos + t1 * sin], -1)

    def rms(z, g):
        return z * torch.rsqrt(z.pow(2).mean(-1, keepdim=True) + cfg.norm_eps) * g

    B = x.shape[0]
    for l in range(cfg.n_layers):
        p = f"h{l}."
        if cfg.family == "gpt":
            A = F.layer_norm(H, (h,), T[p + "ln1.g"], T[p + "ln1.b"], cfg.norm_eps)
            qkv = F.linear(A, T[p + "qkv.w"], T[p + "qkv.b"])
        else:
            A = rms(H, T[p + "n1.g"])
            qkv = F.linear(A, T[p + "qkv.w"])
        q, k, v = qkv.split(h, -1)
        q, k, v = (t.view(B, s, nh, dh).transpose(1, 2) for t in (q, k, v))
        if cfg.family == "llama":
            q, k = rope(q), rope(k)
        o = F.scaled_dot_product_attention(q, k, v, is_causal=True)
        o = o.transpose(1, 2).reshape(B, s, h)
        if cfg.family == "gpt":
            H = H + F.linear(o, T[p + "proj.w"], T[p + "proj.b"])
            A2 = F.layer_norm(H, (h,), T[p + "ln2.g"], T[p + "ln2.b"], cfg.norm_eps)
            H = H + F.linear(F.gelu(F.linear(A2, T[p + "fc1.w"], T[p + "fc1.b"]), approximate="tanh"),
                             T[p + "fc2.w"], T[p + "fc2.b"])
        else:
            H = H + F.linear(o, T[p + "o.w"])
            A2 = rms(H, T[p + "n2.g"])
            g, u = F.linear(A2, T[p + "gu.w"]).split(cfg.ffn_hidden, -1)
            H = H + F.linear(F.silu(g) * u, T[p + "down.w"])
    if cfg.family == "gpt":
        Hf = F.layer_norm(H, (h,), T["lnf.g"], T["lnf.b"], cfg.norm_eps)
        logits = Hf @ T["wte"].T
    else:
        logits = rms(H, T["nf.g"]) @ T["out.w"].T
    loss = F.cross_entropy(logits.reshape(-1, cfg.vocab), y.reshape(-1), reduction="mean")
    loss.backward()
    return float(loss), {k: t.grad.numpy() for k, t in T.items()}


@pytest.mark.parametrize("cfg", [synth.TINY_GPT, synth.tiny_llama()], ids=["gpt", "llama"])
def test_torch_fp64_crosscheck(cfg):
    P = synth.make_weights(cfg, seed=3, dtype=np.float64)
    toks = synth.make_tokens(cfg, n_micro=3, seed=5)
    loss, G = om.step(cfg, P, toks, 3, np.float64)
    tl, tG = torch_step(cfg, P, toks, 3)
    assert abs(loss - tl) < 1e-12 * abs(tl)
    for k in P:
        assert _rel(G[k], tG[k]) < 1e-10, k


def test_fp32_close_to_fp64():
    cfg = synth.TINY_GPT
    P = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 4)
    l64, G64 = om.step(cfg, P, toks, 4, np.float64)
    l32, G32 = om.step(cfg, P, toks, 4, np.float32)
    assert abs(l32 - l64) / l64 < 1e-6
    for k in P:
        assert G32[k].dtype == np.float32
        assert _rel(G32[k], G64[k]) < 1e-4, k


# ------------------------------------------------------------------- closed forms
@pytest.mark.parametrize("cfg", [synth.TINY_GPT, synth.tiny_llama()], ids=["gpt", "llama"])
def test_zero_head_loss_is_lnV(cfg):
    """Head matrix = 0 => logits == 0 => loss = ln V exactly; every grad upstream of the
    logits is exactly 0; head-grad rows sum to 0 (CE rows sum to 0)."""
    P = synth.make_weights(cfg, dtype=np.float64)
    hname = "wte" if cfg.family == "gpt" else "out.w"
    P[hname][:] = 0.0
    toks = synth.make_tokens(cfg, 2)
    loss, G = om.step(cfg, P, toks, 2, np.float64)
    assert abs(loss - math.log(cfg.vocab)) < 1e-13
    for k, g in G.items():
        if k == hname:
            # dhead = dlogits^T Hf with dlogits = (1/V - onehot)/Ntok: sum over vocab rows = 0
            assert np.abs(g.sum(axis=0)).max() < 1e-15
            assert np.abs(g).max() > 0
        else:
            assert np.all(g == 0.0), k


def test_attention_q_zero_is_prefix_mean():
    rng = np.random.default_rng(0)
    b, nh, s, dh = 2, 3, 7, 4
    q = np.zeros((b, nh, s, dh))
    k = rng.standard_normal((b, nh, s, dh))
    v = rng.standard_normal((b, nh, s, dh))
    O, lse = om.attention_fwd(q, k, v)
    expect = np.cumsum(v, axis=2) / np.arange(1, s + 1)[None, None, :, None]
    assert np.allclose(O, expect, atol=1e-14)
    assert np.allclose(lse[..., 0], np.log(np.arange(1, s + 1))[None, None], atol=1e-14)


def test_attention_s1_is_v():
    rng = np.random.default_rng(1)
    q, k, v = (rng.standard_normal((1, 2, 1, 8)) for _ in range(3))
    O, _ = om.attention_fwd(q, k, v)
    assert np.array_equal(O, v)


def test_attention_bwd_matches_torch_sdpa():
    rng = np.random.default_rng(2)
    q, k, v, dO = (rng.standard_normal((2, 3, 9, 8)) for _ in range(4))
    O, lse = om.attention_fwd(q, k, v)
    dq, dk, dv = om.attention_bwd(dO, q, k, v, lse)
    tq, tk, tv = (torch.tensor(a, requires_grad=True) for a in (q, k, v))
    to = F.scaled_dot_product_attention(tq, tk, tv, is_causal=True)
    to.backward(torch.tensor(dO))
    assert np.allclose(O, to.detach().numpy(), atol=1e-13)
    for a, t in ((dq, tq), (dk, tk), (dv, tv)):
        assert np.allclose(a, t.grad.numpy(), atol=1e-12)


def test_norm_moments_and_dx_invariants():
    rng = np.random.default_rng(3)
    x = rng.standard_normal((5, 64)) * 3 + 1
    eps = 1e-5
    y, cache = om.layernorm_fwd(x, np.ones(64), np.zeros(64), eps)
    var = x.var(axis=-1)
    assert np.allclose(y.mean(-1), 0, atol=1e-13)
    assert np.allclose(y.var(-1), var / (var + eps), atol=1e-12)
    dy = rng.standard_normal((5, 64))
    dx, _, _ = om.layernorm_bwd(dy, cache, rng.standard_normal(64))
    assert np.allclose(dx.sum(-1), 0, atol=1e-12)
    y, cache = om.rmsnorm_fwd(x, np.ones(64), eps)
    ms = (x * x).mean(-1)
    assert np.allclose((y * y).mean(-1), ms / (ms + eps), atol=1e-12)


def test_cross_entropy_dlogits_rows_sum_zero():
    rng = np.random.default_rng(4)
    z = rng.standard_normal((3, 5, 11))
    y = rng.integers(0, 11, (3, 5))
    l, probs = om.cross_entropy(z, y)
    ref = np.log(np.exp(z).sum(-1)) - np.take_along_axis(z, y[..., None], -1)[..., 0]
    assert np.allclose(l, ref, atol=1e-13)
    assert np.allclose(probs.sum(-1), 1, atol=1e-14)


# -------------------------------------------------------------------- invariances
@pytest.mark.parametrize("cfg", [synth.TINY_GPT, synth.tiny_llama()], ids=["gpt", "llama"])
def test_causality(cfg):
    P = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 1)[:, :-1]
    t = 13
    L1 = om.forward_logits(cfg, P, toks)
    toks2 = toks.copy()
    toks2[:, t + 1:] = (toks2[:, t + 1:] + 7) % cfg.vocab
    L2 = om.forward_logits(cfg, P, toks2)
    assert np.array_equal(L1[:, : t + 1], L2[:, : t + 1])
    assert not np.allclose(L1[:, t + 1:], L2[:, t + 1:])


@pytest.mark.parametrize("cfg", [synth.TINY_GPT, synth.tiny_llama()], ids=["gpt", "llama"])
def test_microbatch_split_invariance(cfg):
    """One big batch vs N micro-batches, summed (c4 Pipelining (1))."""
    P = synth.make_weights(cfg, dtype=np.float64)
    toks = synth.make_tokens(cfg, 4)
    big = synth.with_(cfg, micro_batch=cfg.micro_batch * 4)
    l1, G1 = om.step(big, P, toks, 1, np.float64)
    l4, G4 = om.step(cfg, P, toks, 4, np.float64)
    assert abs(l1 - l4) < 1e-13 * l1
    for k in P:
        assert _rel(G4[k], G1[k]) < 1e-12, k


def test_sample_permutation_invariance():
    cfg = synth.TINY_GPT
    P = synth.make_weights(cfg, dtype=np.float64)
    toks = synth.make_tokens(cfg, 4)
    l1, G1 = om.step(cfg, P, toks, 4, np.float64)
    l2, G2 = om.step(cfg, P, toks[::-1].copy(), 4, np.float64)
    assert abs(l1 - l2) < 1e-13 * l1
    for k in P:
        assert _rel(G1[k], G2[k]) < 1e-12


def test_initial_loss_near_lnV():
    cfg = synth.TINY_GPT
    P = synth.make_weights(cfg, parity=False)
    loss, _ = om.step(cfg, P, synth.make_tokens(cfg, 2), 2, np.float32)
    assert abs(loss - math.log(cfg.vocab)) < 0.05


def test_adamw_oracle_closed_forms():
    """Pins for oracle/optim.py: step 1 with g != 0 moves every weight by lr*(sign(g) + wd*p)
    up to eps (bias-corrected m/sqrt(v) = g/|g|); zero grads only decay; a constant gradient
    keeps the normalized update at 1."""
    from oracle import optim
    rng = np.random.default_rng(0)
    p = {"w": rng.standard_normal(50)}
    g = {"w": rng.standard_normal(50)}
    m = {"w": np.zeros(50)}
    v = {"w": np.zeros(50)}
    p0 = p["w"].copy()
    optim.adamw_step(p, g, m, v, 1, lr=1e-2, eps=0.0, weight_decay=0.1)
    assert np.allclose(p["w"], p0 - 1e-2 * (np.sign(g["w"]) + 0.1 * p0), atol=1e-15)
    q = {"w": p0.copy()}
    z = {"w": np.zeros(50)}
    optim.adamw_step(q, z, {"w": np.zeros(50)}, {"w": np.zeros(50)}, 1, lr=1e-2, eps=1e-8, weight_decay=0.1)
    assert np.allclose(q["w"], p0 * (1 - 1e-3), atol=1e-15)
    c = {"w": np.full(50, 0.3)}
    r = {"w": np.zeros(50)}
    mm, vv = {"w": np.zeros(50)}, {"w": np.zeros(50)}
    for t in range(1, 6):
        before = r["w"].copy()
        optim.adamw_step(r, c, mm, vv, t, lr=1.0, eps=0.0, weight_decay=0.0)
        assert np.allclose(before - r["w"], 1.0, atol=1e-12)
