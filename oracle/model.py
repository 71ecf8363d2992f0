"""ORACLE (test infrastructure only) — decoder LM forward/backward, plain numpy.

What it computes: the loss and per-parameter gradients of one training iteration of a
GPT-3 / LLaMA2-style decoder over the whole global batch, UNPIPELINED and WITHOUT
activation checkpointing. This is the plain definition every Mario plan must reproduce:
checkpointing "drops the activation tensors ... and recomputes them by replaying the
forward" and the pipeline is synchronous with a flush so every
micro-batch sees the same weights. The model details the paper leaves open
(Table 4, P:292-299 gives only hidden/layers/heads/seqlen) follow SURVEY §8(c) readings
A1 (GPT), A2 (LLaMA2), A4 (labels/loss), A5 (no dropout), A6 (precision), A7 (grads).

Everything is written out op by op; numpy matmul is the only library primitive. The
precision is a parameter: float64 for pins (finite differences), float32 for parity.

Pinned by tests/test_oracle_model.py (central FD in fp64, torch-fp64 autograd
cross-check, zero-head closed form loss = ln V, q=0 uniform attention, s=1, LN/RMS
moments, causality, micro-batch split invariance, CE row sums).
"""
from __future__ import annotations

import math
from typing import Dict, Tuple

import numpy as np

# ----------------------------------------------------------------------------- norms
# A1: LN(z) = (z - mean) / sqrt(var + eps) * g + b, biased variance over the hidden dim.


def layernorm_fwd(x, g, b, eps):
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    rstd = 1.0 / np.sqrt(var + eps)
    xhat = (x - mu) * rstd
    return xhat * g + b, (xhat, rstd)


def layernorm_bwd(dy, cache, g):
    """SURVEY §8(c) c1 backward: g' = dy*gamma; dx = (g' - mean g' - xhat*mean(g'*xhat))*rstd."""
    xhat, rstd = cache
    gp = dy * g
    dx = (gp - gp.mean(axis=-1, keepdims=True) - xhat * (gp * xhat).mean(axis=-1, keepdims=True)) * rstd
    red = tuple(range(dy.ndim - 1))
    return dx, (dy * xhat).sum(axis=red), dy.sum(axis=red)


# A2: RMS(z) = z / sqrt(mean(z^2) + eps) * g
def rmsnorm_fwd(x, g, eps):
    rstd = 1.0 / np.sqrt((x * x).mean(axis=-1, keepdims=True) + eps)
    xhat = x * rstd
    return xhat * g, (xhat, rstd)


def rmsnorm_bwd(dy, cache, g):
    xhat, rstd = cache
    gp = dy * g
    dx = (gp - xhat * (gp * xhat).mean(axis=-1, keepdims=True)) * rstd
    red = tuple(range(dy.ndim - 1))
    return dx, (dy * xhat).sum(axis=red)


# ----------------------------------------------------------------------- activations
_C = math.sqrt(2.0 / math.pi)


def gelu_tanh(z):
    """A1: G = 0.5 z (1 + tanh(sqrt(2/pi)(z + 0.044715 z^3)))."""
    return 0.5 * z * (1.0 + np.tanh(_C * (z + 0.044715 * z ** 3)))


def gelu_tanh_grad(z):
    t = np.tanh(_C * (z + 0.044715 * z ** 3))
    return 0.5 * (1.0 + t) + 0.5 * z * (1.0 - t * t) * _C * (1.0 + 3 * 0.044715 * z * z)


def sigmoid(u):
    return 1.0 / (1.0 + np.exp(-u))


# ---------------------------------------------------------------------------- RoPE
def rope_tables(s, dh, base, dtype):
    """A2: theta_i = base^(-2i/dh) for i < dh/2, angle t*theta_i at position t."""
    i = np.arange(dh // 2, dtype=np.float64)
    theta = base ** (-2.0 * i / dh)
    ang = np.arange(s, dtype=np.float64)[:, None] * theta[None, :]
    return np.cos(ang).astype(dtype), np.sin(ang).astype(dtype)


def rope_apply(x, cos, sin, inverse=False):
    """Rotate-half: (x_i, x_{i+dh/2}) <- (x_i cos - x_{i+dh/2} sin, x_i sin + x_{i+dh/2} cos).
    x: [b, nh, s, dh]; inverse=True rotates by -t*theta (the backward)."""
    half = x.shape[-1] // 2
    x1, x2 = x[..., :half], x[..., half:]
    sn = -sin if inverse else sin
    return np.concatenate([x1 * cos - x2 * sn, x1 * sn + x2 * cos], axis=-1)


# ------------------------------------------------------------------------ attention
def attention_fwd(q, k, v):
    """Causal softmax attention per (sample, head). q,k,v: [b, nh, s, dh].
    S = q k^T / sqrt(dh); S[t,u] = -inf for u > t; P = softmax_u(S); O = P v.
    Returns O and the row log-sum-exp (the backward recomputes P from it)."""
    s, dh = q.shape[-2], q.shape[-1]
    scale = 1.0 / math.sqrt(dh)
    S = np.matmul(q, np.swapaxes(k, -1, -2)) * scale
    mask = np.triu(np.ones((s, s), dtype=bool), k=1)
    S = np.where(mask, -np.inf, S)
    m = S.max(axis=-1, keepdims=True)
    e = np.exp(S - m)
    l = e.sum(axis=-1, keepdims=True)
    P = e / l
    O = np.matmul(P, v)
    return O, (m + np.log(l))


def attention_bwd(dO, q, k, v, lse):
    """dV = P^T dO; dP = dO V^T; dS = P*(dP - rowsum(dP*P)); dQ = dS K/sqrt(dh); dK = dS^T Q/sqrt(dh)."""
    s, dh = q.shape[-2], q.shape[-1]
    scale = 1.0 / math.sqrt(dh)
    S = np.matmul(q, np.swapaxes(k, -1, -2)) * scale
    mask = np.triu(np.ones((s, s), dtype=bool), k=1)
    P = np.where(mask, 0.0, np.exp(np.where(mask, 0.0, S) - lse)).astype(q.dtype)
    dV = np.matmul(np.swapaxes(P, -1, -2), dO)
    dP = np.matmul(dO, np.swapaxes(v, -1, -2))
    dS = P * (dP - (dP * P).sum(axis=-1, keepdims=True))
    dQ = np.matmul(dS, k) * scale
    dK = np.matmul(np.swapaxes(dS, -1, -2), q) * scale
    return dQ, dK, dV


def _split_heads(x, nh):  # [b, s, h] -> [b, nh, s, dh]
    b, s, h = x.shape
    return x.reshape(b, s, nh, h // nh).transpose(0, 2, 1, 3)


def _merge_heads(x):  # [b, nh, s, dh] -> [b, s, h]
    b, nh, s, dh = x.shape
    return x.transpose(0, 2, 1, 3).reshape(b, s, nh * dh)


# ------------------------------------------------------------------- decoder layer
def _wgrad(dY, X):
    """dW[n, k] = sum over all tokens of dY[.., n] * X[.., k]  (i.e. dY^T X)."""
    return np.matmul(dY.reshape(-1, dY.shape[-1]).T, X.reshape(-1, X.shape[-1]))


def _lin(x, w, b=None):
    y = np.matmul(x, w.T)
    return y if b is None else y + b


def layer_fwd(cfg, P, l, H, rope):
    """One decoder layer on H [b, s, h]; returns (H_out, cache)."""
    p, nh, eps = f"h{l}.", cfg.n_heads, cfg.norm_eps
    h = cfg.hidden
    c = {"H_in": H}
    if cfg.family == "gpt":
        A, c["n1"] = layernorm_fwd(H, P[p + "ln1.g"], P[p + "ln1.b"], eps)
        QKV = _lin(A, P[p + "qkv.w"], P[p + "qkv.b"])
    else:
        A, c["n1"] = rmsnorm_fwd(H, P[p + "n1.g"], eps)
        QKV = _lin(A, P[p + "qkv.w"])
    c["A"] = A
    # qkv.w rows: [0,h)=Q, [h,2h)=K, [2h,3h)=V; head j uses rows j*dh..(j+1)*dh-1 of each block
    q, k, v = (_split_heads(QKV[..., i * h:(i + 1) * h], nh) for i in range(3))
    if cfg.family == "llama":
        cos, sin = rope
        q, k = rope_apply(q, cos, sin), rope_apply(k, cos, sin)
    O, lse = attention_fwd(q, k, v)
    c.update(q=q, k=k, v=v, O=O, lse=lse)
    Om = _merge_heads(O)
    c["Om"] = Om
    if cfg.family == "gpt":
        H1 = H + _lin(Om, P[p + "proj.w"], P[p + "proj.b"])
        A2, c["n2"] = layernorm_fwd(H1, P[p + "ln2.g"], P[p + "ln2.b"], eps)
        Z = _lin(A2, P[p + "fc1.w"], P[p + "fc1.b"])
        G = gelu_tanh(Z)
        H2 = H1 + _lin(G, P[p + "fc2.w"], P[p + "fc2.b"])
        c.update(A2=A2, Z=Z, G=G)
    else:
        H1 = H + _lin(Om, P[p + "o.w"])
        A2, c["n2"] = rmsnorm_fwd(H1, P[p + "n2.g"], eps)
        f = cfg.ffn_hidden
        GU = _lin(A2, P[p + "gu.w"])        # gu.w rows: gate [0,f) then up [f,2f)
        g_, u_ = GU[..., :f], GU[..., f:]
        M = g_ * sigmoid(g_) * u_          # SwiGLU: silu(gate) * up
        H2 = H1 + _lin(M, P[p + "down.w"])
        c.update(A2=A2, g=g_, u=u_, M=M)
    return H2, c


def layer_bwd(cfg, P, l, dH2, c, rope, G):
    """Backward of layer_fwd; accumulates into grads dict G; returns dH_in."""
    p, nh = f"h{l}.", cfg.n_heads
    red = (0, 1)
    if cfg.family == "gpt":
        # H2 = H1 + G fc2^T + b
        G[p + "fc2.w"] += _wgrad(dH2, c["G"])
        G[p + "fc2.b"] += dH2.sum(axis=red)
        dG = np.matmul(dH2, P[p + "fc2.w"])
        dZ = dG * gelu_tanh_grad(c["Z"])
        G[p + "fc1.w"] += _wgrad(dZ, c["A2"])
        G[p + "fc1.b"] += dZ.sum(axis=red)
        dA2 = np.matmul(dZ, P[p + "fc1.w"])
        dx, dg, db = layernorm_bwd(dA2, c["n2"], P[p + "ln2.g"])
        G[p + "ln2.g"] += dg
        G[p + "ln2.b"] += db
        dH1 = dH2 + dx
        G[p + "proj.w"] += _wgrad(dH1, c["Om"])
        G[p + "proj.b"] += dH1.sum(axis=red)
        dOm = np.matmul(dH1, P[p + "proj.w"])
    else:
        G[p + "down.w"] += _wgrad(dH2, c["M"])
        dM = np.matmul(dH2, P[p + "down.w"])
        g_, u_ = c["g"], c["u"]
        sg = sigmoid(g_)
        dg_ = dM * u_ * sg * (1.0 + g_ * (1.0 - sg))   # silu'(g) = s(g)(1 + g(1 - s(g)))
        du_ = dM * g_ * sg
        dGU = np.concatenate([dg_, du_], axis=-1)
        G[p + "gu.w"] += _wgrad(dGU, c["A2"])
        dA2 = np.matmul(dGU, P[p + "gu.w"])
        dx, dgam = rmsnorm_bwd(dA2, c["n2"], P[p + "n2.g"])
        G[p + "n2.g"] += dgam
        dH1 = dH2 + dx
        G[p + "o.w"] += _wgrad(dH1, c["Om"])
        dOm = np.matmul(dH1, P[p + "o.w"])
    dO = _split_heads(dOm, nh)
    dq, dk, dv = attention_bwd(dO, c["q"], c["k"], c["v"], c["lse"])
    if cfg.family == "llama":
        cos, sin = rope
        dq, dk = rope_apply(dq, cos, sin, inverse=True), rope_apply(dk, cos, sin, inverse=True)
    dQKV = np.concatenate([_merge_heads(dq), _merge_heads(dk), _merge_heads(dv)], axis=-1)
    G[p + "qkv.w"] += _wgrad(dQKV, c["A"])
    if cfg.family == "gpt":
        G[p + "qkv.b"] += dQKV.sum(axis=red)
    dA = np.matmul(dQKV, P[p + "qkv.w"])
    if cfg.family == "gpt":
        dx, dg, db = layernorm_bwd(dA, c["n1"], P[p + "ln1.g"])
        G[p + "ln1.g"] += dg
        G[p + "ln1.b"] += db
    else:
        dx, dg = rmsnorm_bwd(dA, c["n1"], P[p + "n1.g"])
        G[p + "n1.g"] += dg
    return dH1 + dx


# ------------------------------------------------------------------ embedding / head
def embed_fwd(cfg, P, x):
    if cfg.family == "gpt":
        return P["wte"][x] + P["wpe"][None, : x.shape[1]]
    return P["emb"][x]


def head_weight(cfg, P):
    if cfg.family == "gpt":
        return P["wte"] if cfg.tie_embeddings else P["head.w"]
    return P["out.w"]


def head_fwd(cfg, P, H):
    if cfg.family == "gpt":
        Hf, cache = layernorm_fwd(H, P["lnf.g"], P["lnf.b"], cfg.norm_eps)
    else:
        Hf, cache = rmsnorm_fwd(H, P["nf.g"], cfg.norm_eps)
    return Hf, cache, np.matmul(Hf, head_weight(cfg, P).T)


def cross_entropy(logits, y):
    """l[t] = logsumexp(logits[t]) - logits[t, y_t] (A4); returns per-token losses and softmax."""
    m = logits.max(axis=-1, keepdims=True)
    e = np.exp(logits - m)
    ssum = e.sum(axis=-1, keepdims=True)
    lse = (m + np.log(ssum))[..., 0]
    picked = np.take_along_axis(logits, y[..., None], axis=-1)[..., 0]
    return lse - picked, e / ssum


# ------------------------------------------------------------------------ full model
def forward_logits(cfg, P, x, dtype=np.float64):
    """Logits [b, s, V] for tokens x [b, s] (used by the causality pin)."""
    P = {k: v.astype(dtype) for k, v in P.items()}
    rope = rope_tables(x.shape[1], cfg.head_dim, cfg.rope_base, dtype) if cfg.family == "llama" else None
    H = embed_fwd(cfg, P, x)
    for l in range(cfg.n_layers):
        H, _ = layer_fwd(cfg, P, l, H, rope)
    return head_fwd(cfg, P, H)[2]


def microbatch_fwd_bwd(cfg, P, x, y, n_tok_total, G, dtype):
    """Forward + backward of one micro-batch; grads of (sum of its token losses)/Ntok are
    added into G. Returns the micro-batch's loss SUM (not divided)."""
    s = x.shape[1]
    rope = rope_tables(s, cfg.head_dim, cfg.rope_base, dtype) if cfg.family == "llama" else None
    H = embed_fwd(cfg, P, x)
    caches = []
    for l in range(cfg.n_layers):
        H, c = layer_fwd(cfg, P, l, H, rope)
        caches.append(c)
    Hf, ncache, logits = head_fwd(cfg, P, H)
    tok_loss, probs = cross_entropy(logits, y)
    # dlogits = (softmax - onehot(y)) / Ntok  (SURVEY c1 backward)
    onehot = np.zeros_like(probs)
    np.put_along_axis(onehot, y[..., None], 1.0, axis=-1)
    dlogits = (probs - onehot) / n_tok_total
    W = head_weight(cfg, P)
    hname = "wte" if (cfg.family == "gpt" and cfg.tie_embeddings) else ("head.w" if cfg.family == "gpt" else "out.w")
    G[hname] += _wgrad(dlogits, Hf)
    dHf = np.matmul(dlogits, W)
    if cfg.family == "gpt":
        dH, dg, db = layernorm_bwd(dHf, ncache, P["lnf.g"])
        G["lnf.g"] += dg
        G["lnf.b"] += db
    else:
        dH, dg = rmsnorm_bwd(dHf, ncache, P["nf.g"])
        G["nf.g"] += dg
    for l in reversed(range(cfg.n_layers)):
        dH = layer_bwd(cfg, P, l, dH, caches[l], rope, G)
    # embedding: dwte[v] += sum_{x=v} dH0; dwpe[t] = sum_b dH0[b, t]
    ename = "wte" if cfg.family == "gpt" else "emb"
    np.add.at(G[ename], x.reshape(-1), dH.reshape(-1, cfg.hidden))
    if cfg.family == "gpt":
        G["wpe"][:s] += dH.sum(axis=0)
    return tok_loss.sum(dtype=np.float64)


def step(cfg, params: Dict[str, np.ndarray], tokens: np.ndarray, n_micro: int,
         dtype=np.float64) -> Tuple[float, Dict[str, np.ndarray]]:
    """One training iteration's loss and gradients (plain definition).

    tokens: int [n_micro*mbs, s+1]; x = tokens[:, :s], y = tokens[:, 1:] (A4).
    Loss = (sum over all micro-batches, samples, positions of l) / Ntok. Per-micro-batch
    loss sums are combined in fp64 in micro-batch order (A21). Gradients are summed over
    micro-batches in `dtype` in micro-batch order.
    """
    P = {k: np.asarray(v).astype(dtype) for k, v in params.items()}
    G = {k: np.zeros_like(v) for k, v in P.items()}
    mbs, s = cfg.micro_batch, cfg.seq_len
    assert tokens.shape == (n_micro * mbs, s + 1), tokens.shape
    n_tok = n_micro * mbs * s
    total = 0.0
    for m in range(n_micro):
        blk = tokens[m * mbs:(m + 1) * mbs]
        total += float(microbatch_fwd_bwd(cfg, P, blk[:, :s], blk[:, 1:], n_tok, G, dtype))
    return total / n_tok, G
