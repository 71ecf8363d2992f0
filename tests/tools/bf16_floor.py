"""Oracle-only experiment (test infrastructure; evidence for DESIGN.md reading A19): how far does
storing tensors in bf16 — exactly where the GPU path stores them — move the fp32 definition's
gradients, and which storage point dominates the worst element?

The fp32 oracle (oracle/model.py) is re-run with RNE bf16 rounding inserted at named points of
the GPU's data flow (executor.cu stage_forward / stage_backward):
  forward : A (norm outputs A, A2, Hf), QKV (after the bias / RoPE), O, H (residual stream H1 /
            layer outputs / embedding), Z (fc1 / gate-up output), G (GeLU / SwiGLU output)
  backward: dlog (dlogits), dA (dgrad outputs feeding a norm backward: dHf, dA2, dA),
            dH (residual-stream gradients dH1 / dH_in), dZ, dG (dM, LLaMA), dO, dQKV
Matrices are bf16-rounded as in bf16 mode (reading A6). Prints the worst per-tensor inf- and l2-
relative error with every point on, with each point switched off alone, and with only that
point on.

    python tests/tools/bf16_floor.py gpt13 2 2048 [N]      # family/width, layers, seq len
"""
from __future__ import annotations

import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))

import synth  # noqa: E402
from oracle import model as om  # noqa: E402

POINTS = ["A", "QKV", "O", "H", "Z", "G", "dlog", "dA", "dH", "dZ", "dG", "dO", "dQKV"]
# "dHs": the residual-stream gradient kept in fp32 inside a stage and rounded to bf16 only where it
# crosses a stage boundary (the SG/RG message), every LPS layers
LPS = int(os.environ.get("LPS", "1"))


def rb(x):
    return synth.round_to_bf16(np.asarray(x, np.float32))


def step_rounded(cfg, params, tokens, n_micro, on):
    R = (lambda k, x: rb(x) if k in on else x)
    P = {k: np.asarray(v, np.float32) for k, v in params.items()}
    G = {k: np.zeros_like(v) for k, v in P.items()}
    mbs, s, h, nh = cfg.micro_batch, cfg.seq_len, cfg.hidden, cfg.n_heads
    n_tok = n_micro * mbs * s
    gpt = cfg.family == "gpt"
    rope = om.rope_tables(s, cfg.head_dim, cfg.rope_base, np.float32) if not gpt else None
    red = (0, 1)
    total = 0.0
    for mi in range(n_micro):
        blk = tokens[mi * mbs:(mi + 1) * mbs]
        x, y = blk[:, :s], blk[:, 1:]
        H = R("H", om.embed_fwd(cfg, P, x))
        caches = []
        for l in range(cfg.n_layers):
            p = f"h{l}."
            c = {"H_in": H}
            if gpt:
                A, c["n1"] = om.layernorm_fwd(H, P[p + "ln1.g"], P[p + "ln1.b"], cfg.norm_eps)
                A = R("A", A)
                QKV = R("QKV", om._lin(A, P[p + "qkv.w"], P[p + "qkv.b"]))
            else:
                A, c["n1"] = om.rmsnorm_fwd(H, P[p + "n1.g"], cfg.norm_eps)
                A = R("A", A)
                QKV = R("QKV", om._lin(A, P[p + "qkv.w"]))
            c["A"] = A
            q, k, v = (om._split_heads(QKV[..., i * h:(i + 1) * h], nh) for i in range(3))
            if not gpt:
                q, k = R("QKV", om.rope_apply(q, *rope)), R("QKV", om.rope_apply(k, *rope))
            O, lse = om.attention_fwd(q, k, v)
            O = R("O", O)
            c.update(q=q, k=k, v=v, lse=lse)
            Om = om._merge_heads(O)
            c["Om"] = Om
            if gpt:
                H1 = R("H", H + om._lin(Om, P[p + "proj.w"], P[p + "proj.b"]))
                A2, c["n2"] = om.layernorm_fwd(H1, P[p + "ln2.g"], P[p + "ln2.b"], cfg.norm_eps)
                A2 = R("A", A2)
                Zf = om._lin(A2, P[p + "fc1.w"], P[p + "fc1.b"])
                Z = R("Z", Zf)
                Gt = R("G", om.gelu_tanh(Zf))          # the fc1 epilogue: gelu of the fp32 accumulator
                H = R("H", H1 + om._lin(Gt, P[p + "fc2.w"], P[p + "fc2.b"]))
                c.update(A2=A2, Z=Z)
            else:
                H1 = R("H", H + om._lin(Om, P[p + "o.w"]))
                A2, c["n2"] = om.rmsnorm_fwd(H1, P[p + "n2.g"], cfg.norm_eps)
                A2 = R("A", A2)
                f = cfg.ffn_hidden
                GU = R("Z", om._lin(A2, P[p + "gu.w"]))
                g_, u_ = GU[..., :f], GU[..., f:]
                M = R("G", g_ * om.sigmoid(g_) * u_)
                H = R("H", H1 + om._lin(M, P[p + "down.w"]))
                c.update(A2=A2, g=g_, u=u_)
            c["H1"] = H1
            caches.append(c)
        Hf, ncache, logits = om.head_fwd(cfg, P, H)
        Hf = R("A", Hf)
        logits = np.matmul(Hf, om.head_weight(cfg, P).T)
        tok_loss, probs = om.cross_entropy(logits, y)
        total += float(tok_loss.sum(dtype=np.float64))
        onehot = np.zeros_like(probs)
        np.put_along_axis(onehot, y[..., None], 1.0, axis=-1)
        dlog = R("dlog", (probs - onehot) / n_tok)
        hname = "wte" if (gpt and cfg.tie_embeddings) else ("head.w" if gpt else "out.w")
        G[hname] += om._wgrad(dlog, Hf)
        dHf = R("dA", np.matmul(dlog, om.head_weight(cfg, P)))
        if gpt:
            dH, dg, db = om.layernorm_bwd(dHf, ncache, P["lnf.g"])
            G["lnf.g"] += dg
            G["lnf.b"] += db
        else:
            dH, dg = om.rmsnorm_bwd(dHf, ncache, P["nf.g"])
            G["nf.g"] += dg
        dH = R("dH", dH)
        for l in reversed(range(cfg.n_layers)):
            p, c = f"h{l}.", caches[l]
            if gpt:
                Gt = R("G", om.gelu_tanh(c["Z"]))      # recomputed from the stored Z
                dHo = R("dHop", dH)                   # bf16 GEMM operand copy of an fp32 dH
                G[p + "fc2.w"] += om._wgrad(dHo, Gt)
                G[p + "fc2.b"] += dH.sum(axis=red)
                dZ = R("dZ", np.matmul(dHo, P[p + "fc2.w"]) * om.gelu_tanh_grad(c["Z"]))
                G[p + "fc1.w"] += om._wgrad(dZ, c["A2"])
                G[p + "fc1.b"] += dZ.sum(axis=red)
                dA2 = R("dA", np.matmul(dZ, P[p + "fc1.w"]))
                dx, dg, db = om.layernorm_bwd(dA2, c["n2"], P[p + "ln2.g"])
                G[p + "ln2.g"] += dg
                G[p + "ln2.b"] += db
                dH1 = R("dH", dH + dx)
                dH1o = R("dHop", dH1)
                G[p + "proj.w"] += om._wgrad(dH1o, c["Om"])
                G[p + "proj.b"] += dH1.sum(axis=red)
                dOm = R("dO", np.matmul(dH1o, P[p + "proj.w"]))
            else:
                g_, u_ = c["g"], c["u"]
                sg = om.sigmoid(g_)
                M = R("G", g_ * sg * u_)
                dHo = R("dHop", dH)
                G[p + "down.w"] += om._wgrad(dHo, M)
                dM = R("dG", np.matmul(dHo, P[p + "down.w"]))
                dg_ = dM * u_ * sg * (1.0 + g_ * (1.0 - sg))
                du_ = dM * g_ * sg
                dGU = R("dZ", np.concatenate([dg_, du_], axis=-1))
                G[p + "gu.w"] += om._wgrad(dGU, c["A2"])
                dA2 = R("dA", np.matmul(dGU, P[p + "gu.w"]))
                dx, dgam = om.rmsnorm_bwd(dA2, c["n2"], P[p + "n2.g"])
                G[p + "n2.g"] += dgam
                dH1 = R("dH", dH + dx)
                dH1o = R("dHop", dH1)
                G[p + "o.w"] += om._wgrad(dH1o, c["Om"])
                dOm = R("dO", np.matmul(dH1o, P[p + "o.w"]))
            dO = om._split_heads(dOm, nh)
            dq, dk, dv = om.attention_bwd(dO, c["q"], c["k"], c["v"], c["lse"])
            if not gpt:
                dq, dk = om.rope_apply(dq, *rope, inverse=True), om.rope_apply(dk, *rope, inverse=True)
            dQKV = R("dQKV", np.concatenate([om._merge_heads(dq), om._merge_heads(dk), om._merge_heads(dv)], axis=-1))
            G[p + "qkv.w"] += om._wgrad(dQKV, c["A"])
            if gpt:
                G[p + "qkv.b"] += dQKV.sum(axis=red)
            dA = R("dA", np.matmul(dQKV, P[p + "qkv.w"]))
            if gpt:
                dx, dg, db = om.layernorm_bwd(dA, c["n1"], P[p + "ln1.g"])
                G[p + "ln1.g"] += dg
                G[p + "ln1.b"] += db
            else:
                dx, dg = om.rmsnorm_bwd(dA, c["n1"], P[p + "n1.g"])
                G[p + "n1.g"] += dg
            dH = R("dH", dH1 + dx)
            if "dHs" in on and l % LPS == 0 and l > 0:
                dH = rb(dH)
        ename = "wte" if gpt else "emb"
        np.add.at(G[ename], x.reshape(-1), dH.reshape(-1, h))
        if gpt:
            G["wpe"][:s] += dH.sum(axis=0)
    return total / n_tok, G


def errors(g, o):
    wi = max((float(np.abs(g[k] - o[k]).max() / max(np.abs(o[k]).max(), 1e-30)), k) for k in o)
    wl = max((float(np.linalg.norm(g[k] - o[k]) / max(np.linalg.norm(o[k]), 1e-30)), k) for k in o)
    return wi, wl


CFGS = {"tiny": synth.TINY_GPT, "tinyl": synth.tiny_llama(), "gpt13": synth.GPT3_1P3B, "gpt27": synth.GPT3_2P7B,
        "llama7": synth.LLAMA2_7B, "llama13": synth.LLAMA2_13B}


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "tiny"
    L = int(sys.argv[2]) if len(sys.argv) > 2 else 2
    s = int(sys.argv[3]) if len(sys.argv) > 3 else CFGS[name].seq_len
    N = int(sys.argv[4]) if len(sys.argv) > 4 else 2
    only = sys.argv[5].split(",") if len(sys.argv) > 5 else None
    cfg = synth.with_(CFGS[name], n_layers=L, seq_len=s, micro_batch=min(CFGS[name].micro_batch, 2))
    params = {k: (synth.round_to_bf16(v) if v.ndim == 2 else v) for k, v in synth.make_weights(cfg).items()}
    toks = synth.make_tokens(cfg, N)
    t0 = time.time()
    l_o, g_o = om.step(cfg, params, toks, N, np.float32)
    print(f"{name} L={L} s={s} N={N} h={cfg.hidden}: oracle {time.time() - t0:.1f}s", flush=True)
    fp32dh = set(POINTS) - {"dH"} | {"dHs", "dHop"}
    variants = [("all", set(POINTS)), ("fp32-dH", fp32dh)]
    if os.environ.get("FP32DH_ONLY"):
        variants += [(f"fp32-dH-{p}", fp32dh - {p}) for p in POINTS if p != "dH"]
        for tag, on in [variants[0], variants[1]] + variants[2:]:
            pass
    pts = only or POINTS
    if not os.environ.get("FP32DH_ONLY"):
        variants += [(f"all-{p}", set(POINTS) - {p}) for p in pts]
        variants += [(f"only-{p}", {p}) for p in pts]
    keep = os.environ.get("VARIANTS")
    if keep:
        variants = [v for v in variants if v[0] in keep.split(",")]
    for tag, on in variants:
        l1, g1 = step_rounded(cfg, params, toks, N, on)
        (ei, ki), (el, kl) = errors(g1, g_o)
        print(f"{tag:10s} loss {abs(l1 - l_o) / l_o:.2e}  inf {ei:.4f} ({ki})  l2 {el:.4f} ({kl})", flush=True)


if __name__ == "__main__":
    main()
