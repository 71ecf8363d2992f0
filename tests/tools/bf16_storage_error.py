# Evidence for DESIGN.md reading A19 (oracle-only experiment, not a test): how far does *storing*
# fp32 oracle's gradients at LLaMA2-7B width?  Monkey-patch rounding into a copy of the oracle.
import sys, numpy as np
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__)))))
import synth
from oracle import model as om

def rb(x):
    return synth.round_to_bf16(np.asarray(x, np.float32))

which = set(sys.argv[1].split(",")) if len(sys.argv) > 1 else set()
seq = int(sys.argv[2]) if len(sys.argv) > 2 else 256
base = {"7b": synth.LLAMA2_7B, "13b": synth.LLAMA2_13B}[sys.argv[3] if len(sys.argv) > 3 else "7b"]
cfg = synth.with_(base, n_layers=2, micro_batch=1, seq_len=seq)
P = {k: (synth.round_to_bf16(v) if v.ndim == 2 else v) for k, v in synth.make_weights(cfg).items()}
toks = synth.make_tokens(cfg, 2)
l0, g0 = om.step(cfg, P, toks, 2, np.float32)
orig_lin, orig_rms, orig_attn, orig_attn_b = om._lin, om.rmsnorm_fwd, om.attention_fwd, om.attention_bwd
if "lin" in which:
    om._lin = lambda x, w, b=None: rb(orig_lin(x, w, b))
if "norm" in which:
    def rms(x, g, eps):
        y, c = orig_rms(x, g, eps); return rb(y), c
    om.rmsnorm_fwd = rms
if "attn" in which:
    def af(q, k, v):
        O, l = orig_attn(q, k, v); return rb(O), l
    om.attention_fwd = af
    def ab(dO, q, k, v, lse):
        return tuple(rb(t) for t in orig_attn_b(dO, q, k, v, lse))
    om.attention_bwd = ab
l1, g1 = om.step(cfg, P, toks, 2, np.float32)
worst = max((float(np.abs(g1[k]-g0[k]).max()/np.abs(g0[k]).max()), k) for k in g0)
worst_l2 = max((float(np.linalg.norm(g1[k]-g0[k])/np.linalg.norm(g0[k])), k) for k in g0)
print(sorted(which), cfg.hidden, seq, "loss rel", abs(l1-l0)/l0, "worst inf", worst, "worst l2", worst_l2)
