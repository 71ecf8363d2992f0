import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth
from oracle import model as om
from paper_conf_ppopp_liultj25_b200 import _lib, api
from tests.test_gpu_parity import run_plan, rounded
cfg = synth.with_(synth.LLAMA2_7B, n_layers=2, micro_batch=1, seq_len=2048)
params = synth.make_weights(cfg)
toks = synth.make_tokens(cfg, 2)
l_o, g_o = om.step(cfg, rounded(params), toks, 2, np.float32)
L = _lib.lib()
for av, gv in [(-1, -1), (0, -1), (-1, 0), (0, 0)]:
    L.mario_k_attn_set_variant(av); L.mario_k_gemm_set_variant(gv)
    loss, grads, _ = run_plan(cfg, 2, 2, "1f1b", "mario", "bf16", params, toks)
    errs = sorted(((float(np.linalg.norm(grads[k] - v) / np.linalg.norm(v)), k) for k, v in g_o.items()), reverse=True)[:4]
    print("attn", av, "gemm", gv, "loss", loss, l_o, "worst l2", [(k, round(e, 4)) for e, k in errs], flush=True)
