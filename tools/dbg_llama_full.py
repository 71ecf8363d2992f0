import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth
from oracle import model as om
from paper_conf_ppopp_liultj25_b200 import api
from tests.test_gpu_parity import run_plan, rounded
for cfg, S in [(synth.with_(synth.LLAMA2_7B, n_layers=2, micro_batch=1, seq_len=2048), 2),
               (synth.with_(synth.LLAMA2_7B, n_layers=2, micro_batch=1, seq_len=256), 2),
               (synth.with_(synth.LLAMA2_7B, n_layers=2, micro_batch=1, seq_len=256, hidden=1024, n_heads=8, ffn_hidden=2048, vocab=4096), 2)]:
    params = synth.make_weights(cfg)
    toks = synth.make_tokens(cfg, 2)
    loss, grads, _ = run_plan(cfg, S, 2, "1f1b", "mario", "bf16", params, toks)
    l_o, g_o = om.step(cfg, rounded(params), toks, 2, np.float32)
    print("cfg", cfg.hidden, cfg.seq_len, "loss", loss, l_o)
    for k, v in g_o.items():
        err = float(np.abs(grads[k] - v).max() / max(np.abs(v).max(), 1e-30))
        if err > 5e-3: print("  ", k, round(err, 4), float(np.abs(v).max()))
