import sys, torch
sys.path.insert(0, ".")
import synth
from paper_conf_ppopp_liultj25_b200 import _lib, api
cfg = synth.with_(synth.GPT3_1P3B, n_layers=1)
plan = api.Plan(cfg, 1, 2, "1f1b", "mario", dtype="bf16")
ctx = api.Context(0, 1, 0)
w, g, ws = api.alloc_for(plan, 0)
w.normal_(0, 0.02)
tok = torch.from_numpy(synth.make_tokens(cfg, 2)).cuda()
try:
    print("loss", ctx.run_iter(plan, w, tok, g, ws))
except Exception as e:
    print("ERR", e)
