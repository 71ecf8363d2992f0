"""The paper's schedule tuner with MEASURED estimators (§5.3 Eq. 1; profile step P:242):
api.profile_costs times, per micro-batch size, one loopback iteration of a 2-layer, 2-stage slice of
the model (per-layer forward / backward time and the head's extra time, mario_last_costs); mario_tune
then grid-searches scheme x PP x DP x mbs x level for the full model on 8 GPUs under a memory budget and
names the "Auto" configuration.

    python tools/tune_measured.py [cfg2|cfg3|cfg4] [budget_GB]
"""
import json
import os
import sys


sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_ppopp_liultj25_b200 import api  # noqa: E402

CFG = {"cfg2": synth.GPT3_1P3B, "cfg3": synth.LLAMA2_7B, "cfg4": synth.GPT3_2P7B}
name = sys.argv[1] if len(sys.argv) > 1 else "cfg2"
budget = int(float(sys.argv[2]) * 1e9) if len(sys.argv) > 2 else 40 * 10 ** 9
gbs = {"cfg2": 128, "cfg3": 32, "cfg4": 32}[name]
full = CFG[name]
costs = api.profile_costs(full, (1, 2, 4, 8))
rows, best = api.tune(full, 8, gbs, mem_budget=budget, costs=costs)
feas = sorted([r for r in rows if r["feasible"]], key=lambda r: -r["samples_per_s"])
out = {"config": name, "devices": 8, "global_batch": gbs, "mem_budget_GB": budget / 1e9,
       "measured_costs_per_mbs": costs, "best": rows[best] if best >= 0 else None, "top5": feas[:5],
       "evaluated": len(rows), "feasible": len(feas)}
print(json.dumps(out))
