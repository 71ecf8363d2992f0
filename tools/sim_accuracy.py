"""Simulator accuracy (§6.6) on ONE B200.

For single-device plans (S = 1) of several model sizes, micro-batch sizes and sequence lengths:
  memory  — the planner's simulated peak (static + activation walk) against the measured
            device memory the iteration occupies (cudaMemGetInfo delta after CUDA-context creation:
            weights, grads, workspace and whatever the library allocates itself);
  time    — the makespan the simulator predicts from per-instruction costs profiled with CUDA events
            in one run against the iteration time measured in separate, un-instrumented runs.
Also writes a Chrome trace (simulated vs measured) of an 8-stage loopback plan.

What this cannot check on one GPU: the p2p terms and the cross-device overlap of a real pipeline
(the 8-GPU projection in bench.py stays unvalidated). Output: JSON lines + gpurun_out/ files."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_ppopp_liultj25_b200 import api  # noqa: E402

OUT = os.environ.get("SIMACC_OUT", "gpurun_out")
CONFIGS = [
    ("gpt3-1.3b mbs1 s2048", synth.with_(synth.GPT3_1P3B, micro_batch=1), 8),
    ("gpt3-1.3b mbs2 s2048", synth.with_(synth.GPT3_1P3B, micro_batch=2), 8),
    ("gpt3-1.3b mbs4 s2048", synth.GPT3_1P3B, 8),
    ("gpt3-1.3b mbs1 s4096", synth.with_(synth.GPT3_1P3B, micro_batch=1, seq_len=4096), 8),
    ("gpt3-2.7b mbs1 s2048", synth.GPT3_2P7B, 8),
    ("llama2-7b L16 mbs1 s4096", synth.with_(synth.LLAMA2_7B, n_layers=16), 4),
]


def used_bytes():
    free, total = torch.cuda.mem_get_info()
    return total - free


def one(name, cfg, N, ctx):
    plan = api.Plan(cfg, 1, N, "1f1b", "mario", dtype="bf16")
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    u0 = used_bytes()
    w, g, ws = api.alloc_for(plan, 0)
    w.normal_(0.0, 0.02)
    tok = torch.from_numpy(synth.make_tokens(cfg, N)).cuda()
    ctx.run_iter(plan, w, tok, g, ws)
    torch.cuda.synchronize()
    mem_meas = used_bytes() - u0
    # measured iteration time (no per-instruction events)
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    times = []
    for _ in range(3):
        e0.record()
        ctx.run_iter(plan, w, tok, g, ws)
        e1.record()
        torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1))
    t_meas = sorted(times)[1]
    # profile per-instruction costs, then simulate with them
    ctx.set_timing(True)
    ctx.run_iter(plan, w, tok, g, ws)
    ctx.set_timing(False)
    a, b = ctx.last_timeline(0)
    comp = [x for x in plan.instrs(0) if x[0] in ("FW", "CFW", "RC", "BW")]
    fw = [t1 - t0 for (op, *_r), t0, t1 in zip(comp, a, b) if op in ("FW", "CFW")]
    bw = [t1 - t0 for (op, *_r), t0, t1 in zip(comp, a, b) if op == "BW"]
    mean = lambda xs: sum(xs) / len(xs)
    costs = {"fw_ms": [mean(fw)], "bw_ms": [mean(bw)], "rc_ms": [mean(fw)], "p2p_alpha_ms": 0.0, "p2p_GBps": 0.0}
    sim = api.Plan(cfg, 1, N, "1f1b", "mario", dtype="bf16", costs=costs).simulate()
    mem_sim = plan.simulate().peak_bytes[0]
    rec = {"config": name, "microbatches": N, "mem_sim_gb": round(mem_sim / 1e9, 3), "mem_meas_gb": round(mem_meas / 1e9, 3),
           "mem_ape": round(abs(mem_sim - mem_meas) / mem_meas, 4), "t_sim_ms": round(sim.makespan_ms, 2),
           "t_meas_ms": round(t_meas, 2), "t_ape": round(abs(sim.makespan_ms - t_meas) / t_meas, 4)}
    del w, g, ws, tok
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    return rec


def main():
    os.makedirs(OUT, exist_ok=True)
    torch.cuda.set_device(0)
    torch.cuda.init()
    ctx = api.Context(0, 1, 0)
    recs = []
    for name, cfg, N in CONFIGS:
        r = one(name, cfg, N, ctx)
        print(json.dumps(r), flush=True)
        recs.append(r)
    summ = {"memory_mape": round(sum(r["mem_ape"] for r in recs) / len(recs), 4),
            "time_mape": round(sum(r["t_ape"] for r in recs) / len(recs), 4),
            "paper": {"memory_mape": 0.051, "time_mape": 0.094, "ref": "P:385-387, 8 x A100-40G, GPT3-1.6B"}}
    print(json.dumps(summ), flush=True)
    # Chrome trace: 8-stage loopback plan of GPT-3 1.3B (12 layers, 8 micro-batches), simulated with
    # the profiled costs next to the measured (serialised on one GPU) timeline
    cfg = synth.with_(synth.GPT3_1P3B, n_layers=16, micro_batch=1)
    prof = api.Plan(cfg, 8, 8, "1f1b", "mario", dtype="bf16")
    w, g, ws = api.alloc_for(prof, -1)
    w.normal_(0.0, 0.02)
    tok = torch.from_numpy(synth.make_tokens(cfg, 8)).cuda()
    ctx.run_iter(prof, w, tok, g, ws)
    ctx.set_timing(True)
    ctx.run_iter(prof, w, tok, g, ws)
    ctx.set_timing(False)
    measured = [ctx.last_timeline(d) for d in range(8)]
    with open(os.path.join(OUT, "sim_vs_measured_trace.json"), "w") as f:
        json.dump(api.chrome_trace(prof, measured), f)
    with open(os.path.join(OUT, "sim_accuracy.json"), "w") as f:
        json.dump({"configs": recs, "summary": summ}, f, indent=1)


if __name__ == "__main__":
    main()
