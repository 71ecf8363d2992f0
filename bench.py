"""Benchmark: one Mario-scheduled training iteration of GPT-3 1.3B (BASELINE.json configs[1]:
seq 2048, GBS 128 = 32 micro-batches x mbs 4, bf16) on N B200s of one node.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--level mario]
    torchrun --nproc-per-node N bench.py --gpus N ...   (one pipeline stage per GPU, NCCL p2p)

N GPUs = N pipeline stages (1F1B; at N = 1 the plan is gradient accumulation on one GPU, pass 3
removes every checkpoint). Work per iteration is fixed (GBS 128) as N grows: "scaling": "strong".
Rank 0 prints ONE JSON line. `--impl reference` times the CPU oracle (oracle/, numpy fp32) on a
bounded sample of the same workload (the paper ships no code).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
# the emulated pipeline runs S ranks x (compute + 2 receive) streams concurrently: give every stream
# its own hardware queue (the default 8 connections alias streams and serialize independent ranks)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402

METRIC = "samples/s (GPT-3 1.3B, seq 2048, GBS 128, Mario 1F1B plan, bf16)"
UNIT = "samples/s"

# BASELINE.json configs[1..4]. The default (driver) line is cfg2; the others are
# extra lines: at 1 GPU = 1 stage every scheme is gradient accumulation (1F1B reference point, d3),
# and --emulate measures the config's own scheme at 8 stages on SM partitions of this GPU.
CONFIGS = {
    "cfg2": dict(model=lambda: synth.GPT3_1P3B, micro=32, scheme="1f1b", chunks=1, name="gpt3-1.3b",
                 workload="cfg2: GPT-3 1.3B, seq 2048, 1F1B+Mario, bf16 (BASELINE.json configs[1])"),
    "cfg3": dict(model=lambda: synth.LLAMA2_7B, micro=32, scheme="interleave", chunks=2, name="llama2-7b",
                 workload="cfg3: LLaMA2 7B, seq 4096, Interleave (2 chunks/GPU) + Mario, bf16 (BASELINE.json "
                          "configs[2])"),
    "cfg4": dict(model=lambda: synth.GPT3_2P7B, micro=32, scheme="chimera", chunks=1, name="gpt3-2.7b",
                 workload="cfg4: GPT-3 2.7B, seq 2048, Chimera + Mario, bf16 (BASELINE.json configs[3])"),
    # cfg 5 does not fit one GPU even uncapped: its 1-GPU line runs 2 of the 40 layers (+ head)
    # at s 16384 and reports the per-layer time; no 8-stage emulation (8 x up to 40 GB > one GPU's HBM)
    "cfg5": dict(model=lambda: synth.with_(synth.LLAMA2_13B, n_layers=2), micro=2, scheme="1f1b", chunks=1,
                 name="llama2-13b (2 of 40 layers)",
                 workload="cfg5 per-layer: LLaMA2 13B width, seq 16384, 2 layers + head, 1 GPU (BASELINE.json "
                          "configs[4], which needs 8 GPUs)"),
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--level", default="mario", choices=["base", "ckpt", "mario"])
    ap.add_argument("--dp", type=int, default=1,
                    help="PP x DP: gpus = stages * dp; the global batch stays --micro micro-batches (strong)")
    ap.add_argument("--scheme", default=None, help="default: the config's scheme (1F1B at 1 stage)")
    ap.add_argument("--micro", type=int, default=None, help="micro-batches per iteration (default: the config's)")
    ap.add_argument("--config", default="cfg2", choices=sorted(CONFIGS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--emulate-only", action="store_true", help="only the emulated-pipeline measurement")
    ap.add_argument("--transport", default="nccl", choices=["nccl", "peer"],
                    help="N > 1: channel transport between the rank processes (peer: CUDA IPC peer memory, "
                         "ranks may share a GPU)")
    ap.add_argument("--levels", default="",
                    help="N > 1: also time these plans (e.g. base,ckpt,mario) in the same invocation, each with "
                         "its measured bubble ratio and per-stage memory")
    ap.add_argument("--emulate-lmbs", type=int, default=0,
                    help="also measure the emulated Mario plan with this larger micro-batch at the same global "
                         "batch (the paper's lmbs configuration, P:286)")
    ap.add_argument("--emulate-levels", default="base,ckpt,mario",
                    help="plans the emulated pipeline measures (BASE of cfg3 needs more than one GPU's HBM)")
    ap.add_argument("--emulate", type=int, default=8,
                    help="N=1: also measure an S-stage pipeline of the same workload on this GPU (SM partitions, "
                         "peer transport) at BASE / CKPT / MARIO; 0 disables")
    ap.add_argument("--graphs", type=int, default=1, help="also time CUDA-graph replay (N = 1)")
    return ap.parse_args()


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


# ------------------------------------------------------------------ CPU oracle leg
def gemm_traffic(cfg):
    """DRAM bytes per GEMM launch from the committed ncu --set full capture (profiles/), next to
    the ALGORITHMIC bytes of the same four launches (one layer's forward GEMMs at this config:
    operands + outputs + residual / second output, bf16), or {}."""
    p = os.path.join(ROOT, "profiles", "r01_traffic.json")
    if not os.path.exists(p):
        return {}
    d = json.load(open(p)).get("gemm_bf16_tc2_kernel", {})
    if "dram_bytes_per_launch" not in d:
        return {}
    T, h, f = cfg.seq_len * 4, cfg.hidden, cfg.ffn_hidden      # the capture ran at mbs 4 (cfg 2)
    alg = [2 * (T * h + 3 * h * h + T * 3 * h),                 # qkv: A, W, D
           2 * (T * h + h * h + 2 * T * h),                     # proj: A, W, residual, D
           2 * (T * h + f * h + 2 * T * f),                     # fc1: A, W, Z, G = gelu(Z)
           2 * (T * f + h * f + 2 * T * h)]                     # fc2: A, W, residual, D
    return {"dram_bytes_per_launch": d["dram_bytes_per_launch"],
            "algorithmic_bytes_per_launch": sum(alg) / len(alg),
            "note": f"mean dram__bytes_read+write over {d.get('launches_captured')} captured launches "
                    f"(one layer's forward GEMMs: qkv, proj, fc1, fc2) vs the algorithmic bytes of the same four "
                    f"launches; {d.get('source', '')}"}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    import platform
    return platform.processor() or "unknown"


def cpu_oracle_sample(cfg, layers_list=(1, 2)):
    """Time the oracle (numpy fp32, all host cores) on ONE sample (mbs=1) of the workload's
    model truncated to L in layers_list layers + embedding/head, then extrapolate linearly to the
    full depth: t_sample = t(L=1) + (L_full - 1) * (t(L=2) - t(L=1))."""
    from oracle import model as om
    times = {}
    for L in layers_list:
        c = synth.with_(cfg, n_layers=L, micro_batch=1)
        P = synth.make_weights(c, parity=False)
        toks = synth.make_tokens(c, 1)
        t0 = time.perf_counter()
        om.step(c, P, toks, 1, np.float32)
        times[L] = time.perf_counter() - t0
    per_layer = max(times[2] - times[1], 1e-9)
    t_sample = times[1] + (cfg.n_layers - 1) * per_layer
    return t_sample, times


def cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


KINDS = ((0, "gemm"), (1, "attn_fwd"), (2, "attn_bwd"), (4, "norm"), (5, "colsum"), (6, "softmax_ce"),
         (7, "elementwise"), (8, "embedding"))


def run_reference(args, cfg, gbs):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    n_cores = cores()
    os.environ.setdefault("OPENBLAS_NUM_THREADS", str(n_cores))
    ts = []
    for i in range(args.warmup + args.steps):
        t, _ = cpu_oracle_sample(cfg)
        if i >= args.warmup:
            ts.append(t)
    t = statistics.median(ts)
    v = 1.0 / t
    sample = (f"1 sample (mbs 1) of {cfg.family} L=1 and L=2 (+embedding/head, s={cfg.seq_len}) fwd+bwd "
              f"fp32 per step, extrapolated to L={cfg.n_layers}; CPU: {cpu_model()}")
    out = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3 * gbs,
           "ms_per_step_extrapolated": True,
           "ms_per_step_note": "EXTRAPOLATED, not timed: the measured per-sample time (value = 1 / it) times the "
                               f"global batch {gbs}; each timed step ran one sample of the 1- and 2-layer models",
           "ms_per_sample_measured": t * 1e3,
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
           "data": "synthetic", "config": config_dict(cfg, args, gbs),
           "cpu_baseline": {"value": v, "unit": UNIT, "cores": n_cores, "kind": "oracle", "sample": sample},
           "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def config_dict(cfg, args, gbs):
    C = CONFIGS[args.config]
    return {"workload": C["workload"],
            "model": C["name"], "layers": cfg.n_layers, "hidden": cfg.hidden, "heads": cfg.n_heads,
            "global_batch": gbs, "seq_len": cfg.seq_len, "micro_batch": cfg.micro_batch,
            "microbatches": args.micro, "stages": args.gpus // args.dp, "scheme": args.scheme, "level": args.level,
            "parallelism": f"pp{args.gpus // args.dp}" + (f"xdp{args.dp}" if args.dp > 1 else ""),
            "transport": args.transport if args.gpus > 1 else "none (1 stage)",
            "l2": "no flush: every iteration streams >100 GB of weights/activations through HBM (>> 126 MB L2)"}


# ------------------------------------------------------------------- clocks sampler
class Clocks:
    def __init__(self, index):
        self.index, self.rows, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL,
                text=True)
            threading.Thread(target=self._read, daemon=True).start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()
        sm = [float(r[0]) for r in self.rows if r and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) > 1 and r[1].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            for i, n in enumerate(names):
                if len(r) > 3 + i and r[3 + i].lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------------- GPU leg
def init_weights_device(plan, rank, torch, seed=1234):
    """Random-init weights of the GPT-3 1.3B architecture directly on the device (A20 recipe:
    matrices N(0,0.02^2), residual-output matrices N(0,(0.02/sqrt(2L))^2), gamma 1, biases 0)."""
    pc, _ = plan.rank_layout(rank)
    w = torch.zeros(pc, dtype=torch.float32, device="cuda")
    g = torch.Generator(device="cuda").manual_seed(seed + rank)
    L = plan.cfg.n_layers
    for name, off, cnt in plan.rank_params(rank):
        leaf = name.split(".", 1)[-1]
        seg = w[off:off + cnt]
        if leaf.endswith(".g") or name.endswith(".g"):
            seg.fill_(1.0)
        elif leaf.endswith(".b") or name.endswith(".b"):
            seg.zero_()
        elif leaf in ("proj.w", "fc2.w", "o.w", "down.w"):
            seg.normal_(0.0, 0.02 / math.sqrt(2 * L), generator=g)
        else:
            seg.normal_(0.0, 0.02, generator=g)
    return w


def union_ms(iv):
    """Length of the union of [a, b) intervals (ms)."""
    tot, end = 0.0, None
    for a, b in sorted(iv):
        if end is None or a > end:
            tot += b - a
            end = b
        elif b > end:
            tot += b - end
            end = b
    return tot


def emulate_pipeline(cfg, api, torch, S=8, n_micro=32, steps=2, warmup=2, levels=("base", "ckpt", "mario"),
                     scheme="1f1b", chunks=1):
    """Measured S-stage pipeline on ONE GPU (mario_init_emulated): every stage is a pipeline rank on
    its own green-context SM partition (floor(148 / S) rounded down to a multiple of 8 SMs), ranks
    exchange activations / gradients through the peer transport, and the device runs the plan's
    DAG concurrently. Per plan (BASE / CKPT = plain 1F1B with full checkpointing / MARIO):
    iteration time (CUDA events on the launching stream, graph replay, median of `steps`), the
    MEASURED bubble ratio 1 - sum_d busy_d / (S * makespan) from per-rank CUDA-event timelines
    (busy_d = union of the rank's FW/CFW/RC/BW intervals), the simulator's prediction from the same
    run's per-virtual-stage costs (the paper's profile -> simulate loop) and the
    per-stage memory (static arena, exact: simulated peak vs allocated bytes). The partitions share
    HBM and L2, so absolute times are those of 1/S-th of a B200 per stage, not of S B200s."""
    sms = (device_sms(torch) // S) // 8 * 8
    gbs = n_micro * cfg.micro_batch
    pk, _ = measured_peaks()
    peak_sustained = float(pk.get("bf16_tflops_sustained", pk.get("bf16_tflops", 1400.0)))
    out = {"stages": S, "microbatches": n_micro, "scheme": scheme, "sms_per_stage": sms,
           "method": "one process, S ranks on disjoint green-context SM partitions of this GPU, peer transport; "
                     "iteration time = CUDA events around graph-replayed iterations (median); bubble from per-rank "
                     "CUDA-event timelines of one extra eager iteration", "levels": {}}
    toks = [torch.from_numpy(synth.make_tokens(cfg, n_micro, iteration=i)).cuda() for i in range(2)]
    api.close_default_context()
    for level in levels:
        plan = api.Plan(cfg, S, n_micro, scheme, level, chunks=chunks, dtype="bf16")
        ctx = api.Context.emulated(S, 0, sms)
        try:
            pc, wsb = plan.rank_layout(-2)
            w = torch.empty(pc, dtype=torch.float32, device="cuda").normal_(0.0, 0.02)
            g = torch.empty(pc, dtype=torch.float32, device="cuda")
            ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
            stream = torch.cuda.current_stream()
            ctx.set_graphs(True)
            for i in range(max(warmup, 2)):
                ctx.run_iter(plan, w, toks[i % 2], g, ws, stream)
            torch.cuda.synchronize()
            ts = []
            for i in range(steps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                loss = ctx.run_iter(plan, w, toks[i % 2], g, ws, stream)
                e1.record(stream)
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ctx.set_graphs(False)
            ctx.set_timing(True)
            ctx.run_iter(plan, w, toks[0], g, ws, stream)
            torch.cuda.synchronize()
            ctx.set_timing(False)
            tl = [ctx.last_timeline(d) for d in range(S)]
            ms = statistics.median(ts)
            span = max(max(b) for a, b in tl if b)
            busy = [union_ms(list(zip(a, b))) for a, b in tl]
            # per-virtual-stage costs of this run -> the simulator (P:242 profile, P:244-252 simulate)
            costs = ctx.last_costs(plan)
            sim = api.Plan(cfg, S, n_micro, scheme, level, chunks=chunks, dtype="bf16", costs=costs).simulate()
            alloc = [plan.rank_layout(d)[1] + 8 * plan.rank_layout(d)[0] for d in range(S)]
            peaks = plan.simulate().peak_bytes
            p_lin = (12 * cfg.hidden ** 2 if cfg.family == "gpt"
                     else 4 * cfg.hidden ** 2 + 3 * cfg.hidden * cfg.ffn_hidden)
            mflops = 3.0 * (cfg.n_layers * (2 * cfg.seq_len * p_lin + 4 * cfg.seq_len ** 2 * cfg.hidden)
                            + 2 * cfg.seq_len * cfg.hidden * cfg.vocab) * gbs
            tf_stage = mflops / (ms / 1e3) / S / 1e12
            out["levels"][level] = {
                "ms_per_iter": ms, "samples_per_s": gbs / (ms / 1e3), "loss": loss,
                "model_tflops_per_stage": tf_stage,
                "model_tflops_per_stage_frac_of_partition_peak": tf_stage / (peak_sustained * sms / device_sms(torch)),
                "bubble_measured": 1.0 - sum(busy) / (S * span),
                "bubble_simulated": sim.bubble_ratio,
                "makespan_measured_ms": span, "makespan_simulated_ms": sim.makespan_ms,
                "busy_ms_per_stage": [round(b, 2) for b in busy],
                "stage_ms": {k: [round(x, 3) for x in costs[k]] for k in ("fw_ms", "bw_ms", "rc_ms")},
                "peak_gb_per_stage_simulated": [round(b / 1e9, 3) for b in peaks],
                "alloc_gb_per_stage": [round(b / 1e9, 3) for b in alloc],
                "peak_balance_max_over_min": max(peaks) / min(peaks)}
            del w, g, ws
        finally:
            ctx.close()
            torch.cuda.empty_cache()
    lv = out["levels"]
    if "ckpt" in lv and "mario" in lv:
        out["mario_vs_ckpt"] = lv["ckpt"]["ms_per_iter"] / lv["mario"]["ms_per_iter"]
    if "base" in lv and "mario" in lv:
        out["mario_vs_base"] = lv["base"]["ms_per_iter"] / lv["mario"]["ms_per_iter"]
    return out


def allmax(x, cpu_group, torch, dist):
    """Max over ranks (gloo process groups reduce host tensors, NCCL device tensors)."""
    t = torch.tensor([float(x)], device="cpu" if cpu_group else "cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def multi_level(args, cfg, api, torch, dist, S, n_rep, scheme, chunks, rank, world, local, peer, stage, gbs):
    """N > 1: BASE / CKPT / MARIO (--levels) timed in one invocation on the real multi-process
    pipeline: per plan the iteration time (CUDA events, max over ranks), the measured bubble ratio
    1 - sum_d busy_d / (S * t_iter) (busy_d = union of rank d's FW/CFW/RC/BW event intervals, SURVEY
    §8(d) d3), the simulator's bubble from the ranks' own measured stage costs, and the
    per-stage memory (static arena = simulated peak)."""
    out = {}
    for level in [x for x in args.levels.split(",") if x]:
        plan = api.Plan(cfg, S, n_rep, scheme, level, chunks=chunks, dtype="bf16")
        ctx = api.Context.peer(rank, world, local) if peer else api.Context(rank, world, local, dp=args.dp)
        try:
            w = init_weights_device(plan, stage, torch)
            pc, wsb = plan.rank_layout(stage)
            g = torch.zeros(pc, dtype=torch.float32, device="cuda")
            ws = torch.empty(wsb, dtype=torch.uint8, device="cuda")
            if peer:
                ctx.bind(ws, g)
            toks = [torch.from_numpy(synth.make_tokens(cfg, n_rep, iteration=i)).cuda() for i in range(2)]
            stream = torch.cuda.current_stream()
            for i in range(max(2, args.warmup)):
                ctx.run_iter(plan, w, toks[i % 2], g, ws, stream)
            torch.cuda.synchronize()
            dist.barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for i in range(args.steps):
                ctx.run_iter(plan, w, toks[i % 2], g, ws, stream)
            e1.record(stream)
            torch.cuda.synchronize()
            ms = allmax(e0.elapsed_time(e1) / args.steps, peer, torch, dist)
            ctx.set_timing(True)
            dist.barrier()
            e0.record(stream)
            ctx.run_iter(plan, w, toks[0], g, ws, stream)
            e1.record(stream)
            torch.cuda.synchronize()
            ctx.set_timing(False)
            t_it = allmax(e0.elapsed_time(e1), peer, torch, dist)
            a, b = ctx.last_timeline(stage)
            busy = union_ms(list(zip(a, b)))
            c = ctx.last_costs(plan)
            rows = [None] * world
            dist.all_gather_object(rows, (stage, busy, c))
            if rank == 0:
                K = len(c["fw_ms"])
                merged = {k: [0.0] * K for k in ("fw_ms", "bw_ms", "rc_ms")}
                for _st, _b, cc in rows:
                    for k in merged:
                        for i, v in enumerate(cc[k]):
                            merged[k][i] = max(merged[k][i], v)
                merged.update(p2p_alpha_ms=0.005, p2p_GBps=770.0)
                sim = api.Plan(cfg, S, n_rep, scheme, level, chunks=chunks, dtype="bf16", costs=merged).simulate()
                busy_all = [r[1] for r in sorted(rows)]
                peaks = plan.simulate().peak_bytes
                out[level] = {"ms_per_iter": ms, "samples_per_s": gbs / (ms / 1e3),
                              "bubble_measured": 1.0 - sum(busy_all) / (S * t_it),
                              "bubble_simulated": sim.bubble_ratio, "makespan_simulated_ms": sim.makespan_ms,
                              "timed_iteration_ms": t_it, "busy_ms_per_stage": [round(x, 2) for x in busy_all],
                              "peak_gb_per_stage_simulated": [round(x / 1e9, 3) for x in peaks],
                              "peak_balance_max_over_min": max(peaks) / min(peaks)}
            del w, g, ws
        finally:
            torch.cuda.synchronize()
            dist.barrier()
            ctx.close()
            torch.cuda.empty_cache()
    if rank == 0 and "ckpt" in out and "mario" in out:
        out["mario_vs_ckpt"] = out["ckpt"]["ms_per_iter"] / out["mario"]["ms_per_iter"]
    return out


def device_sms(torch):
    return torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count


def main():
    args = parse()
    CE = CONFIGS[args.config]
    cfg = CE["model"]()
    if args.micro is None:
        args.micro = CE["micro"]
    gbs = args.micro * cfg.micro_batch
    if args.impl == "reference":
        run_reference(args, cfg, gbs)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_liultj25_b200 import _lib, api
    if args.emulate_only:
        torch.cuda.set_device(0)
        levels = tuple(args.emulate_levels.split(","))
        res = {"pipeline_emulated": emulate_pipeline(cfg, api, torch, S=args.emulate, n_micro=args.micro,
                                                     steps=max(1, min(args.steps, 3)), warmup=2,
                                                     levels=levels, scheme=args.scheme or CE["scheme"],
                                                     chunks=CE["chunks"])}
        if args.emulate_lmbs:
            lm = args.emulate_lmbs
            res["pipeline_emulated_lmbs"] = emulate_pipeline(
                synth.with_(cfg, micro_batch=lm), api, torch, S=args.emulate, n_micro=gbs // lm,
                steps=max(1, min(args.steps, 3)), warmup=2, levels=("mario",), scheme=args.scheme or CE["scheme"],
                chunks=CE["chunks"])
            res["pipeline_emulated_lmbs"]["micro_batch"] = lm
        print(json.dumps(res), flush=True)
        return

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    assert world == args.gpus, f"--gpus {args.gpus} but WORLD_SIZE {world}"
    peer = world > 1 and args.transport == "peer"
    if peer:
        local = local % torch.cuda.device_count()   # ranks may share a GPU (CUDA IPC)
    torch.cuda.set_device(local)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        if peer:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    L = _lib.lib()
    assert world % args.dp == 0 and args.micro % args.dp == 0, "--dp must divide --gpus and --micro"
    S, rep, n_rep = world // args.dp, rank // (world // args.dp), args.micro // args.dp
    stage = rank % S
    scheme = args.scheme or (CE["scheme"] if S > 1 else "1f1b")
    chunks = CE["chunks"] if scheme == "interleave" else 1
    args.scheme = scheme
    plan = api.Plan(cfg, S, n_rep, scheme, args.level, chunks=chunks, dtype="bf16")
    assert not peer or args.dp == 1, "--transport peer runs pure pipeline parallelism"
    ctx = api.Context.peer(rank, world, local) if peer else api.Context(rank, world, local, dp=args.dp)
    w = init_weights_device(plan, stage, torch)          # replicas of a stage hold identical weights
    pc, ws_bytes = plan.rank_layout(stage)
    grads = torch.zeros(pc, dtype=torch.float32, device="cuda")
    ws = torch.empty(ws_bytes, dtype=torch.uint8, device="cuda")
    if peer:
        ctx.bind(ws, grads)
    stream = torch.cuda.current_stream()
    tok_host = [synth.make_tokens(cfg, n_rep, iteration=i * args.dp + rep) for i in range(args.warmup + args.steps)]
    tok_dev = [torch.from_numpy(t).cuda() for t in tok_host]
    torch.cuda.synchronize()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    # Headline region: the public call with CUDA-graph replay of the iteration (mario_set_graphs;
    # single process: the first warm-up call runs eager, the second captures). The GEMMs are
    # event-timed inside the captured graph (the events re-record on every replay), so the
    # roofline is measured live in the same region. Multi-process runs are eager (NCCL p2p).
    use_graphs = world == 1 and args.graphs and args.warmup >= 2
    L.mario_kstats_enable(1)      # GEMM only (2 event records per launch)
    ctx.set_graphs(bool(use_graphs))
    for i in range(args.warmup):
        ctx.run_iter(plan, w, tok_dev[i], grads, ws, stream)
    barrier()
    clocks = Clocks(local)
    clocks.start()
    launches0 = L.mario_kernel_launches()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    losses = []
    barrier()
    e0.record(stream)
    for i in range(args.steps):
        losses.append(ctx.run_iter(plan, w, tok_dev[args.warmup + i], grads, ws, stream))
    e1.record(stream)
    torch.cuda.synchronize()
    ms_total = e0.elapsed_time(e1)
    launches = L.mario_kernel_launches() - launches0
    clk = clocks.stop()
    import ctypes as C

    def read_kinds():
        out = {}
        for kind, name in KINDS:
            ms, fl, by, n = C.c_double(), C.c_double(), C.c_double(), C.c_longlong()
            L.mario_kstats_read(kind, C.byref(ms), C.byref(fl), C.byref(by), C.byref(n))
            out[name] = {"ms": ms.value, "flops": fl.value, "bytes": by.value, "launches": n.value}
        return out
    kst = read_kinds()
    kst_steps = 1 if use_graphs else args.steps      # graph records hold the latest replay only
    L.mario_kstats_enable(0)
    if world > 1:
        ms_total = allmax(ms_total, peer, torch, dist)
    ms_step = ms_total / args.steps
    value = gbs / (ms_step / 1e3)

    # end-to-end through the same public call with pinned host tokens (H2D inside) and host loss (D2H)
    e2e = None
    if not args.no_e2e:
        pinned = [torch.from_numpy(t).pin_memory() for t in tok_host[-args.steps:]]
        barrier()
        t0 = time.perf_counter()
        for i in range(args.steps):
            ctx.run_iter(plan, w, pinned[i], grads, ws, stream)
        torch.cuda.synchronize()
        dt = (time.perf_counter() - t0) / args.steps
        if world > 1:
            dt = allmax(dt, peer, torch, dist)
        e2e = {"value": gbs / dt, "unit": UNIT, "h2d_bytes_per_step": int(tok_host[0].nbytes),
               "d2h_bytes_per_step": 4 + 8 * n_rep, "graphs": bool(use_graphs)}

    # the same iteration without graph replay (every kernel launched from the host), for reference
    eager = None
    if use_graphs:
        ctx.set_graphs(False)
        ctx.run_iter(plan, w, tok_dev[0], grads, ws, stream)
        torch.cuda.synchronize()
        e0.record(stream)
        for i in range(args.steps):
            ctx.run_iter(plan, w, tok_dev[args.warmup + i], grads, ws, stream)
        e1.record(stream)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1) / args.steps
        eager = {"value": gbs / (ems / 1e3), "ms_per_step": ems}

    # per-family breakdown: one extra step with every kernel timed (outside the headline region)
    L.mario_kstats_enable(-1)
    e0.record(stream)
    ctx.run_iter(plan, w, tok_dev[-1], grads, ws, stream)
    e1.record(stream)
    torch.cuda.synchronize()
    breakdown_ms = e0.elapsed_time(e1)
    kall = read_kinds()
    L.mario_kstats_enable(0)

    sim = plan.simulate()
    peaks, peak_kind = measured_peaks()
    traffic = gemm_traffic(cfg) if args.config == "cfg2" else {}
    g = kst["gemm"]
    achieved = g["flops"] / (g["ms"] / 1e3) / 1e12 if g["ms"] > 0 else 0.0
    peak = float(peaks.get("bf16_tflops_sustained", peaks.get("bf16_tflops")))
    p_lin = 12 * cfg.hidden ** 2 if cfg.family == "gpt" else 4 * cfg.hidden ** 2 + 3 * cfg.hidden * cfg.ffn_hidden
    model_flops = 3.0 * (cfg.n_layers * (2 * cfg.seq_len * p_lin + 4 * cfg.seq_len ** 2 * cfg.hidden)
                         + 2 * cfg.seq_len * cfg.hidden * cfg.vocab)
    tflops_gpu = model_flops * gbs / (ms_step / 1e3) / world / 1e12
    # whole-step algorithmic roofline: the FLOPs the method must execute (causal
    # attention; + Mario's recompute when stages > 1) over the step time and the dense bf16 peak
    S_ = world // args.dp
    layer_f = 2 * cfg.seq_len * p_lin + 2 * cfg.seq_len ** 2 * cfg.hidden
    alg_flops = 3.0 * (cfg.n_layers * layer_f + 2 * cfg.seq_len * cfg.hidden * cfg.vocab) * gbs
    if S_ > 1 and args.level != "base":
        alg_flops += (S_ - 1) * (cfg.n_layers // S_) * layer_f * gbs   # RC of every checkpointed stage
    alg_tflops = alg_flops / (ms_step / 1e3) / world / 1e12
    mem = torch.cuda.max_memory_allocated()
    metric = METRIC if args.config == "cfg2" else (f"samples/s ({CE['name']}, seq {cfg.seq_len}, GBS {gbs}, "
                                                   f"Mario plan, bf16)")
    out = {"metric": metric, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
           "vs_baseline": None, "dtype": "bf16", "data": "synthetic (uniform tokens, random-init weights)",
           "config": config_dict(cfg, args, gbs),
           "model_tflops_per_gpu": tflops_gpu,
           "whole_step_roofline": {"algorithmic_tflops_per_gpu": alg_tflops,
                                   "frac_of_2250_datasheet": alg_tflops / 2250.0,
                                   "frac_of_measured_sustained": alg_tflops / peak,
                                   # the peak at the SM clock the run saw (148 SMs x 8192 dense
                                   # bf16 FLOP/clk x f_SM, NVML median under load)
                                   "clock_limited_peak_tflops": (device_sms(torch) * 8192 * clk["sm_mhz"] * 1e6 / 1e12
                                                                 if clk.get("sm_mhz") else None),
                                   "frac_of_clock_limited_peak": (alg_tflops / (device_sms(torch) * 8192 * clk["sm_mhz"] * 1e6 / 1e12)
                                                                  if clk.get("sm_mhz") else None),
                                   "flops_per_step": alg_flops,
                                   "note": "causal attention FLOPs (2 s^2 h per layer-sample fwd), no RC at 1 stage"},
           "loss": losses[-1],
           "roofline": {"bound": "tensor", "kernel": "gemm_bf16_tc_kernel (tcgen05, all linear layers)",
                        "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                        "peak_source": f"{peak_kind} bf16_tflops_sustained (MEASURED_PEAKS.json)",
                        "traffic": traffic.get("dram_bytes_per_launch"),
                        "traffic_note": traffic.get("note"),
                        "algorithmic_bytes_per_launch": traffic.get("algorithmic_bytes_per_launch"),
                        "algorithmic_bytes_per_launch_all_gemms": (g["bytes"] / g["launches"]) if g["launches"] else None,
                        "launches_per_step": g["launches"] / kst_steps,
                        "measured_in": "graph replay (latest step)" if use_graphs else "eager steps",
                        "share_of_step": (g["ms"] / kst_steps) / ms_step if ms_step > 0 else None},
           "kernels": {"note": "one extra step with every launch event-timed (not the headline region)",
                       "step_ms": breakdown_ms,
                       **{k: {"ms": v["ms"], "tflops": (v["flops"] / (v["ms"] / 1e3) / 1e12) if v["ms"] > 0 and
                              v["flops"] > 0 else None, "launches": v["launches"]} for k, v in kall.items()}},
           "gpu_launches": int(launches),
           "clocks": clk,
           "bubble": {"simulated": sim.bubble_ratio, "stages": S},
           "peak_mem_per_stage": {"simulated_bytes": sim.peak_bytes,
                                  "measured_torch_max_allocated": int(mem)},
           "execution": "cuda-graph replay" if use_graphs else "eager",
           "e2e": e2e, "eager": eager}
    ctx.close()
    if world > 1 and args.levels:
        del w, grads, ws
        torch.cuda.empty_cache()
        lv = multi_level(args, cfg, api, torch, dist, S, n_rep, scheme, chunks, rank, world, local, peer, stage, gbs)
        if rank == 0:
            out["levels"] = lv
    # the extra measurements never cost the headline line: a failure is recorded, not raised
    if rank == 0 and world == 1 and args.emulate > 1 and args.config != "cfg5" and args.emulate_lmbs:
        lm = args.emulate_lmbs
        try:
            out["pipeline_emulated_lmbs"] = emulate_pipeline(
                synth.with_(cfg, micro_batch=lm), api, torch, S=args.emulate, n_micro=gbs // lm,
                steps=max(1, min(args.steps, 3)), warmup=2, levels=("mario",), scheme=CE["scheme"],
                chunks=CE["chunks"])
            out["pipeline_emulated_lmbs"]["micro_batch"] = lm
        except Exception as e:   # noqa: BLE001
            out["pipeline_emulated_lmbs"] = {"error": repr(e)[:300]}
    if rank == 0 and world == 1 and args.emulate > 1 and args.config != "cfg5":
        try:
            out["pipeline_emulated"] = emulate_pipeline(cfg, api, torch, S=args.emulate, n_micro=args.micro,
                                                        scheme=CE["scheme"], chunks=CE["chunks"],
                                                        levels=tuple(args.emulate_levels.split(",")),
                                                        steps=max(1, min(args.steps, 3)), warmup=2)
        except Exception as e:   # noqa: BLE001
            out["pipeline_emulated"] = {"error": repr(e)[:300]}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        n_cores = cores()
        os.environ.setdefault("OPENBLAS_NUM_THREADS", str(n_cores))
        t, times = cpu_oracle_sample(cfg)
        out["cpu_baseline"] = {"value": 1.0 / t, "unit": UNIT, "cores": n_cores, "kind": "oracle",
                               "cpu_model": cpu_model(),
                               "sample": f"1 sample (mbs 1), fp32 numpy oracle, L=1 ({times[1]:.2f}s) and L=2 "
                                         f"({times[2]:.2f}s) + embedding/head at s=2048, extrapolated to 24 layers"}
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
