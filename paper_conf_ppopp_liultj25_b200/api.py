"""Thin Python binding over libmario.so (include/mario.h). Argument marshalling only:
planning, simulation and every step of the training iteration run inside the library.

    plan = Plan(model, stages=8, microbatches=32, scheme="1f1b", level="mario")
    ctx  = Context(rank, world, device)            # NCCL / loopback executor
    loss = ctx.run_iter(plan, weights, tokens, grads, workspace)
"""
from __future__ import annotations

import ctypes as C
from dataclasses import replace, dataclass
from typing import Dict, List, Optional, Sequence, Tuple

from . import _lib

SCHEMES = {"1f1b": 0, "v": 0, "interleave": 1, "w": 1, "chimera": 2, "x": 2}
LEVELS = {"base": 0, "ckpt": 1, "mario": 2, "ovlp": 2, "mario_budget": 3}
OPS = ["FW", "CFW", "RC", "BW", "SA", "RA", "SG", "RG"]
STATUS = {0: "OK", -1: "EINVAL", -2: "EBUDGET", -3: "EDEADLOCK", -4: "ECUDA", -5: "ENCCL", -6: "ESTATE"}


class MarioError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code


class CModel(C.Structure):
    _fields_ = [("family", C.c_int32), ("n_layers", C.c_int32), ("hidden", C.c_int32), ("n_heads", C.c_int32),
                ("ffn_hidden", C.c_int32), ("vocab", C.c_int32), ("seq_len", C.c_int32),
                ("micro_batch", C.c_int32), ("tie_embeddings", C.c_int32), ("dtype", C.c_int32),
                ("norm_eps", C.c_float), ("rope_base", C.c_float)]


class CInstr(C.Structure):
    _fields_ = [("op", C.c_int32), ("micro", C.c_int32), ("part", C.c_int32), ("vstage", C.c_int32),
                ("peer", C.c_int32), ("slot", C.c_int32), ("aslot", C.c_int32)]


class CCosts(C.Structure):
    _fields_ = [("fw_ms", C.POINTER(C.c_double)), ("bw_ms", C.POINTER(C.c_double)), ("rc_ms", C.POINTER(C.c_double)),
                ("p2p_alpha_ms", C.c_double), ("p2p_GBps", C.c_double),
                ("act_bytes", C.POINTER(C.c_double)), ("ckpt_bytes", C.POINTER(C.c_double)),
                ("work_bytes", C.POINTER(C.c_double)), ("static_bytes", C.c_double)]


class CCommOp(C.Structure):
    _fields_ = [("kind", C.c_int32), ("a", C.c_int32), ("b", C.c_int32), ("c", C.c_int32), ("micro", C.c_int32),
                ("part", C.c_int32), ("list_index", C.c_int32), ("count", C.c_int64)]


class CSim(C.Structure):
    _fields_ = [("makespan_ms", C.c_double), ("bubble_ratio", C.c_double), ("n_dev", C.c_int32),
                ("busy_ms", C.POINTER(C.c_double)), ("peak_bytes", C.POINTER(C.c_uint64)),
                ("max_live_act", C.POINTER(C.c_int32)), ("max_live_ckpt", C.POINTER(C.c_int32))]


class CTuneCosts(C.Structure):
    _fields_ = [("n_mbs", C.c_int32), ("mbs", C.POINTER(C.c_int32)), ("layer_fw_ms", C.POINTER(C.c_double)),
                ("layer_bw_ms", C.POINTER(C.c_double)), ("head_fw_ms", C.POINTER(C.c_double)),
                ("head_bw_ms", C.POINTER(C.c_double)), ("p2p_alpha_ms", C.c_double), ("p2p_GBps", C.c_double),
                ("dp_efficiency", C.c_double)]


class CTuneResult(C.Structure):
    _fields_ = [("scheme", C.c_int32), ("pp", C.c_int32), ("chunks", C.c_int32), ("dp", C.c_int32),
                ("micro_batch", C.c_int32), ("microbatches", C.c_int32), ("level", C.c_int32),
                ("feasible", C.c_int32), ("makespan_ms", C.c_double), ("samples_per_s", C.c_double),
                ("bubble_ratio", C.c_double), ("peak_bytes", C.c_uint64)]


_P = C.c_void_p
_lib.register("mario_plan", C.c_int32, [C.POINTER(CModel), C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_uint64,
                                        C.c_int32, C.POINTER(CCosts), C.POINTER(_P)])
_lib.register("mario_plan_instrs", C.c_int32, [_P, C.c_int32, C.POINTER(C.POINTER(CInstr)), C.POINTER(C.c_int32)])
_lib.register("mario_plan_simulate", C.c_int32, [_P, C.POINTER(CSim)])
_lib.register("mario_plan_timeline", C.c_int32, [_P, C.c_int32, C.POINTER(C.POINTER(C.c_double)),
                                                 C.POINTER(C.POINTER(C.c_double)), C.POINTER(C.c_int32)])
_lib.register("mario_plan_comm_ops_dp", C.c_int32, [_P, C.c_int32, C.c_int32, C.POINTER(C.POINTER(CCommOp)),
                                                    C.POINTER(C.c_int32)])
_lib.register("mario_plan_comm_ops", C.c_int32, [_P, C.c_int32, C.POINTER(C.POINTER(CCommOp)), C.POINTER(C.c_int32)])
_lib.register("mario_plan_serialize", C.c_int32, [_P, C.c_char_p, C.c_size_t, C.POINTER(C.c_size_t)])
_lib.register("mario_plan_rank_layout", C.c_int32, [_P, C.c_int32, C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)])
_lib.register("mario_plan_rank_params", C.c_int32, [_P, C.c_int32, C.POINTER(C.POINTER(C.c_int32)),
                                                    C.POINTER(C.POINTER(C.c_uint64)),
                                                    C.POINTER(C.POINTER(C.c_uint64)), C.POINTER(C.c_int32)])
_lib.register("mario_param_name", C.c_char_p, [_P, C.c_int32])
_lib.register("mario_param_count", C.c_int32, [_P])
_lib.register("mario_param_shape", C.c_int32, [_P, C.c_int32, C.POINTER(C.c_int64), C.POINTER(C.c_int32)])
_lib.register("mario_plan_destroy", None, [_P])
_lib.register("mario_plan_unckpt_tail", C.c_int32, [_P])
_lib.register("mario_plan_store_act", C.c_int32, [_P])
_lib.register("mario_last_error", C.c_char_p, [])
_lib.register("mario_tune", C.c_int32, [C.POINTER(CModel), C.c_int32, C.c_int32, C.c_uint64, C.POINTER(CTuneCosts),
                                        C.POINTER(CTuneResult), C.c_int32, C.POINTER(C.c_int32), C.POINTER(C.c_int32)])
_lib.register("mario_nccl_unique_id", C.c_int32, [C.c_void_p])
_lib.register("mario_init", C.c_int32, [C.c_int32, C.c_int32, C.c_int32, C.c_void_p])
_lib.register("mario_init_dp", C.c_int32, [C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_void_p])
_lib.register("mario_init_emulated", C.c_int32, [C.c_int32, C.c_int32, C.c_int32])
_lib.register("mario_emulated_sms", C.c_int32, [])
_lib.register("mario_init_peer", C.c_int32, [C.c_int32, C.c_int32, C.c_int32])
_lib.register("mario_peer_export", C.c_int32, [C.c_void_p, C.c_void_p, C.c_void_p])
_lib.register("mario_peer_import", C.c_int32, [C.c_void_p])
_lib.register("mario_run_iter", C.c_int32, [_P, C.c_void_p, C.c_void_p, C.POINTER(C.c_float), C.c_void_p,
                                            C.c_void_p, C.c_void_p])
_lib.register("mario_set_timing", C.c_int32, [C.c_int32])
_lib.register("mario_set_graphs", C.c_int32, [C.c_int32])
_lib.register("mario_last_timeline", C.c_int32, [C.c_int32, C.POINTER(C.POINTER(C.c_double)),
                                                 C.POINTER(C.POINTER(C.c_double)), C.POINTER(C.c_int32)])
_lib.register("mario_finalize", C.c_int32, [])
_lib.register("mario_last_costs", C.c_int32, [_P, C.POINTER(C.c_double), C.POINTER(C.c_double),
                                              C.POINTER(C.c_double)])
_lib.register("mario_adamw_step", C.c_int32, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_uint64, C.c_float,
                                              C.c_float, C.c_float, C.c_float, C.c_float, C.c_int32, C.c_void_p])


def _check(code):
    if code != 0:
        raise MarioError(code, (_lib.lib().mario_last_error() or b"").decode())


def cmodel(cfg, dtype: str = "bf16") -> CModel:
    """synth.ModelCfg (or any object with the same fields) -> mario_model."""
    return CModel(0 if cfg.family == "gpt" else 1, cfg.n_layers, cfg.hidden, cfg.n_heads, cfg.ffn_hidden,
                  cfg.vocab, cfg.seq_len, cfg.micro_batch, int(cfg.tie_embeddings),
                  1 if dtype == "bf16" else 0, cfg.norm_eps, cfg.rope_base)


def _darr(xs):
    if xs is None:
        return None
    return (C.c_double * len(xs))(*xs)


@dataclass
class SimReport:
    makespan_ms: float
    bubble_ratio: float
    busy_ms: List[float]
    peak_bytes: List[int]
    max_live_act: List[int]
    max_live_ckpt: List[int]


class Plan:
    """mario_plan(model, stages, microbatches, scheme, mem_budget) (north_star)."""

    def __init__(self, cfg, stages: int, microbatches: int, scheme: str = "1f1b", level: str = "mario",
                 chunks: int = 1, mem_budget: int = 0, dtype: str = "bf16", costs: Optional[dict] = None):
        L = _lib.lib()
        self.cfg, self.dtype = cfg, dtype
        self.S, self.N, self.scheme, self.level, self.chunks = stages, microbatches, scheme, level, chunks
        self._m = cmodel(cfg, dtype)
        cc = None
        if costs is not None:
            self._keep = [_darr(costs.get(k)) for k in ("fw_ms", "bw_ms", "rc_ms", "act_bytes", "ckpt_bytes",
                                                        "work_bytes")]
            cc = CCosts(self._keep[0], self._keep[1], self._keep[2], costs.get("p2p_alpha_ms", 0.0),
                        costs.get("p2p_GBps", 0.0), self._keep[3], self._keep[4], self._keep[5],
                        costs.get("static_bytes", -1.0))
        h = _P()
        _check(L.mario_plan(C.byref(self._m), stages, microbatches, SCHEMES[scheme], chunks, mem_budget,
                            LEVELS[level], C.byref(cc) if cc is not None else None, C.byref(h)))
        self.handle = h

    def __del__(self):
        h = getattr(self, "handle", None)
        try:
            if h and _lib is not None and _lib._lib is not None:
                _lib._lib.mario_plan_destroy(h)
        except Exception:
            pass
        self.handle = None

    @property
    def _as_param(self):
        return self.handle

    def instrs(self, d: int) -> List[Tuple]:
        p = C.POINTER(CInstr)()
        n = C.c_int32()
        _check(_lib.lib().mario_plan_instrs(self.handle, d, C.byref(p), C.byref(n)))
        return [(OPS[p[i].op], p[i].micro, p[i].part, p[i].vstage, p[i].peer, p[i].slot, p[i].aslot)
                for i in range(n.value)]

    @property
    def unckpt_tail(self) -> int:
        """MARIO_LEVEL_BUDGET: how many tail devices keep full activations (reading A28)."""
        return int(_lib.lib().mario_plan_unckpt_tail(self.handle))

    @property
    def store_act(self) -> bool:
        """Activation sets keep the norm outputs and the MLP activation (else the lean set: the backward
        recomputes them)."""
        return bool(_lib.lib().mario_plan_store_act(self.handle))

    def lists(self) -> List[List[Tuple[str, int, int]]]:
        return [[(op, m, p) for (op, m, p, *_r) in self.instrs(d)] for d in range(self.S)]

    def simulate(self) -> SimReport:
        s = CSim()
        _check(_lib.lib().mario_plan_simulate(self.handle, C.byref(s)))
        n = s.n_dev
        return SimReport(s.makespan_ms, s.bubble_ratio, [s.busy_ms[i] for i in range(n)],
                         [s.peak_bytes[i] for i in range(n)], [s.max_live_act[i] for i in range(n)],
                         [s.max_live_ckpt[i] for i in range(n)])

    def timeline(self, d: int):
        a, b, n = C.POINTER(C.c_double)(), C.POINTER(C.c_double)(), C.c_int32()
        _check(_lib.lib().mario_plan_timeline(self.handle, d, C.byref(a), C.byref(b), C.byref(n)))
        return [a[i] for i in range(n.value)], [b[i] for i in range(n.value)]

    def comm_ops(self, rank: int):
        """Rank's NCCL program: [(kind, a, b, c, micro, part, list_index, count)] (mario_commop)."""
        p, n = C.POINTER(CCommOp)(), C.c_int32()
        _check(_lib.lib().mario_plan_comm_ops(self.handle, rank, C.byref(p), C.byref(n)))
        return [(p[i].kind, p[i].a, p[i].b, p[i].c, p[i].micro, p[i].part, p[i].list_index, p[i].count)
                for i in range(n.value)]

    def comm_ops_dp(self, rank: int, dp: int):
        """World rank's program under PP x DP (world = S * dp; mario_plan_comm_ops_dp)."""
        p, n = C.POINTER(CCommOp)(), C.c_int32()
        _check(_lib.lib().mario_plan_comm_ops_dp(self.handle, dp, rank, C.byref(p), C.byref(n)))
        return [(p[i].kind, p[i].a, p[i].b, p[i].c, p[i].micro, p[i].part, p[i].list_index, p[i].count)
                for i in range(n.value)]

    def serialize(self) -> str:
        need = C.c_size_t()
        _check(_lib.lib().mario_plan_serialize(self.handle, None, 0, C.byref(need)))
        buf = C.create_string_buffer(need.value)
        _check(_lib.lib().mario_plan_serialize(self.handle, buf, need.value, C.byref(need)))
        return buf.value.decode()

    def rank_layout(self, rank: int) -> Tuple[int, int]:
        """(packed parameter count, workspace bytes); rank=-1: loopback totals."""
        pc, ws = C.c_uint64(), C.c_uint64()
        _check(_lib.lib().mario_plan_rank_layout(self.handle, rank, C.byref(pc), C.byref(ws)))
        return pc.value, ws.value

    def param_names(self) -> List[str]:
        L = _lib.lib()
        return [L.mario_param_name(self.handle, i).decode() for i in range(L.mario_param_count(self.handle))]

    def rank_params(self, rank: int) -> List[Tuple[str, int, int]]:
        """[(name, element offset, element count)] of rank's packed buffer, in order."""
        idx, off, cnt, n = C.POINTER(C.c_int32)(), C.POINTER(C.c_uint64)(), C.POINTER(C.c_uint64)(), C.c_int32()
        _check(_lib.lib().mario_plan_rank_params(self.handle, rank, C.byref(idx), C.byref(off), C.byref(cnt),
                                                 C.byref(n)))
        names = self.param_names()
        return [(names[idx[i]], off[i], cnt[i]) for i in range(n.value)]


# ------------------------------------------------------------------------- executor
def pack_params(plan: Plan, params: Dict[str, "object"], rank: int):
    """Pack a {name: array} model into rank's fp32 buffer (rank=-1 loopback / -2 emulated ranks:
    all ranks concatenated). Pure layout marshalling (offsets come from the library)."""
    import numpy as np
    ranks = range(plan.S) if rank < 0 else [rank]
    bufs = []
    for r in ranks:
        total = plan.rank_layout(r)[0]
        b = np.zeros(total, dtype=np.float32)
        for name, off, cnt in plan.rank_params(r):
            b[off:off + cnt] = np.asarray(params[name], dtype=np.float32).reshape(-1)
        bufs.append(b)
    return np.concatenate(bufs) if bufs else np.zeros(0, np.float32)


def unpack_params(plan: Plan, flat, rank: int) -> Dict[str, "object"]:
    """Inverse of pack_params for grads: {name: array} (first copy of every tensor)."""
    import numpy as np
    shapes = {n: s for n, s in _shapes(plan)}
    out = {}
    ranks = range(plan.S) if rank < 0 else [rank]
    base = 0
    for r in ranks:
        for name, off, cnt in plan.rank_params(r):
            if name not in out:
                out[name] = np.asarray(flat[base + off: base + off + cnt]).reshape(shapes[name])
        base += plan.rank_layout(r)[0]
    return out


def _shapes(plan: Plan):
    """(name, shape) of every global parameter, from the library (mario_param_shape)."""
    L = _lib.lib()
    out = []
    dims, nd = (C.c_int64 * 4)(), C.c_int32()
    for i, name in enumerate(plan.param_names()):
        _check(L.mario_param_shape(plan.handle, i, dims, C.byref(nd)))
        out.append((name, tuple(int(dims[j]) for j in range(nd.value))))
    return out


class Context:
    """mario_init_dp(rank, world, device, dp, nccl_id). world > 1 uses torch.distributed (already
    initialised) only to broadcast the 128-byte NCCL unique id. dp > 1: PP x DP, world = S * dp,
    rank = replica * S + stage (reading A29)."""

    def __init__(self, rank: int = 0, world: int = 1, device: int = 0, dp: int = 1):
        L = _lib.lib()
        uid = C.create_string_buffer(128)
        if world > 1:
            import torch
            import torch.distributed as dist
            if rank == 0:
                _check(L.mario_nccl_unique_id(uid))
            t = torch.tensor(list(uid.raw), dtype=torch.uint8)
            if dist.get_backend() == "nccl":      # NCCL process groups only move device tensors
                t = t.to(torch.device("cuda", device))
            dist.broadcast(t, src=0)
            uid = C.create_string_buffer(bytes(t.cpu().tolist()), 128)
        _check(L.mario_init_dp(rank, world, device, dp, uid if world > 1 else None))
        self.rank, self.world, self.dp = rank, world, dp

    @classmethod
    def emulated(cls, world: int, device: int = 0, sms_per_rank: int = 0) -> "Context":
        """mario_init_emulated: `world` pipeline ranks in this process on one GPU, each on its own
        streams (and, with sms_per_rank > 0, its own green-context SM partition), exchanging
        activations and gradients through the peer transport. Buffers: alloc_for(plan, -2)."""
        self = cls.__new__(cls)
        _check(_lib.lib().mario_init_emulated(world, device, sms_per_rank))
        self.rank, self.world, self.dp = 0, world, 1
        self.sms_per_rank = int(_lib.lib().mario_emulated_sms())
        return self

    @classmethod
    def peer(cls, rank: int, world: int, device: int = 0) -> "Context":
        """mario_init_peer: one process per pipeline rank exchanging activations and gradients through
        the peer transport over CUDA IPC (same GPU, or GPUs with peer access). Call bind() with the
        rank's workspace and grads before run_iter."""
        self = cls.__new__(cls)
        _check(_lib.lib().mario_init_peer(rank, world, device))
        self.rank, self.world, self.dp = rank, world, 1
        return self

    def bind(self, workspace, grads, allgather=None):
        """Publish this rank's buffers (mario_peer_export) and map every other rank's
        (mario_peer_import). allgather(bytes) -> [bytes per rank]; default: torch.distributed
        all_gather_object on the current process group (argument marshalling only)."""
        rec = C.create_string_buffer(256)
        _check(_lib.lib().mario_peer_export(C.c_void_p(workspace.data_ptr()), C.c_void_p(grads.data_ptr()), rec))
        if allgather is None:
            import torch.distributed as dist
            out = [None] * self.world
            dist.all_gather_object(out, rec.raw)
        else:
            out = allgather(rec.raw)
        buf = C.create_string_buffer(b"".join(out), 256 * self.world)
        _check(_lib.lib().mario_peer_import(buf))

    def run_iter(self, plan: Plan, weights, tokens, grads, workspace, stream=None) -> float:
        """weights/grads/workspace: device tensors (data_ptr used); tokens: host int32 array."""
        import numpy as np
        if hasattr(tokens, "data_ptr"):          # torch tensor (host or device), int32 contiguous
            assert tokens.dtype.__str__() == "torch.int32" and tokens.is_contiguous()
            tok_ptr = C.c_void_p(tokens.data_ptr())
        else:
            tok = np.ascontiguousarray(tokens, dtype=np.int32)
            tok_ptr = tok.ctypes.data_as(C.c_void_p)
        loss = C.c_float()
        st = stream.cuda_stream if stream is not None else None
        _check(_lib.lib().mario_run_iter(plan.handle, C.c_void_p(weights.data_ptr()),
                                         tok_ptr, C.byref(loss),
                                         C.c_void_p(grads.data_ptr()), C.c_void_p(workspace.data_ptr()),
                                         C.c_void_p(st) if st else None))
        return float(loss.value)

    def set_graphs(self, on: bool):
        _check(_lib.lib().mario_set_graphs(int(on)))

    def set_timing(self, on: bool):
        _check(_lib.lib().mario_set_timing(int(on)))

    def last_timeline(self, d: int):
        a, b, n = C.POINTER(C.c_double)(), C.POINTER(C.c_double)(), C.c_int32()
        _check(_lib.lib().mario_last_timeline(d, C.byref(a), C.byref(b), C.byref(n)))
        return [a[i] for i in range(n.value)], [b[i] for i in range(n.value)]

    def last_costs(self, plan: Plan, p2p_alpha_ms: float = 0.005, p2p_GBps: float = 1500.0) -> dict:
        """mario_last_costs: the measured per-virtual-stage costs of the last timed iteration, as the
        `costs` dict Plan() takes (the paper's profile -> simulate loop)."""
        K = plan.S * (plan.chunks if plan.scheme == "interleave" else 1)
        fw, bw, rc = (C.c_double * K)(), (C.c_double * K)(), (C.c_double * K)()
        _check(_lib.lib().mario_last_costs(plan.handle, fw, bw, rc))
        return {"fw_ms": list(fw), "bw_ms": list(bw), "rc_ms": list(rc), "p2p_alpha_ms": p2p_alpha_ms,
                "p2p_GBps": p2p_GBps}

    def close(self):
        _lib.lib().mario_finalize()


_DEFAULT_CTX = []


def default_context(device: int = 0) -> "Context":
    """The process's single-GPU context (rank 0 of world 1), created on first use. The library
    holds one executor context per process, so every single-process caller shares this one."""
    if not _DEFAULT_CTX:
        import torch
        torch.cuda.set_device(device)
        _DEFAULT_CTX.append(Context(0, 1, device))
    return _DEFAULT_CTX[0]


def close_default_context() -> None:
    """Finalize the process's default context (the library holds one executor context per
    process), e.g. before creating an emulated one."""
    if _DEFAULT_CTX:
        _DEFAULT_CTX.pop().close()


def alloc_for(plan: Plan, rank: int, device="cuda"):
    """Allocate (weights, grads, workspace) device tensors sized from the plan (torch is
    used only as the device allocator). rank -1: loopback, -2: emulated ranks (peer transport)."""
    import torch
    pc, ws = plan.rank_layout(rank)
    w = torch.zeros(pc, dtype=torch.float32, device=device)
    g = torch.zeros(pc, dtype=torch.float32, device=device)
    work = torch.empty(max(ws, 1), dtype=torch.uint8, device=device)
    return w, g, work


SCHEME_NAMES = {0: "1f1b", 1: "interleave", 2: "chimera"}
LEVEL_NAMES = {0: "base", 1: "ckpt", 2: "mario", 3: "mario_budget"}


def tune(cfg, devices: int, global_batch: int, mem_budget: int = 0, costs: Optional[dict] = None,
         dtype: str = "bf16"):
    """mario_tune (Eq. 1): returns (all evaluated configurations as dicts, index of the best)."""
    m = cmodel(cfg, dtype)
    cc = None
    keep = []
    if costs is not None:
        mbs = costs.get("mbs", [])
        keep = [(C.c_int32 * len(mbs))(*mbs)] + [_darr(costs.get(k)) for k in ("layer_fw_ms", "layer_bw_ms",
                                                                               "head_fw_ms", "head_bw_ms")]
        cc = CTuneCosts(len(mbs), keep[0], keep[1], keep[2], keep[3], keep[4], costs.get("p2p_alpha_ms", 0.01),
                        costs.get("p2p_GBps", 700.0), costs.get("dp_efficiency", 0.95))
    cap = 1024
    res = (CTuneResult * cap)()
    n, best = C.c_int32(), C.c_int32()
    _check(_lib.lib().mario_tune(C.byref(m), devices, global_batch, mem_budget, C.byref(cc) if cc else None, res,
                                 cap, C.byref(n), C.byref(best)))
    rows = []
    for i in range(n.value):
        r = res[i]
        rows.append({"scheme": SCHEME_NAMES[r.scheme], "pp": r.pp, "chunks": r.chunks, "dp": r.dp,
                     "micro_batch": r.micro_batch, "microbatches": r.microbatches, "level": LEVEL_NAMES[r.level],
                     "feasible": bool(r.feasible), "makespan_ms": r.makespan_ms, "samples_per_s": r.samples_per_s,
                     "bubble_ratio": r.bubble_ratio, "peak_bytes": r.peak_bytes})
    return rows, best.value


def profile_costs(cfg, mbs_list=(1, 2, 4, 8), ctx: Optional["Context"] = None, dtype: str = "bf16",
                  p2p_alpha_ms: float = 0.01, p2p_GBps: float = 770.0, dp_efficiency: float = 0.95,
                  seed: int = 0) -> dict:
    """The paper's profiling step ("we profile the execution time of each layer ... under
    different micro-batch sizes") as the measured estimators mario_tune takes (Eq. 1):
    for every micro-batch size, a 2-layer slice of `cfg` runs as a 2-stage BASE 1F1B plan with 2
    micro-batches in loopback, timed per instruction (mario_set_timing); stage 0's FW / BW give
    the per-layer forward / backward time, the last stage's excess over it the embedding + head
    (+ loss) time. Weights N(0, 0.02) and uniform tokens on the device (the dense model's speed
    does not depend on their values). Returns the `costs` dict tune() takes."""
    import torch
    ctx = ctx or default_context()
    gen = torch.Generator(device="cuda").manual_seed(seed)
    out = {"mbs": [], "layer_fw_ms": [], "layer_bw_ms": [], "head_fw_ms": [], "head_bw_ms": [],
           "p2p_alpha_ms": p2p_alpha_ms, "p2p_GBps": p2p_GBps, "dp_efficiency": dp_efficiency}
    for mbs in mbs_list:
        sl = replace(cfg, n_layers=2, micro_batch=mbs)
        plan = Plan(sl, 2, 2, "1f1b", "base", dtype=dtype)
        w, g, ws = alloc_for(plan, -1)
        w.normal_(0.0, 0.02, generator=gen)
        toks = torch.randint(0, cfg.vocab, (2 * mbs, cfg.seq_len + 1), dtype=torch.int32, device="cuda",
                             generator=gen)
        for _ in range(2):   # warm-up (first-call setup, graph capture)
            ctx.run_iter(plan, w, toks, g, ws)
        ctx.set_timing(True)
        try:
            ctx.run_iter(plan, w, toks, g, ws)
        finally:
            ctx.set_timing(False)
        c = ctx.last_costs(plan)
        out["mbs"].append(mbs)
        out["layer_fw_ms"].append(c["fw_ms"][0])
        out["layer_bw_ms"].append(c["bw_ms"][0])
        out["head_fw_ms"].append(max(0.0, c["fw_ms"][1] - c["fw_ms"][0]))
        out["head_bw_ms"].append(max(0.0, c["bw_ms"][1] - c["bw_ms"][0]))
        del w, g, ws, toks
        torch.cuda.empty_cache()
    return out


def max_seq_len(cfg, stages: int, microbatches: int, level: str, mem_budget: int, scheme: str = "1f1b",
                chunks: int = 1, start: int = 1024, step: int = 64, limit: int = 1 << 20) -> int:
    """Sequence-length scaling (§6.5): the largest s = start + i*step
    whose plan's simulated per-device peak (static + activations) fits mem_budget, or 0 when
    `start` does not fit. Planner only: nothing is executed. Peaks grow with s, so the search is a
    doubling phase then a bisection over multiples of `step`."""
    def fits(s_len):
        try:
            Plan(replace(cfg, seq_len=s_len), stages, microbatches, scheme, level, chunks=chunks,
                 mem_budget=mem_budget)
            return True
        except MarioError as e:
            if e.code != -2:
                raise
            return False
    if not fits(start):
        return 0
    lo, hi = 0, 1   # in steps beyond start: lo fits, hi unknown
    while start + hi * step <= limit and fits(start + hi * step):
        lo, hi = hi, hi * 2
    hi = min(hi, (limit - start) // step + 1)
    while hi - lo > 1:
        mid = (lo + hi) // 2
        if fits(start + mid * step):
            lo = mid
        else:
            hi = mid
    return start + lo * step


def adamw_step(params, grads, m, v, step: int, lr: float, beta1=0.9, beta2=0.95, eps=1e-8, weight_decay=0.1,
               stream=None):
    """mario_adamw_step on packed device buffers (torch tensors)."""
    st = stream.cuda_stream if stream is not None else None
    _check(_lib.lib().mario_adamw_step(C.c_void_p(params.data_ptr()), C.c_void_p(grads.data_ptr()),
                                       C.c_void_p(m.data_ptr()), C.c_void_p(v.data_ptr()), params.numel(), lr, beta1,
                                       beta2, eps, weight_decay, step, C.c_void_p(st) if st else None))


def chrome_trace(plan: Plan, measured: Optional[List[Tuple[List[float], List[float]]]] = None) -> dict:
    """Chrome-trace (chrome://tracing / Perfetto) of a plan's simulated timeline (pid 0) and,
    optionally, a measured one from Context.last_timeline per device (pid 1): the visualization of
    PAPER.md P:256 (Fig. 5), one row per device, one box per FW/CFW/RC/BW instruction."""
    events = []
    for pid, label, src in ((0, "simulated", None), (1, "measured", measured)):
        if pid == 1 and measured is None:
            continue
        events.append({"name": "process_name", "ph": "M", "pid": pid, "args": {"name": label}})
        for d in range(plan.S):
            comp = [x for x in plan.instrs(d) if x[0] in ("FW", "CFW", "RC", "BW")]
            starts, fins = plan.timeline(d) if src is None else src[d]
            events.append({"name": "thread_name", "ph": "M", "pid": pid, "tid": d, "args": {"name": f"device {d}"}})
            for (op, m, p, k, *_r), t0, t1 in zip(comp, starts, fins):
                events.append({"name": f"{op}{m}" + (f".{p}" if plan.scheme != "1f1b" else ""), "cat": op, "ph": "X",
                               "pid": pid, "tid": d, "ts": t0 * 1e3, "dur": (t1 - t0) * 1e3,
                               "args": {"micro": m, "part": p, "vstage": k}})
    return {"traceEvents": events, "displayTimeUnit": "ms"}
