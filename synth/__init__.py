"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no layer maths, no schedule logic):
only model descriptions, parameter names/shapes in the packed order of SURVEY §8(c) c1,
and seeded random generators (SURVEY §8(c) reading A20).

The paper trains GPT3 / LLaMA2 on unnamed real data (Table 4
P:292-299); we use synthetic tokens uniform in [0, V) and random-init weights.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, asdict, replace
from typing import Dict, List, Tuple

import numpy as np

GPT, LLAMA = "gpt", "llama"


@dataclass(frozen=True)
class ModelCfg:
    family: str          # "gpt" | "llama"
    n_layers: int
    hidden: int
    n_heads: int
    ffn_hidden: int
    vocab: int
    seq_len: int
    micro_batch: int
    tie_embeddings: bool = True   # GPT: head tied to wte (A1); LLaMA: untied (A2)
    norm_eps: float = 1e-5
    rope_base: float = 10000.0

    @property
    def head_dim(self) -> int:
        return self.hidden // self.n_heads

    def to_dict(self) -> dict:
        return asdict(self)


# --- BASELINE.json configs (sizes per SURVEY §8(d) d1) ---------------------------------
TINY_GPT = ModelCfg(GPT, 4, 64, 4, 256, 256, 32, 2, True)
GPT3_1P3B = ModelCfg(GPT, 24, 2048, 16, 8192, 50304, 2048, 4, True)
LLAMA2_7B = ModelCfg(LLAMA, 32, 4096, 32, 11008, 32000, 4096, 1, False)
GPT3_2P7B = ModelCfg(GPT, 32, 2560, 32, 10240, 50304, 2048, 1, True)
LLAMA2_13B = ModelCfg(LLAMA, 40, 5120, 40, 13824, 32000, 16384, 1, False)

# (model, stages S, micro-batches N, scheme, chunks v) per BASELINE.json configs[0..4]
CONFIGS = {
    "cfg1_tiny_gpt": (TINY_GPT, 2, 4, "1f1b", 1),
    "cfg2_gpt3_1.3b": (GPT3_1P3B, 8, 32, "1f1b", 1),
    "cfg3_llama2_7b": (LLAMA2_7B, 8, 32, "interleave", 2),
    "cfg4_gpt3_2.7b": (GPT3_2P7B, 8, 32, "chimera", 1),
    "cfg5_llama2_13b": (LLAMA2_13B, 8, 16, "1f1b", 1),
}


def tiny_llama() -> ModelCfg:
    return ModelCfg(LLAMA, 4, 64, 4, 96, 256, 32, 2, False)


# --- parameter naming / packed order ---------------------------------
def embed_param_shapes(cfg: ModelCfg) -> List[Tuple[str, Tuple[int, ...]]]:
    if cfg.family == GPT:
        return [("wte", (cfg.vocab, cfg.hidden)), ("wpe", (cfg.seq_len, cfg.hidden))]
    return [("emb", (cfg.vocab, cfg.hidden))]


def layer_param_shapes(cfg: ModelCfg, l: int) -> List[Tuple[str, Tuple[int, ...]]]:
    h, f = cfg.hidden, cfg.ffn_hidden
    p = f"h{l}."
    if cfg.family == GPT:
        return [(p + "ln1.g", (h,)), (p + "ln1.b", (h,)),
                (p + "qkv.w", (3 * h, h)), (p + "qkv.b", (3 * h,)),
                (p + "proj.w", (h, h)), (p + "proj.b", (h,)),
                (p + "ln2.g", (h,)), (p + "ln2.b", (h,)),
                (p + "fc1.w", (f, h)), (p + "fc1.b", (f,)),
                (p + "fc2.w", (h, f)), (p + "fc2.b", (h,))]
    return [(p + "n1.g", (h,)), (p + "qkv.w", (3 * h, h)), (p + "o.w", (h, h)),
            (p + "n2.g", (h,)), (p + "gu.w", (2 * f, h)), (p + "down.w", (h, f))]


def head_param_shapes(cfg: ModelCfg) -> List[Tuple[str, Tuple[int, ...]]]:
    h = cfg.hidden
    if cfg.family == GPT:
        out = [("lnf.g", (h,)), ("lnf.b", (h,))]
        if not cfg.tie_embeddings:
            out.append(("head.w", (cfg.vocab, h)))
        return out
    return [("nf.g", (h,)), ("out.w", (cfg.vocab, h))]


def param_shapes(cfg: ModelCfg) -> List[Tuple[str, Tuple[int, ...]]]:
    out = list(embed_param_shapes(cfg))
    for l in range(cfg.n_layers):
        out += layer_param_shapes(cfg, l)
    out += head_param_shapes(cfg)
    return out


def n_params(cfg: ModelCfg) -> int:
    return sum(int(np.prod(s)) for _, s in param_shapes(cfg))


_RESIDUAL_OUT = ("proj.w", "fc2.w", "o.w", "down.w")


def _init_kind(name: str) -> str:
    leaf = name.split(".", 1)[1] if name.startswith("h") and "." in name and name[1].isdigit() else name
    if leaf.endswith(".g"):
        return "gamma"
    if leaf.endswith(".b"):
        return "beta" if leaf.startswith(("ln", "lnf")) else "bias"
    if leaf in _RESIDUAL_OUT:
        return "resid"
    return "matrix"


def make_weights(cfg: ModelCfg, seed: int = 1234, parity: bool = True,
                 dtype=np.float32) -> Dict[str, np.ndarray]:
    """Seeded weights (reading A20): PCG64(seed); matrices/embeddings N(0,0.02^2);
    residual-output matrices N(0,(0.02/sqrt(2L))^2). parity=True: biases N(0,0.02^2),
    gamma = 1 + N(0,0.1^2), beta N(0,0.02^2); parity=False (perf): 0 / 1 / 0."""
    rng = np.random.Generator(np.random.PCG64(seed))
    out = {}
    std_res = 0.02 / math.sqrt(2 * cfg.n_layers)
    for name, shape in param_shapes(cfg):
        kind = _init_kind(name)
        if kind == "matrix":
            w = rng.standard_normal(shape, dtype=np.float32) * 0.02
        elif kind == "resid":
            w = rng.standard_normal(shape, dtype=np.float32) * std_res
        elif kind == "gamma":
            w = (1.0 + 0.1 * rng.standard_normal(shape, dtype=np.float32)) if parity else np.ones(shape, np.float32)
        else:  # bias / beta
            w = (0.02 * rng.standard_normal(shape, dtype=np.float32)) if parity else np.zeros(shape, np.float32)
        out[name] = w.astype(dtype)
    return out


def make_tokens(cfg: ModelCfg, n_micro: int, iteration: int = 0, seed: int = 4321) -> np.ndarray:
    """Tokens uniform in [0, V): int32 [n_micro * mbs, s + 1] (reading A4/A20)."""
    rng = np.random.Generator(np.random.PCG64(seed + iteration))
    return rng.integers(0, cfg.vocab, size=(n_micro * cfg.micro_batch, cfg.seq_len + 1), dtype=np.int32)


def round_to_bf16(a: np.ndarray) -> np.ndarray:
    """Round fp32 -> bf16 (round-to-nearest-even) and back to fp32 (reading A6: the
    oracle consumes the bf16-rounded weights in bf16 mode). Pure bit manipulation."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    rounding = ((u >> 16) & 1) + 0x7FFF
    r = ((u + rounding) >> 16) << 16
    return r.astype(np.uint32).view(np.float32).reshape(a.shape)


def with_(cfg: ModelCfg, **kw) -> ModelCfg:
    return replace(cfg, **kw)
