"""Write tests/golden/* files that are derived values. Calls ONLY oracle/ (and synth for
shapes) — never the CUDA/C++ product. Usage: python tests/tools/make_goldens.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from oracle import schedule as osch  # noqa: E402


def serialize(cfg, dtype, pipe, level, lists):
    fam = cfg.family
    s = "mario-plan v1\n"
    s += (f"model family={fam} L={cfg.n_layers} h={cfg.hidden} heads={cfg.n_heads} f={cfg.ffn_hidden} "
          f"V={cfg.vocab} s={cfg.seq_len} mbs={cfg.micro_batch} tie={int(cfg.tie_embeddings)} dtype={dtype}\n")
    s += f"pipe scheme={pipe.scheme} S={pipe.S} N={pipe.N} v={pipe.v} level={level}\n"
    for d, L in enumerate(lists):
        s += f"dev {d}:" + "".join(f" {op}{m}.{p}" for op, m, p in L) + "\n"
    return s


def main():
    g = os.path.join(ROOT, "tests", "golden")
    # Fig. 2: 4-stage 1F1B, 4 micro-batches, unit costs, Mario passes 1-4
    cfg = synth.with_(synth.TINY_GPT, n_layers=4)
    pipe = osch.Pipe(osch.V_1F1B, 4, 4)
    lists = osch.transform(pipe, osch.MARIO, osch.UnitCosts())
    open(os.path.join(g, "plan_fig2_mario.txt"), "w").write(serialize(cfg, "f32", pipe, "mario", lists))


if __name__ == "__main__":
    main()
