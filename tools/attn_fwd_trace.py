"""Per-CTA timeline of the two-Q-tile attention forward (MARIO_ATTN_FWD_TRACE) at the cfg-2 shape:
CTA duration against its work (key-tile steps), SM busy fraction, gaps between CTAs on an SM."""
import collections
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
os.environ["MARIO_ATTN_FWD_TRACE"] = "/tmp/fwd_trace.txt"
from paper_conf_ppopp_liultj25_b200 import _lib  # noqa: E402

L = _lib.lib()
B, s, nh, dh = 4, 2048, 16, 128
h = nh * dh
qkv = torch.randn(B * s, 3 * h, device="cuda").bfloat16()
O = torch.empty(B * s, h, device="cuda", dtype=torch.bfloat16)
lse = torch.empty(nh, B * s, device="cuda")
L.mario_k_attn_set_variant(3)
for _ in range(3):
    assert L.mario_k_attn_fwd(qkv.data_ptr(), O.data_ptr(), lse.data_ptr(), B, s, nh, dh, 1, None) == 0
torch.cuda.synchronize()
rows = [list(map(int, l.split())) for l in open("/tmp/fwd_trace.txt")]
BH, nqb = B * nh, s // 256
t0 = min(r[2] for r in rows)
dur = collections.defaultdict(list)
per_sm = collections.defaultdict(list)
for j, sm, a, b in rows:
    qb = nqb - 1 - j // BH
    steps = (2 * qb + 1) + (2 * qb + 2)     # key tiles of Q tile 0 + Q tile 1
    dur[steps].append((b - a) / 1e3)
    per_sm[sm].append((a - t0, b - t0))
span = (max(r[3] for r in rows) - t0) / 1e3
print(f"kernel span {span:.1f} us over {len(per_sm)} SMs, {len(rows)} CTAs")
xs, ys = [], []
for k in sorted(dur):
    v = dur[k]
    print(f"  {k:3d} key-tile steps: CTA {np.mean(v):7.2f} us avg ({min(v):.2f}-{max(v):.2f}), n={len(v)}")
    xs += [k] * len(v)
    ys += v
a, b = np.polyfit(xs, ys, 1)
print(f"fit: CTA us = {b:.2f} + {a:.3f} * steps  ({a * 1e3 * 1.965 / 2:.0f} SM-clk per Q-tile step at 1965 MHz)")
gaps, busy = [], 0.0
for sm, iv in per_sm.items():
    iv.sort()
    busy += sum(e - st for st, e in iv)
    gaps += [(iv[i + 1][0] - iv[i][1]) / 1e3 for i in range(len(iv) - 1)]
print(f"gap between CTAs on an SM: median {np.median(gaps):.2f} us; SM busy fraction {busy / 1e3 / (span * len(per_sm)):.3f}")
