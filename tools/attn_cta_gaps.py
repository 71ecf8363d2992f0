"""Per-SM CTA timeline of fa_bwd_dkdv_ts from the MARIO_ATTN_TRACE_CTAS dump (CTA, SM, start ns,
end ns): CTA durations by key block, idle gaps between consecutive CTAs on an SM, and SM busy
fraction over the kernel.

    python tools/attn_cta_gaps.py ctas.txt [n_key_blocks=16]
"""
import collections
import sys

rows = [tuple(int(x) for x in ln.split()) for ln in open(sys.argv[1]) if ln.strip()]
nkb = int(sys.argv[2]) if len(sys.argv) > 2 else 16
t0 = min(r[2] for r in rows)
t1 = max(r[3] for r in rows)
per_sm = collections.defaultdict(list)
for cta, sm, a, b in rows:
    per_sm[sm].append((a - t0, b - t0, cta))
bh = len(rows) // nkb
dur = collections.defaultdict(list)
for cta, sm, a, b in rows:
    dur[cta // bh].append(b - a)
print(f"kernel span {(t1 - t0) / 1e3:.1f} us over {len(per_sm)} SMs, {len(rows)} CTAs")
for kb in sorted(dur):
    d = dur[kb]
    print(f"  key block {kb:2d} ({2 * (nkb - kb)} tiles): CTA {sum(d) / len(d) / 1e3:6.2f} us avg, "
          f"{min(d) / 1e3:6.2f}-{max(d) / 1e3:6.2f}")
gaps, busy, ends = [], 0, []
for sm, L in per_sm.items():
    L.sort()
    busy += sum(b - a for a, b, _ in L)
    ends.append(L[-1][1])
    gaps += [L[j + 1][0] - L[j][1] for j in range(len(L) - 1)]
gaps.sort()
print(f"gap between CTAs on an SM: median {gaps[len(gaps) // 2] / 1e3:.2f} us, p90 {gaps[int(len(gaps) * .9)] / 1e3:.2f} us")
print(f"SM busy fraction {busy / (len(per_sm) * (t1 - t0)):.3f}; SM finish times {min(ends) / 1e3:.1f}-{max(ends) / 1e3:.1f} us")
