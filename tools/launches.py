"""Aggregate an ncu --metrics gpu__time_duration.sum CSV launch list by kernel name."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, agg = None, collections.defaultdict(lambda: [0.0, 0])
for r in rows:
    if 'Kernel Name' in r:
        hdr = r
        continue
    if hdr is None or len(r) != len(hdr):
        continue
    d = dict(zip(hdr, r))
    if d.get('Metric Name') != 'gpu__time_duration.sum':
        continue
    v = float(d['Metric Value'].replace(',', ''))
    v *= {'nsecond': 1e-3, 'ns': 1e-3, 'usecond': 1.0, 'us': 1.0, 'msecond': 1e3, 'ms': 1e3}.get(d['Metric Unit'], 1.0)
    k = d['Kernel Name'][:80]
    agg[k][0] += v
    agg[k][1] += 1
tot = sum(a[0] for a in agg.values())
print("| share | ms | launches | us/launch | kernel |\n|---|---|---|---|---|")
for k, (t, n) in sorted(agg.items(), key=lambda x: -x[1][0])[:int(sys.argv[2]) if len(sys.argv) > 2 else 30]:
    print(f"| {100 * t / tot:.2f}% | {t / 1e3:.3f} | {n} | {t / n:.1f} | `{k}` |")
print(f"total {tot / 1e3:.3f} ms")
