"""Hot SASS lines of one kernel from `ncu -i rep --page source --csv --print-source sass` output."""
import csv
import sys

r = list(csv.reader(open(sys.argv[1])))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr = None
rows = []
for x in r:
    if 'Address' in x and 'Source' in x:
        hdr = x
        continue
    if hdr and len(x) == len(hdr) and x[0].startswith('0x'):
        rows.append(x)
ai, si, wi, ei = hdr.index('Address'), hdr.index('Source'), hdr.index('Warp Stall Sampling (All Samples)'), \
    hdr.index('Instructions Executed')
iv = lambda s: int(s) if s.isdigit() else 0
tot = sum(iv(x[wi]) for x in rows)
print('total samples', tot, 'instructions', len(rows))
for i, x in enumerate(rows):
    x.append(i)
for x in sorted(rows, key=lambda x: -iv(x[wi]))[:n]:
    print(f"{iv(x[wi]):6d} {100 * iv(x[wi]) / max(tot, 1):5.1f}% {x[ei]:>8s} #{x[-1]:5d} {x[si].strip()[:100]}")
