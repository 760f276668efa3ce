#!/usr/bin/env python
"""Per-kernel mean duration and share of an ncu --metrics gpu__time_duration.sum CSV."""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hi]; ki = h.index('Kernel Name'); vi = h.index('Metric Value')
agg = {}
order = []
for r in rows[hi + 1:]:
    if len(r) <= vi:
        continue
    name = r[ki].split('(')[0]
    try:
        v = float(r[vi].replace(',', ''))
    except ValueError:
        continue
    if name not in agg:
        order.append(name)
    agg.setdefault(name, []).append(v)
tot = sum(sum(v) for v in agg.values())
for k in order:
    v = agg[k]
    print(f"{k[:60]:60s} n={len(v):4d} mean={sum(v)/len(v)/1e3:9.2f} us share={sum(v)/tot:.3f}")
