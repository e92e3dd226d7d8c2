#!/usr/bin/env python
"""Per-kernel times of the last bench step in an ncu launch list (gpurun_out/launches.csv)."""
import collections, csv, sys
rows = [r for r in csv.reader(open(sys.argv[1] if len(sys.argv) > 1 else 'gpurun_out/launches.csv')) if len(r) > 5]
h = rows[0]
ki, vi, ui = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
agg = collections.OrderedDict()
for r in rows[1:]:
    k = r[ki].split('(')[0].replace('void ', '').split('<')[0]
    v = float(r[vi].replace(',', ''))
    v *= {'nsecond': 1e-6, 'ns': 1e-6, 'usecond': 1e-3, 'us': 1e-3, 'msecond': 1.0, 'ms': 1.0}.get(r[ui], 1.0)
    agg.setdefault(k, []).append(v)
tot = 0.0
for k, v in agg.items():
    if k == 'k_int_peak':
        continue
    print(f"{k:24s} n={len(v):3d} last={v[-1]:.3f} ms")
    tot += v[-1]
print(f"{'sum of last':24s} {tot:.3f} ms")
