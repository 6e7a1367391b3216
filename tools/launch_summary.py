"""Median per-kernel duration from an ncu launch list (--metrics gpu__time_duration.sum --csv)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = None
d = collections.defaultdict(list)
for r in rows:
    if 'Kernel Name' in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr) and r[hdr.index('Metric Name')] == 'gpu__time_duration.sum':
        unit = r[hdr.index('Metric Unit')]
        v = float(r[hdr.index('Metric Value')].replace(',', ''))
        v *= {'nsecond': 1e-3, 'ns': 1e-3, 'usecond': 1.0, 'us': 1.0, 'msecond': 1e3, 'ms': 1e3}.get(unit, 1.0)
        d[r[hdr.index('Kernel Name')][:90]].append(v)
for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1])):
    v = sorted(v)
    print(f"{k:92s} n={len(v):3d} median={v[len(v) // 2]:9.1f} us  total={sum(v):10.1f} us")
