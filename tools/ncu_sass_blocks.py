"""Instruction share of an .ncu-rep's SASS in blocks of N instructions: python tools/ncu_sass_blocks.py <rep> [N]"""
import csv
import io
import subprocess
import sys

txt = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hi = next(i for i, r in enumerate(rows) if "Source" in r and "Address" in r)
h = rows[hi]
si, ii = h.index("Source"), h.index("Instructions Executed")
data = [(float(r[ii] or 0), r[si].strip()) for r in rows[hi + 1:] if len(r) == len(h)]
tot = sum(d[0] for d in data)
N = int(sys.argv[2]) if len(sys.argv) > 2 else 20
for b in range(0, len(data), N):
    s = sum(d[0] for d in data[b:b + N])
    if s / tot > 0.01:
        print(f"{b:4d}-{b + N - 1:4d} {s / tot:6.1%}  {data[b][1][:44]} ... {data[min(b + N - 1, len(data) - 1)][1][:40]}")
