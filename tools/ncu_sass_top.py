"""SASS-level instruction counts of an .ncu-rep: totals per opcode and the hottest instructions.
python tools/ncu_sass_top.py <rep> [n]"""
import collections
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hi = next(i for i, r in enumerate(rows) if "Source" in r and "Address" in r)
h = rows[hi]
si, ii, ss = h.index("Source"), h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
data = []
for r in rows[hi + 1:]:
    if len(r) != len(h):
        continue
    try:
        data.append((float(r[ii] or 0), float(r[ss] or 0), r[0], r[si].strip()))
    except ValueError:
        pass
tot_i = sum(d[0] for d in data) or 1
tot_s = sum(d[1] for d in data) or 1
op = collections.Counter()
for d in data:
    o = d[3].split()
    o = o[1] if o and o[0].startswith("@") and len(o) > 1 else (o[0] if o else "?")
    op[o.split(".")[0]] += d[0]
print(f"total warp instructions {tot_i:.3e}, stall samples {tot_s:.0f}")
print("by opcode:", ", ".join(f"{k}={v / tot_i:.1%}" for k, v in op.most_common(14)))
for idx, d in sorted(enumerate(data), key=lambda x: -x[1][1])[:n]:
    print(f"#{idx:4d} {d[0] / tot_i:6.2%} inst {d[1] / tot_s:6.2%} stall  {d[3][:90]}")
