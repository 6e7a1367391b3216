"""Per-source-line instruction counts and stall samples of an .ncu-rep (needs -lineinfo):
python tools/ncu_source_top.py <rep> [n]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hi = next(i for i, r in enumerate(rows) if "Source" in r)
h = rows[hi]
li = h.index("# Line") if "# Line" in h else None
si, ii, ss = h.index("Source"), h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
data = []
for r in rows[hi + 1:]:
    if len(r) != len(h):
        continue
    try:
        data.append((float(r[ii] or 0), float(r[ss] or 0), r[li] if li is not None else "", r[si].strip()[:110]))
    except ValueError:
        pass
tot_i = sum(d[0] for d in data) or 1
tot_s = sum(d[1] for d in data) or 1
print(f"total warp instructions {tot_i:.3e}, stall samples {tot_s:.0f}")
for d in sorted(data, reverse=True)[:n]:
    print(f"{d[0] / tot_i:6.1%} inst {d[1] / tot_s:6.1%} stall  L{d[2]:>4s}  {d[3]}")
