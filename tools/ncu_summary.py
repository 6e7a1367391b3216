#!/usr/bin/env python
"""Summarise an ncu evidence pass into profiles/<round>/summary.md and profiles/ncu_traffic.json.

usage: python tools/ncu_summary.py <round_dir>   (expects *.raw.csv and launches_*.csv inside)
"""
import collections
import csv
import glob
import json
import os
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__grid_size", "sm__cycles_elapsed.avg.per_second",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "us": 1e-6, "ms": 1e-3, "ns": 1e-9, "s": 1}
WL = {"tmm": "tmm8192_bf16", "stencil": "stencil32768", "spmv": "spmv4m", "tf32": "tmm8192_f32"}


def raw(path):
    rows = list(csv.reader(open(path)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = {}
    for i, h in enumerate(hdr):
        d[h] = (vals[i], units[i])
    return d


def num(v):
    return float(v[0].replace(",", "")) * SCALE.get(v[1], 1)


def main(rdir):
    out = ["# ncu evidence, " + os.path.basename(rdir.rstrip("/")), "",
           "Captured with `tools/ncu_pass.sh` under gpurun (1x B200, `--clock-control none`). "
           "`--set full` numbers are from one launch of each kernel; launch lists are cold-cache and serialised, "
           "so compare SHARES, not absolute times.", ""]
    traffic = {}
    tp = os.path.join(os.path.dirname(rdir.rstrip("/")), "ncu_traffic.json")
    if os.path.exists(tp):
        traffic = json.load(open(tp))
    for f in sorted(glob.glob(os.path.join(rdir, "prof_*.raw.csv"))):
        d = raw(f)
        name = d["Kernel Name"][0]
        tag = os.path.basename(f).replace(".raw.csv", "")
        out.append(f"## {tag}")
        out.append(f"`{name[:150]}`")
        out.append("")
        out.append("| metric | value |")
        out.append("|---|---|")
        for k in KEYS:
            if k in d:
                out.append(f"| {k} | {d[k][0]} {d[k][1]} |")
        rd, wr = num(d["dram__bytes_read.sum"]), num(d["dram__bytes_write.sum"])
        out.append(f"| dram read+write per launch | {rd + wr:.4g} B |")
        out.append("")
        wl = WL["stencil" if "stencil" in tag else ("spmv" if "spmv" in tag else ("tf32" if "tf32" in tag else "tmm"))]
        kern = name.split("<")[0].split("::")[-1].replace("void ", "").strip()
        if "recover" in tag:
            kern += "_list_mode"
        traffic.setdefault(wl, {})[kern] = int(rd + wr)
    for f in sorted(glob.glob(os.path.join(rdir, "launches_*.csv"))):
        rows = [r for r in csv.reader(open(f)) if len(r) > 5]
        hdr = rows[0]
        ix = {h: i for i, h in enumerate(hdr)}
        tot, cnt = collections.defaultdict(float), collections.Counter()
        for r in rows[1:]:
            if r[ix["Metric Name"]] != "gpu__time_duration.sum":
                continue
            nm = r[ix["Kernel Name"]].split("(")[0].replace("void ", "").replace("(anonymous namespace)::", "")
            v = float(r[ix["Metric Value"]].replace(",", "")) * SCALE.get(r[ix["Metric Unit"]], 1e-9) * 1e6
            tot[nm[:90]] += v
            cnt[nm[:90]] += 1
        T = sum(tot.values())
        out.append(f"## launch list {os.path.basename(f)} (total {T:.1f} us)")
        out.append("")
        out.append("| share | total us | launches | avg us | kernel |")
        out.append("|---|---|---|---|---|")
        for k, v in sorted(tot.items(), key=lambda x: -x[1])[:14]:
            out.append(f"| {100 * v / T:.2f}% | {v:.1f} | {cnt[k]} | {v / cnt[k]:.1f} | `{k}` |")
        out.append("")
    with open(os.path.join(rdir, "summary.md"), "w") as fo:
        fo.write("\n".join(out) + "\n")
    with open(tp, "w") as fo:
        json.dump(traffic, fo, indent=1, sort_keys=True)
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1])
