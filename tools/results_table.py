#!/usr/bin/env python
"""Summarise gpurun_out/results/*.json (bench lines) into a markdown table."""
import glob
import json
import os
import sys

rows = []
for f in sorted(glob.glob(os.path.join(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/results", "*.json"))):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        continue
    r = d["roofline"]
    iqr = d.get("lp_overhead_detail", {}).get("iqr_pct", [float("nan")] * 2)
    rows.append("| {w} | {ck} | {st} | {tp:.3f} | {tu:.3f} | {ov:+.2f}% [{q0:+.2f}, {q1:+.2f}] | {ach} {unit} ({frac:.1%}) | {tv:.3f} | {vf:.1%} | {trec:.3f} | {val} | {col} | {mhz} |".format(
        q0=iqr[0], q1=iqr[1], mhz=d["clocks"].get("sm_mhz"),
        w=d["config"]["workload"], ck=d["config"]["cksum"].replace("|", "\\|"), st=d["config"]["store"], tp=d["t_protected_ms"],
        tu=d["t_unprotected_ms"], ov=d["lp_overhead_pct"], ach=r["achieved"], unit=r["unit"].split()[0],
        frac=r["frac"], tv=d["t_validate_ms"], vf=d["roofline_validate"]["frac"], trec=d["t_recovery_phase_ms"],
        val=d["value"], col=d.get("hash_collisions")))
print("| workload | checksum | store | t_prot ms | t_unprot ms | LP overhead [pair IQR] | body roofline | t_validate ms | validate frac | recovery phase ms | value GB/s | collisions | SM MHz (median) |")
print("|---|---|---|---|---|---|---|---|---|---|---|---|---|")
print("\n".join(rows))
