#!/usr/bin/env python
"""Summarise gpurun_out/cksum_sweep_<w>.csv (ncu --csv, one row per metric per launch) into a markdown table:
the profiled (second) launch of each checksum set, and the deltas against the unprotected twin."""
import csv
import sys
from collections import OrderedDict

MASKS = [0, 1, 2, 3, 4, 7]
NAMES = {0: "none (twin)", 1: "MOD", 2: "XOR", 3: "MOD|XOR", 4: "ADLER32", 7: "MOD|XOR|ADLER32"}


def load(path):
    rows = [r for r in csv.reader(open(path)) if r and not r[0].startswith("==")]
    hdr = rows[0]
    iid, imn, imv, iunit = hdr.index("ID"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    per = OrderedDict()
    for r in rows[1:]:
        per.setdefault(int(r[iid]), {})[r[imn]] = (float(r[imv].replace(",", "")), r[iunit])
    return list(per.values())


def main():
    w = sys.argv[1]
    launches = load(f"gpurun_out/cksum_sweep_{w}.csv")
    assert len(launches) == 2 * len(MASKS), len(launches)
    prof = {m: launches[2 * i + 1] for i, m in enumerate(MASKS)}

    def val(m, k, scale=1.0):
        v, unit = prof[m][k]
        if unit in ("usecond", "us"):
            v *= 1e-3
        if unit in ("nsecond", "ns"):
            v *= 1e-6
        if unit in ("msecond", "ms"):
            v *= 1.0
        if unit in ("Kbyte",):
            v *= 1e3
        if unit in ("Mbyte",):
            v *= 1e6
        if unit in ("Gbyte",):
            v *= 1e9
        return v * scale

    t0 = val(0, "gpu__time_duration.sum")
    w0 = val(0, "dram__bytes_write.sum")
    i0 = val(0, "sm__inst_executed.sum")
    print(f"| checksum | time (ms) | vs twin | tensor pipe % | ALU pipe % | FMA pipe % | ALU inst (M) | inst (M) | "
          f"DRAM read (MB) | DRAM write (MB) | extra DRAM writes vs twin (E9 analog) |")
    print("|---|---|---|---|---|---|---|---|---|---|---|")
    for m in MASKS:
        t = val(m, "gpu__time_duration.sum")
        wr = val(m, "dram__bytes_write.sum")
        print(f"| {NAMES[m]} | {t:.4f} | {100 * (t / t0 - 1):+.2f}% | "
              f"{val(m, 'sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed'):.1f} | "
              f"{val(m, 'sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_elapsed'):.1f} | "
              f"{val(m, 'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_elapsed'):.1f} | "
              f"{val(m, 'sm__inst_executed_pipe_alu.sum') / 1e6:.1f} | {val(m, 'sm__inst_executed.sum') / 1e6:.1f} | "
              f"{val(m, 'dram__bytes_read.sum') / 1e6:.1f} | {wr / 1e6:.2f} | {wr - w0:+.0f} B ({100 * (wr / w0 - 1):+.3f}%) |")


if __name__ == "__main__":
    main()
