#!/usr/bin/env python
"""Distribution of the 3xTF32 fp32 body's time (8192^3, 128x128 regions) over many reps: protected vs twin,
alternating, L2 flushed before each, SM clock sampled by NVML around every rep.  Prints sorted times and a
2-bin split, to see whether the run-to-run bimodality (4.36 / 4.72 ms in round 1) follows the variant, the
clock, or the rep order."""
import statistics
import sys
import time

import torch

sys.path.insert(0, ".")
import lpsynth  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

try:
    import pynvml
    pynvml.nvmlInit()
    hnd = pynvml.nvmlDeviceGetHandleByIndex(0)
    clk = lambda: pynvml.nvmlDeviceGetClockInfo(hnd, pynvml.NVML_CLOCK_SM)  # noqa: E731
    rsn = lambda: pynvml.nvmlDeviceGetCurrentClocksEventReasons(hnd)  # noqa: E731
    pwr = lambda: pynvml.nvmlDeviceGetPowerUsage(hnd) / 1000.0  # noqa: E731
except Exception:
    clk = rsn = pwr = lambda: -1  # noqa: E731
NAMES = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal", 0x40: "hw_thermal", 0x80: "hw_power_brake"}
wl_name = sys.argv[1] if len(sys.argv) > 1 else "f32"
n = 8192
dt = torch.float32 if wl_name == "f32" else torch.bfloat16
a = torch.empty((n, n), dtype=dt, device="cuda")
b = torch.empty((n, n), dtype=dt, device="cuda")
lpsynth.device_fill(a, 1, "uniform", wl_name)
lpsynth.device_fill(b, 2, "uniform", wl_name)
wl = lp.Workload.tmm(a, b, out_dtype=wl_name)
h = lp.LP(128, 128, cksum="mod|xor")
h0 = lp.LP(128, 128, cksum=0)
out, ck, failed, d_n, ws = h.alloc(wl)
out0 = torch.empty_like(out)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
rows = []
for i in range(60):
    prot = i % 2 == 0
    if prot:
        h.cksum_init(wl, ck)
    flush.zero_()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    c0 = clk()
    e0.record()
    if prot:
        h.run_protected(wl, out, ck)
    else:
        h0.run_protected(wl, out0, None)
    e1.record()
    torch.cuda.synchronize()
    rr = rsn()
    rows.append((i, "prot" if prot else "twin", e0.elapsed_time(e1), c0, clk(), pwr(),
                 ",".join(v for k, v in NAMES.items() if rr & k) if rr >= 0 else "?"))
for r in rows:
    print(f"{r[0]:3d} {r[1]} {r[2]:.4f} ms  clk {r[3]}->{r[4]} MHz  {r[5]:.0f} W  reasons [{r[6]}]")
for v in ("prot", "twin"):
    ts = sorted(r[2] for r in rows if r[1] == v and r[0] >= 4)
    print(v, "min", ts[0], "median", statistics.median(ts), "max", ts[-1])
