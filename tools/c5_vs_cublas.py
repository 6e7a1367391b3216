#!/usr/bin/env python
"""C5 body (TMM 65536^3 bf16 -> bf16, 128x128 regions, MOD|XOR) vs its unprotected twin vs cuBLAS
(torch.matmul, bf16) at the same shape, interleaved, under the same power cap.  CUDA-event times with the
NVML SM clock (median of 10 ms samples during each run) and throttle reasons."""
import statistics
import sys
import threading
import time

import torch

sys.path.insert(0, ".")
import lpsynth  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

import pynvml  # noqa: E402

pynvml.nvmlInit()
hnd = pynvml.nvmlDeviceGetHandleByIndex(0)
n = int(sys.argv[1]) if len(sys.argv) > 1 else 65536
a = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
b = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
lpsynth.device_fill(a, 1, "uniform", "bf16")
lpsynth.device_fill(b, 2, "uniform", "bf16")
wl = lp.Workload.tmm(a, b, out_dtype="bf16")
h = lp.LP(128, 128, cksum="mod|xor")
h0 = lp.LP(128, 128, cksum=0)
out, ck, failed, d_n, ws = h.alloc(wl)
c = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
flops = 2.0 * n ** 3


def run(name):
    samples, stop = [], [False]

    def poll():
        while not stop[0]:
            samples.append((pynvml.nvmlDeviceGetClockInfo(hnd, pynvml.NVML_CLOCK_SM),
                            pynvml.nvmlDeviceGetCurrentClocksEventReasons(hnd)))
            time.sleep(0.01)
    th = threading.Thread(target=poll, daemon=True)
    if name == "lp":
        h.cksum_init(wl, ck)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    th.start()
    e0.record()
    if name == "lp":
        h.run_protected(wl, out, ck)
    elif name == "twin":
        h0.run_protected(wl, out, None)
    else:
        torch.matmul(a, b, out=c)
    e1.record()
    torch.cuda.synchronize()
    stop[0] = True
    th.join()
    t = e0.elapsed_time(e1)
    mhz = statistics.median(s[0] for s in samples) if samples else -1
    cap = sum(1 for s in samples if s[1] & 0x4)
    return t, mhz, cap, len(samples)


for name in ("lp", "twin", "cublas"):
    run(name)  # warm-up (module load, cuBLAS heuristics)
res = {"lp": [], "twin": [], "cublas": []}
for rep in range(3):
    for name in ("lp", "twin", "cublas"):
        t, mhz, cap, ns = run(name)
        res[name].append((t, mhz))
        print(f"rep {rep} {name:6s} {t:8.1f} ms  {flops / t / 1e9:7.1f} TFLOP/s  SM {mhz} MHz  sw_power_cap {cap}/{ns} samples",
              flush=True)
for name, v in res.items():
    t = statistics.median(x[0] for x in v)
    print(f"{name:6s} median {t:.1f} ms = {flops / t / 1e9:.1f} TFLOP/s, median SM clock "
          f"{statistics.median(x[1] for x in v)} MHz")
tl = statistics.median(x[0] for x in res["lp"])
tc = statistics.median(x[0] for x in res["cublas"])
print(f"LP-protected body / cuBLAS time = {tl / tc:.3f}")
