"""C5 (65536^3 bf16, 128x128 regions): protected vs unprotected twin in alternating order (PTTP...), SM clock via
NVML around each run, to see whether the bench's +0.5..5.6% LP overhead at this size is systematic."""
import sys
import time

import torch

sys.path.insert(0, ".")
import lpsynth
from paper_conf_iiswc_yudhakzs20_b200 import lp

try:
    import pynvml
    pynvml.nvmlInit()
    nv = pynvml.nvmlDeviceGetHandleByIndex(0)
    clk = lambda: pynvml.nvmlDeviceGetClockInfo(nv, pynvml.NVML_CLOCK_SM)
except Exception:
    clk = lambda: -1
M = N = K = 65536
a = torch.empty((M, K), dtype=torch.bfloat16, device="cuda")
b = torch.empty((K, N), dtype=torch.bfloat16, device="cuda")
lpsynth.device_fill(a, 1, "uniform", "bf16")
lpsynth.device_fill(b, 2, "uniform", "bf16")
hp = lp.LP(128, 128, cksum="mod|xor")
ht = lp.LP(128, 128, cksum=0)
wl = lp.Workload.tmm(a, b, out_dtype="bf16")
out, ck, *_ = hp.alloc(wl)


def run(h, c):
    if c is not None:
        h.cksum_init(wl, c)
    torch.cuda.synchronize()
    c0 = clk()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    h.run_protected(wl, out, c)
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1), c0, clk()


run(hp, ck)
run(ht, None)
order = [1, 0, 0, 1] * 4
for i, prot in enumerate(order):
    t, c0, c1 = run(hp, ck) if prot else run(ht, None)
    print(f"{i:2d} {'prot' if prot else 'twin'} {t:8.2f} ms  SM {c0}->{c1} MHz", flush=True)
