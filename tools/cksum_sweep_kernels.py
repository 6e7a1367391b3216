#!/usr/bin/env python
"""Launches the protected region body once per checksum set (and the unprotected twin), for an ncu metric sweep:
protected vs twin per checksum type (tensor-pipe %, ALU %, extra DRAM writes = the E9
write-amplification analog, L587/L589).  Every body is launched twice (warm-up, then the profiled launch) after an
L2 flush; the marker kernels' order is: for mask in MASKS: [flush, body(mask), flush, body(mask)].

  --workload tmm    : C2 TMM 8192^3 bf16 -> bf16, 128x128 regions (tmm_tc2_kernel)
  --workload tmmf32 : C2 TMM 8192^3 fp32 -> fp32 via 3xTF32, 128x128 regions (tmm_tf32x3_kernel)
  --workload stencil: C4 stencil 32768^2 fp32, 128x128 regions (stencil5_ldg_kernel)
"""
import argparse
import sys

import torch

sys.path.insert(0, ".")
import lpsynth  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

MASKS = [0, 1, 2, 3, 4, 7]

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="tmm", choices=["tmm", "tmmf32", "stencil"])
args = ap.parse_args()
if args.workload == "stencil":
    x = torch.empty((32768, 32768), dtype=torch.float32, device="cuda")
    lpsynth.device_fill(x, 1, "uniform", "f32")
    wl = lp.Workload.stencil(x)
else:
    dt = torch.bfloat16 if args.workload == "tmm" else torch.float32
    name = "bf16" if args.workload == "tmm" else "f32"
    a = torch.empty((8192, 8192), dtype=dt, device="cuda")
    b = torch.empty((8192, 8192), dtype=dt, device="cuda")
    lpsynth.device_fill(a, 1, "uniform", name)
    lpsynth.device_fill(b, 2, "uniform", name)
    wl = lp.Workload.tmm(a, b, out_dtype=name)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
for mask in MASKS:
    h = lp.LP(128, 128, cksum=mask)
    out, ck, failed, d_n, ws = h.alloc(wl)
    for _ in range(2):
        if mask:
            h.cksum_init(wl, ck)
        flush.zero_()
        h.run_protected(wl, out, ck if mask else None)
    torch.cuda.synchronize()
    del out, ck, failed, d_n, ws
print("masks", MASKS)
