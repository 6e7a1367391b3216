"""Probe: does tcgen05 kind::tf32 ignore the low 13 mantissa bits of its 32-bit operands?  The fp32 3xTF32 TMM is
run with the normal build (hi = x & 0xFFFFE000) and with LP_TF32_RAW_HI_PROBE=1 (hi = the raw fp32 word), on
random inputs; identical output bits => the hardware truncates (the masking is redundant).
usage: python tools/probe/tf32_raw_hi.py <out.npy>"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import lpsynth
from paper_conf_iiswc_yudhakzs20_b200 import lp

M = N = 512
K = 1024
a = torch.empty((M, K), dtype=torch.float32, device="cuda")
b = torch.empty((K, N), dtype=torch.float32, device="cuda")
lpsynth.device_fill(a, 1, "uniform", "f32")
lpsynth.device_fill(b, 2, "uniform", "f32")
h = lp.LP(128, 128, cksum="mod|xor", body="tcgen05")
wl = lp.Workload.tmm(a, b, out_dtype="f32")
out, ck, *_ = h.alloc(wl)
h.cksum_init(wl, ck)
h.run_protected(wl, out, ck)
torch.cuda.synchronize()
np.save(sys.argv[1], out.cpu().numpy())
ref = (a.double() @ b.double()).cpu().numpy()
print("relerr", float(np.abs(out.cpu().numpy() - ref).max() / np.abs(ref).max()))
