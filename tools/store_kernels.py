#!/usr/bin/env python
"""Launches the protected C3 body (TMM 16384^3 bf16 -> bf16, MOD|XOR) once per checksum store after a fresh table
init, for an ncu comparison of the stores' atomic traffic (collisions +
l1tex__t_bytes_pipe_lsu_mem_global_op_atom).  --region 128 (R = 16384) or 32 (R = 262144)."""
import argparse
import sys

import torch

sys.path.insert(0, ".")
import lpsynth  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--region", type=int, default=128)
ap.add_argument("--n", type=int, default=16384)
args = ap.parse_args()
n = args.n
a = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
b = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
lpsynth.device_fill(a, 1, "uniform", "bf16")
lpsynth.device_fill(b, 2, "uniform", "bf16")
wl = lp.Workload.tmm(a, b, out_dtype="bf16")
for store in ("array", "quad_cas", "cuckoo", "quad_lock"):
    h = lp.LP(args.region, args.region, cksum="mod|xor", store=store)
    out, ck, failed, d_n, ws = h.alloc(wl)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    print(store, "done", flush=True)
