"""Time of the Listing 7 TMM kernel on a CLEAN image (check phase only, no recompute) vs lp_validate, 8192^3 bf16."""
import sys

import torch

sys.path.insert(0, ".")
import lpsynth  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

n = 8192
for reg in (128, 32):
    a = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
    b = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
    lpsynth.device_fill(a, 1, "uniform", "bf16")
    lpsynth.device_fill(b, 2, "uniform", "bf16")
    h = lp.LP(reg, reg, cksum="mod|xor")
    wl = lp.Workload.tmm(a, b, out_dtype="bf16")
    out, ck, failed, d_n, ws = h.alloc(wl)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    d_rec = torch.zeros(1, dtype=torch.int64, device="cuda")
    for name in ("validate", "check_static", "check_balanced"):
        ts = []
        for _ in range(9):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if name == "validate":
                h.validate(wl, out, ck, failed, d_n, ws)
            elif name == "check_static":
                h.check_recover(wl, out, ck, d_rec)
            else:
                h.check_recover(wl, out, ck, d_rec, workspace=ws)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        print(f"reg {reg} {name:15s} median {sorted(ts)[4] * 1e3:.1f} us", flush=True)
