#!/usr/bin/env python
"""N2: the paper's same-grid check-and-recover kernel (Listing 7) vs validate -> compact -> list-mode
relaunch, on the C4 stencil (32768^2 fp32, 128x128 regions, MOD|XOR) at 1/10/50% STALE_REGION crashes.
Times are CUDA-event medians of 7 reps, L2 flushed; each rep starts from the same corrupted image."""
import sys

import torch

sys.path.insert(0, ".")
import lpsynth  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

H = W = 32768
x = torch.empty((H, W), dtype=torch.float32, device="cuda")
lpsynth.device_fill(x, 1, "uniform", "f32")
h = lp.LP(128, 128, cksum="mod|xor")
wl = lp.Workload.stencil(x)
out, ck, failed, d_n, ws = h.alloc(wl)
h.cksum_init(wl, ck)
h.run_protected(wl, out, ck)
golden = out.clone()
stale = torch.empty_like(out)
lpsynth.device_fill(stale.view(torch.int32), 3, "bits", "u32")
R = h.num_regions(wl)
flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
bad_img = torch.empty_like(out)
ck_img = torch.empty_like(ck)
d_rec = torch.zeros(1, dtype=torch.int64, device="cuda")
print("| crash fraction | failed regions | validate + compact + relaunch (ms) | same-grid check-and-recover (ms) | ratio |")
print("|---|---|---|---|---|")
for frac in (0.01, 0.10, 0.50):
    inj = torch.from_numpy(lp.choose_regions(R, frac, 77)).cuda()
    out.copy_(golden)
    h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=77)
    bad_img.copy_(out)
    ck_img.copy_(ck)
    res = {}
    for name in ("ours", "listing7"):
        ts = []
        for _ in range(7):
            out.copy_(bad_img)
            ck.copy_(ck_img)
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if name == "ours":
                h.validate(wl, out, ck, failed, d_n, ws)
                h.recover(wl, out, ck, failed, d_n, ws)
            else:
                h.check_recover(wl, out, ck, d_rec)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
            assert torch.equal(out, golden)
        res[name] = sorted(ts)[3]
    n = int(d_n.item())
    print(f"| {frac:.0%} | {n} | {res['ours']:.3f} | {res['listing7']:.3f} | {res['listing7'] / res['ours']:.2f} |",
          flush=True)
