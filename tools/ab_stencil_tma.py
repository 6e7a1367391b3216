"""A/B timing of the stencil 32768^2 full run per checksum set (env knobs select the kernel form):
median of adjacent (protected, twin) pairs, L2 flushed before every run.
python tools/ab_stencil_tma.py [masks...]"""
import os
import sys

import torch

sys.path.insert(0, '.')
import lpsynth
from paper_conf_iiswc_yudhakzs20_b200 import lp

H = W = 32768
x = torch.empty((H, W), dtype=torch.float32, device='cuda')
lpsynth.device_fill(x, 1, 'uniform', 'f32')
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
tag = ' '.join(f'{k}={v}' for k, v in sorted(os.environ.items()) if k.startswith('LP_STENCIL'))


def t_run(h, wl, out, ck):
    flush.zero_()
    if ck is not None:
        h.cksum_init(wl, ck)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    h.run_protected(wl, out, ck)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1)


twin = lp.LP(128, 128, cksum=0)
wl = lp.Workload.stencil(x)
tout, _, _, _, _ = twin.alloc(wl)
for mask in [int(a) for a in (sys.argv[1:] or ['3', '4', '7'])]:
    h = lp.LP(128, 128, cksum=mask)
    out, ck, _, _, _ = h.alloc(wl)
    for _ in range(3):
        t_run(h, wl, out, ck)
        t_run(twin, wl, tout, None)
    tp, tu, ratios = [], [], []
    for i in range(12):
        if i % 2 == 0:
            a = t_run(h, wl, out, ck); b = t_run(twin, wl, tout, None)
        else:
            b = t_run(twin, wl, tout, None); a = t_run(h, wl, out, ck)
        tp.append(a); tu.append(b); ratios.append(a / b - 1)
    med = lambda v: sorted(v)[len(v) // 2]
    print(f'{tag} mask={mask} prot={med(tp):.4f} ms twin={med(tu):.4f} ms overhead={100 * med(ratios):+.2f}% '
          f'GB/s={2 * H * W * 4 / med(tp) / 1e6:.0f}', flush=True)
