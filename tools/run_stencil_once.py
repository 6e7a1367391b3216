"""Run the protected and unprotected stencil 32768^2 once each (for ncu)."""
import sys, torch
sys.path.insert(0, '.')
import lpsynth
from paper_conf_iiswc_yudhakzs20_b200 import lp
H = W = 32768
x = torch.empty((H, W), dtype=torch.float32, device='cuda'); lpsynth.device_fill(x, 1, 'uniform', 'f32')
for mask in [int(a) for a in (sys.argv[1:] or ['3', '0'])]:
    h = lp.LP(128, 128, cksum=mask)
    wl = lp.Workload.stencil(x)
    out, ck, failed, d_n, ws = h.alloc(wl)
    if mask: h.cksum_init(wl, ck)
    for _ in range(2):
        h.run_protected(wl, out, ck if mask else None)
    torch.cuda.synchronize()
