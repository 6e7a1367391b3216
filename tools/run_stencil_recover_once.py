"""Stencil 32768^2 MOD|XOR: protected run, 10% of regions crashed (stale words), validate, list-mode recovery
(for ncu: the stencil launches are body, recovery, body, recovery -- -s 1 -c 1 catches the first recovery).
python tools/run_stencil_recover_once.py [frac]"""
import sys

import torch

sys.path.insert(0, '.')
import lpsynth
from paper_conf_iiswc_yudhakzs20_b200 import lp

frac = float(sys.argv[1]) if len(sys.argv) > 1 else 0.1
H = W = 32768
x = torch.empty((H, W), dtype=torch.float32, device='cuda')
lpsynth.device_fill(x, 1, 'uniform', 'f32')
h = lp.LP(128, 128, cksum=3)
wl = lp.Workload.stencil(x)
out, ck, failed, d_n, ws = h.alloc(wl)
stale = torch.empty_like(out)
lpsynth.device_fill(stale.view(torch.int32), 3, 'bits', 'u32')
R = h.num_regions(wl)
inj = torch.from_numpy(lp.choose_regions(R, frac, 1000)).cuda()
for _ in range(2):
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    h.inject(wl, out, ck, stale, inj, mode='stale_words', seed=1000)
    h.validate(wl, out, ck, failed, d_n, ws)
    h.recover(wl, out, ck, failed, d_n, ws)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
out.copy_(stale)
h.cksum_init(wl, ck)
h.run_protected(wl, out, ck)
h.inject(wl, out, ck, stale, inj, mode='stale_words', seed=1000)
h.validate(wl, out, ck, failed, d_n, ws)
torch.empty(512 << 20, dtype=torch.uint8, device='cuda').zero_()
e0.record()
h.recover(wl, out, ck, failed, d_n, ws)
e1.record()
torch.cuda.synchronize()
n = len(inj)
print(f'recover of {n} regions: {e0.elapsed_time(e1) * 1e3:.1f} us, '
      f'{n * (130 * 130 * 4 + 128 * 128 * 4) / e0.elapsed_time(e1) / 1e6:.0f} GB/s')
