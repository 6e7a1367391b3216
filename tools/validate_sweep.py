"""Time lp_validate (validate kernel + ordered compaction) over region shapes, dtypes and checksum
sets, with two L2 preparations: 'dirty' (write 2x L2 -- the flush leaves dirty lines whose write-back
competes with the validate's reads) and 'clean' (write 2x L2, then read another 2x L2 buffer).
Usage: python tools/validate_sweep.py [--quick]"""
import sys

import torch

sys.path.insert(0, '.')
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402
import os  # noqa: E402

if os.environ.get("LP_AB_LIB"):          # A/B runs: time another build of liblp.so
    lp.LIB_PATH = os.environ["LP_AB_LIB"]

l2 = torch.cuda.get_device_properties(0).L2_cache_size
fw = torch.empty(2 * l2, dtype=torch.uint8, device='cuda')
fr = torch.ones(2 * l2 // 8, dtype=torch.int64, device='cuda')
hbm = 6555.2
try:
    import json
    hbm = json.load(open('MEASURED_PEAKS.json'))['hbm_gbs']
except Exception:
    pass


def flush(kind):
    fw.zero_()
    if kind == 'clean':
        fr.max()


cases = [((8192, 8192), torch.bfloat16, 128, 'mod|xor'), ((8192, 8192), torch.bfloat16, 32, 'mod|xor'),
         ((8192, 8192), torch.float32, 128, 'mod|xor'), ((8192, 8192), torch.bfloat16, 128, 'mod|xor|adler'),
         ((16384, 16384), torch.bfloat16, 128, 'mod|xor'), ((16384, 16384), torch.bfloat16, 32, 'mod|xor'),
         ((32768, 32768), torch.float32, 128, 'mod|xor')]
if '--quick' in sys.argv:
    cases = cases[:3]
for shape, dt, reg, ck_set in cases:
    out = torch.randint(-2**31, 2**31 - 1, (shape[0], shape[1] * dt.itemsize // 4), dtype=torch.int32,
                        device='cuda').view(dt)
    h = lp.LP(reg, reg, cksum=ck_set)
    wl = lp.Workload.tmm(None, None, out_dtype='bf16' if dt == torch.bfloat16 else 'f32', m=shape[0], n=shape[1], k=64)
    _, ck, failed, d_n, ws = h.alloc(wl)
    h.region_checksums(wl, out, ck)   # table = records of the current contents -> 0 failures
    b = out.numel() * out.element_size() + h.cksum_bytes(wl)
    res = {}
    for kind in ('dirty', 'clean'):
        ts = []
        for i in range(14):
            flush(kind)
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            h.validate(wl, out, ck, failed, d_n, ws)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        t = sorted(ts[2:])[len(ts[2:]) // 2]
        res[kind] = t
        assert int(d_n.item()) == 0
    name = f"{shape[0]}x{shape[1]} {str(dt)[6:]} {reg}^2 {ck_set}"
    print(f"{name:40s} dirty {res['dirty']*1e3:7.1f} us {b/res['dirty']/1e6:6.0f} GB/s | clean {res['clean']*1e3:7.1f} us "
          f"{b/res['clean']/1e6:6.0f} GB/s ({b/res['clean']/1e6/hbm*100:5.1f}% of {hbm:.0f})", flush=True)
