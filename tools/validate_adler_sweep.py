"""lp_validate with MOD|XOR|ADLER32 records at 128 MiB .. 4 GiB, cold L2 (run once with LP_VAL_ADLER_BIG=0 -> the
3-CTA/SM build everywhere, once with LP_VAL_ADLER_BIG=100000 -> the 4-CTA/SM build everywhere)."""
import os, sys, torch
sys.path.insert(0, '.')
from paper_conf_iiswc_yudhakzs20_b200 import lp
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
tag = os.environ.get('LP_VAL_ADLER_BIG', 'default')
for name, shape, dt, reg in [('8192^2 bf16', (8192, 8192), torch.bfloat16, 128), ('8192^2 f32', (8192, 8192), torch.float32, 128),
                             ('16384^2 bf16', (16384, 16384), torch.bfloat16, 128), ('16384^2 f32', (16384, 16384), torch.float32, 128),
                             ('16384^2 bf16 r32', (16384, 16384), torch.bfloat16, 32), ('32768^2 f32', (32768, 32768), torch.float32, 128)]:
    lo, hi = (-2**31, 2**31 - 1) if dt == torch.float32 else (-2**15, 2**15 - 1)
    out = torch.randint(lo, hi, shape, dtype=torch.int32 if dt == torch.float32 else torch.int16, device='cuda').view(dt)
    h = lp.LP(reg, reg, cksum='mod|xor|adler')
    wl = lp.Workload.tmm(None, None, out_dtype='bf16' if dt == torch.bfloat16 else 'f32', m=shape[0], n=shape[1], k=64)
    _, ck, failed, d_n, ws = h.alloc(wl)
    h.region_checksums(wl, out, ck)
    ts = []
    for i in range(12):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); h.validate(wl, out, ck, failed, d_n, ws); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    t = sorted(ts[2:])[len(ts[2:]) // 2]
    b = out.numel() * out.element_size()
    assert int(d_n.item()) == 0
    print(f"BIG={tag} {name}: validate {t*1e3:.1f} us  {b/t/1e6:.0f} GB/s", flush=True)
    del out, ck, failed, ws
