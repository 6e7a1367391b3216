"""Time lp_validate (validate + compaction) at the bench's TMM and stencil sizes, cold L2."""
import sys, torch
sys.path.insert(0, '.')
import lpsynth
from paper_conf_iiswc_yudhakzs20_b200 import lp
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
for name, shape, dt, reg in [('tmm8192_bf16', (8192, 8192), torch.bfloat16, 128), ('r32_16384', (16384, 16384), torch.bfloat16, 32),
                             ('stencil32768', (32768, 32768), torch.float32, 128)]:
    out = torch.empty(shape, dtype=dt, device='cuda')
    h = lp.LP(reg, reg, cksum='mod|xor')
    wl = lp.Workload.tmm(None, None, out_dtype='bf16' if dt == torch.bfloat16 else 'f32', m=shape[0], n=shape[1], k=64)
    _, ck, failed, d_n, ws = h.alloc(wl)
    h.region_checksums(wl, out, ck)   # table = records of the current contents -> 0 failures
    ts = []
    for i in range(12):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); h.validate(wl, out, ck, failed, d_n, ws); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    t = sorted(ts[2:])[len(ts[2:]) // 2]
    b = out.numel() * out.element_size()
    print(f"{name}: validate {t*1e3:.1f} us  {b/t/1e6:.0f} GB/s  failed={int(d_n.item())}", flush=True)
