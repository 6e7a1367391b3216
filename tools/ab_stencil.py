"""A/B timing of stencil variants (protected MOD|XOR vs unprotected), L2 flushed, CUDA events."""
import sys, torch
sys.path.insert(0, '.')
import lpsynth
from paper_conf_iiswc_yudhakzs20_b200 import lp
H = W = 32768
x = torch.empty((H, W), dtype=torch.float32, device='cuda'); lpsynth.device_fill(x, 1, 'uniform', 'f32')
flush = torch.empty(512 << 20, dtype=torch.uint8, device='cuda')
variants = [int(v) for v in (sys.argv[1:] or ['0', '1', '2'])]
outs = {}
for var in variants:
    res = {}
    for mask in [0, 3]:
        h = lp.LP(128, 128, cksum=mask)
        wl = lp.Workload.stencil(x)
        out, ck, failed, d_n, ws = h.alloc(wl)
        if mask: h.cksum_init(wl, ck)
        ts = []
        for i in range(15):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); h.run_protected(wl, out, ck if mask else None); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        t = sorted(ts[3:])[len(ts[3:]) // 2]
        res[mask] = t
        outs[(var, mask)] = out.clone()
    print(f"variant {var}: unprot {res[0]*1e3:7.1f} us ({2*H*W*4/res[0]/1e6:6.0f} GB/s)  prot {res[3]*1e3:7.1f} us ({2*H*W*4/res[3]/1e6:6.0f} GB/s)  overhead {100*(res[3]/res[0]-1):5.2f}%", flush=True)
ref = outs[(variants[0], 3)]
print("all variants identical:", all(torch.equal(v, ref) for v in outs.values()))
