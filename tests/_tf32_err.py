import sys, numpy as np, torch
sys.path.insert(0, '.')
import oracle, lpsynth
from lpsynth import gen
from paper_conf_iiswc_yudhakzs20_b200 import lp
from tests.gpu_util import dev_to_host
M=N=512
for K in [1024, 2048, 4096, 8192]:
    a = torch.empty((M,K), dtype=torch.float32, device='cuda'); b = torch.empty((K,N), dtype=torch.float32, device='cuda')
    lpsynth.device_fill(a, 1, 'uniform', 'f32'); lpsynth.device_fill(b, 2, 'uniform', 'f32')
    A = dev_to_host(a); B = dev_to_host(b)
    ref = oracle.gemm_block_f64(A, B, 0, 0, 256, 256)
    line = f"K={K}"
    for body in ['simt', 'tcgen05']:
        h = lp.LP(128,128,cksum='mod',body=body)
        wl = lp.Workload.tmm(a,b,out_dtype='f32')
        out,ck,*_ = h.alloc(wl); h.cksum_init(wl,ck); h.run_protected(wl,out,ck); torch.cuda.synchronize()
        got = dev_to_host(out)[:256,:256]
        d = got.astype(np.float64) - ref
        line += f"  {body}: relerr {oracle.rel_err(got, ref):.2e} mean(d) {d.mean():+.2e} std(d) {d.std():.2e}"
    print(line, flush=True)
