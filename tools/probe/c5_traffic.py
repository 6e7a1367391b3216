"""One LP-protected body and one cuBLAS GEMM at n^3 bf16 (for an ncu traffic comparison)."""
import sys

import torch

sys.path.insert(0, ".")
import lpsynth  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

n = int(sys.argv[1])
a = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
b = torch.empty((n, n), dtype=torch.bfloat16, device="cuda")
lpsynth.device_fill(a, 1, "uniform", "bf16")
lpsynth.device_fill(b, 2, "uniform", "bf16")
wl = lp.Workload.tmm(a, b, out_dtype="bf16")
h = lp.LP(128, 128, cksum="mod|xor")
out, ck, failed, d_n, ws = h.alloc(wl)
h.cksum_init(wl, ck)
h.run_protected(wl, out, ck)
c = torch.matmul(a, b)
torch.cuda.synchronize()
