import sys, torch
sys.path.insert(0, ".")
import lpsynth
from paper_conf_iiswc_yudhakzs20_b200 import lp
store, reg, n, k = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
a = torch.empty((n, k), dtype=torch.bfloat16, device="cuda"); b = torch.empty((k, n), dtype=torch.bfloat16, device="cuda")
lpsynth.device_fill(a, 1, "int5", "bf16"); lpsynth.device_fill(b, 2, "int5", "bf16")
h = lp.LP(reg, reg, cksum="mod|xor", store=store)
wl = lp.Workload.tmm(a, b, out_dtype="bf16")
out, ck, failed, d_n, ws = h.alloc(wl)
h.cksum_init(wl, ck); h.run_protected(wl, out, ck); torch.cuda.synchronize()
print("ok", sys.argv[1:], flush=True)
