import sys, time
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_iiswc_yudhakzs20_b200 import lp
from tests.gpu_util import dev_to_host, host_to_dev, make_inputs
store = sys.argv[1] if len(sys.argv) > 1 else "cuckoo"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 16384
reg = int(sys.argv[3]) if len(sys.argv) > 3 else 32
h = lp.LP(reg, reg, cksum="mod|xor", store=store)
A, B = make_inputs(41, n, n, 64, "int5", "bf16")
a, b = host_to_dev(A, "bf16"), host_to_dev(B, "bf16")
wl = lp.Workload.tmm(a, b, out_dtype="bf16")
out, ck, failed, d_n, ws = h.alloc(wl)
h.cksum_init(wl, ck); torch.cuda.synchronize(); print("init", flush=True)
t = time.time(); h.run_protected(wl, out, ck); torch.cuda.synchronize(); print("run", time.time() - t, flush=True)
ck_h = dev_to_host(ck); print("header cap seed lock err coll stash rehash", ck_h[:9], flush=True)
d_stats = torch.zeros(2, dtype=torch.int64, device=out.device)
h.stats(wl, ck, d_stats); torch.cuda.synchronize(); print("stats", d_stats.tolist(), flush=True)
h.validate(wl, out, ck, failed, d_n, ws); torch.cuda.synchronize(); print("validate", int(d_n.item()), flush=True)
