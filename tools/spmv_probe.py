"""Tiny SpMV probe: one protected run per case, prints max error vs a float64 CSR product.
python tools/spmv_probe.py"""
import sys

import numpy as np
import torch

sys.path.insert(0, '.')
from lpsynth import csr, gen  # noqa: E402
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

for rows, RN, lens_kind in [(4096, 1024, 'recipe'), (256, 16, 'short'), (2048, 256, 'mixed')]:
    rng = np.random.default_rng(rows)
    if lens_kind == 'recipe':
        rp = csr.row_ptr(5, rows)
    else:
        lens = rng.integers(0, 4, rows) if lens_kind == 'short' else rng.choice([0, 1, 2, 9, 300, 3000], rows)
        rp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    nnz = int(rp[-1])
    cols = rng.integers(0, rows, nnz).astype(np.int32)
    vals = gen.values_f32(7, 1, nnz, 'uniform')[0]
    x = gen.values_f32(8, 1, rows, 'uniform')[0]
    ref = np.array([np.dot(vals[rp[i]:rp[i + 1]].astype(np.float64), x[cols[rp[i]:rp[i + 1]]].astype(np.float64))
                    for i in range(rows)])
    h = lp.LP(1, RN, cksum='mod|xor')
    wl = lp.Workload.spmv(torch.from_numpy(vals).cuda(), torch.from_numpy(x).cuda(), torch.from_numpy(rp).cuda(),
                          torch.from_numpy(cols).cuda())
    out, ck, failed, d_n, ws = h.alloc(wl)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    y = out.cpu().numpy().reshape(-1).astype(np.float64)
    err = np.abs(y - ref).max() / max(np.abs(ref).max(), 1e-30)
    bad = np.nonzero(np.abs(y - ref) > 1e-5 * max(np.abs(ref).max(), 1e-30))[0]
    print(f"rows={rows} RN={RN} {lens_kind}: nnz={nnz} relerr={err:.2e} bad_rows={bad[:10]}", flush=True)
