"""A/B of lp_validate between two liblp builds (graph-differential timing, cold L2), run in separate
processes: python tools/ab_validate_libs.py <lib>   (prints one line per size)"""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_iiswc_yudhakzs20_b200.lp as lp  # noqa: E402

lp.LIB_PATH = sys.argv[1]
l2 = torch.cuda.get_device_properties(0).L2_cache_size
fw = torch.empty(2 * l2, dtype=torch.uint8, device="cuda")
fr = torch.ones(2 * l2 // 8, dtype=torch.int64, device="cuda")


def flush():
    fw.zero_()
    fr.max()


def graph_diff(fn, n=8, reps=7):
    gs = []
    for with_k in (False, True):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(n):
                flush()
                if with_k:
                    fn()
        gs.append(g)
    ds = []
    for _ in range(reps):
        tt = []
        for g in gs:
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            g.replay()
            e1.record()
            torch.cuda.synchronize()
            tt.append(e0.elapsed_time(e1))
        ds.append((tt[1] - tt[0]) / n)
    return sorted(ds)[len(ds) // 2] * 1e3


for name, shape, dt, reg in [("bf16 8192^2 128^2", (8192, 8192), "bf16", 128), ("bf16 8192^2 32^2", (8192, 8192), "bf16", 32),
                             ("f32 32768^2 128^2", (32768, 32768), "f32", 128)]:
    out = torch.randn(shape, device="cuda").to(torch.bfloat16 if dt == "bf16" else torch.float32)
    h = lp.LP(reg, reg, cksum="mod|xor")
    wl = lp.Workload.tmm(None, None, out_dtype=dt, m=shape[0], n=shape[1], k=64)
    _, ck, failed, d_n, ws = h.alloc(wl)
    h.region_checksums(wl, out, ck)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    t = graph_diff(lambda: h.validate(wl, out, ck, failed, d_n, ws))
    b = out.numel() * out.element_size()
    print(f"{sys.argv[1][-28:]:28s} {name:20s} {t:8.1f} us {b / t / 1e3:7.0f} GB/s", flush=True)
    del out
