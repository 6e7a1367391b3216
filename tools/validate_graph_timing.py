"""How much of lp_validate's measured time is the validate kernel itself?
Times, cold L2 (clean lines), for the bench's three output shapes:
  eager   = events around an eager lp_validate call (validate kernel + PDL compaction scatter)
  graph   = events around the replay of a CUDA graph holding that one lp_validate call
  records = events around lp_region_checksums (the validate kernel in record-writing mode: same
            reads, no compare/flags/compaction) -- a lower bound for the kernel alone.
Usage: python tools/validate_graph_timing.py"""
import sys

import torch

sys.path.insert(0, '.')
from paper_conf_iiswc_yudhakzs20_b200 import lp  # noqa: E402

l2 = torch.cuda.get_device_properties(0).L2_cache_size
fw = torch.empty(2 * l2, dtype=torch.uint8, device='cuda')
fr = torch.ones(2 * l2 // 8, dtype=torch.int64, device='cuda')


def flush():
    fw.zero_()
    fr.max()


def med(x):
    x = sorted(x)
    return x[len(x) // 2]


def timed(fn, reps=15):
    ts = []
    for _ in range(reps):
        flush()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return med(ts[3:]) * 1e3


for name, shape, dt, rm, rn in [('tmm8192_bf16', (8192, 8192), 'bf16', 128, 128),
                                ('tmm8192_f32', (8192, 8192), 'f32', 128, 128),
                                ('spmv4m_y', (4096, 1024), 'f32', 1, 1024),
                                ('stencil32768', (32768, 32768), 'f32', 128, 128)]:
    tdt = torch.bfloat16 if dt == 'bf16' else torch.float32
    out = torch.randn(shape, device='cuda').to(tdt)
    h = lp.LP(rm, rn, cksum='mod|xor')
    wl = lp.Workload.tmm(None, None, out_dtype=dt, m=shape[0], n=shape[1], k=64)
    _, ck, failed, d_n, ws = h.alloc(wl)
    h.region_checksums(wl, out, ck)
    recs = torch.empty_like(ck)
    torch.cuda.synchronize()
    te = timed(lambda: h.validate(wl, out, ck, failed, d_n, ws))
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.current_stream().wait_stream(s)
    with torch.cuda.graph(g):
        h.validate(wl, out, ck, failed, d_n, ws)
    tg = timed(g.replay)
    tr = timed(lambda: h.region_checksums(wl, out, recs))
    b = out.numel() * out.element_size() + ck.numel() * ck.element_size()
    print(f"{name:14s} {b / 2**20:8.1f} MiB  eager {te:7.1f} us ({b / te / 1e3:6.0f} GB/s)  graph {tg:7.1f} us "
          f"({b / tg / 1e3:6.0f} GB/s)  records {tr:7.1f} us ({b / tr / 1e3:6.0f} GB/s)  failed={int(d_n.item())}",
          flush=True)
