"""GPU parity of the validate kernel over every warp-task geometry.

The validate kernel maps a strip of G = 32 / LR horizontally adjacent regions onto one warp
(LR = min(32, 16-byte chunks per region row) lanes per region, xor-butterfly or redux.sync
reduction, 2^k chunks per lane per row when a region row is wider than 512 B).  These cases
cover LR = 1 .. 32, 1/2/4 chunks per lane per row, strips that wrap a region row
(Q % G != 0), odd region heights and CTA ranges with a ragged tail, for every checksum
set -- records (lp_region_checksums) and failed lists (lp_validate) against the oracle.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
from paper_conf_iiswc_yudhakzs20_b200 import lp
from tests.gpu_util import dev_to_host, host_to_dev, oracle_validate

pytestmark = pytest.mark.gpu

# (M, N, RM, RN, dtype): row bytes RN*es -> chunks per row 1 .. 128
GEOMS = [
    (24, 4 * 37, 3, 4, "f32"),        # LR=1, G=32, Q=37 (wraps)
    (14, 8 * 40, 7, 8, "f32"),        # LR=2, G=16
    (64, 16 * 24, 1, 16, "f32"),      # LR=4, single-row regions
    (96, 32 * 21, 32, 32, "f32"),     # LR=8, G=4, Q=21
    (130, 64 * 10, 13, 64, "f32"),    # LR=16, G=2, Q odd... 10 (even)
    (256, 128 * 5, 128, 128, "f32"),  # LR=32, G=1
    (64, 256 * 3, 16, 256, "f32"),    # 2 chunks per lane per row
    (32, 512 * 2, 8, 512, "f32"),     # 4 chunks per lane per row
    (64, 32 * 33, 32, 32, "bf16"),    # LR=4, G=8, Q=33
    (384, 128 * 7, 128, 128, "bf16"),  # LR=16, G=2, Q=7 (wraps)
    (40, 256 * 3, 5, 256, "bf16"),    # LR=32
    (16, 1024 * 2, 4, 1024, "bf16"),  # 4 chunks per lane per row
    (2048, 32 * 64, 32, 32, "bf16"),  # many regions: several CTAs, ragged last CTA
    (300 * 7, 128 * 3, 300, 128, "bf16"),  # RM > 256: strip kernel only
    (1536, 128 * 12, 128, 128, "f32"),     # 144 fp32 128x128 regions (64 KiB each): fewer regions than SMs
    (4096, 32 * 96, 32, 32, "f32"),        # G = 8 units (GC = 64), 1536 units over the SMs
]


def _random_out(rng, M, N, dt):
    if dt == "f32":
        return rng.integers(0, 2**32, size=(M, N), dtype=np.uint64).astype(np.uint32).view(np.float32)
    return rng.integers(0, 2**16, size=(M, N), dtype=np.uint64).astype(np.uint16)


@pytest.fixture(params=["fused", "two_launch"])
def kernel_path(request):
    """Tables of R <= 16384 regions are compacted by the last validate CTA (one launch); larger ones by
    a dependent scatter launch.  LP(fused_compact=False) (LP_FLAG_NO_FUSED_COMPACT) forces the two-launch
    form so both compaction paths are checked on every geometry."""
    return request.param


@pytest.mark.parametrize("geom", GEOMS, ids=[f"{g[0]}x{g[1]}_{g[2]}x{g[3]}_{g[4]}" for g in GEOMS])
@pytest.mark.parametrize("mask", ["mod|xor", "mod|xor|adler", "adler"])
def test_validate_geometries(geom, mask, kernel_path):
    M, N, RM, RN, dt = geom
    rng = np.random.default_rng(M * 7919 + N + RM)
    out_h = _random_out(rng, M, N, dt)
    h = lp.LP(RM, RN, cksum=mask, fused_compact=(kernel_path == "fused"))
    wl = lp.Workload.tmm(None, None, out_dtype=dt, m=M, n=N, k=16)
    out = host_to_dev(out_h, dt)
    _, ck, failed, d_n, ws = h.alloc(wl)
    R = h.num_regions(wl)
    sel = oracle.selem(h.mask)
    # records of the current contents == the oracle's (lp_region_checksums = validate MODE 2)
    h.region_checksums(wl, out, ck)
    torch.cuda.synchronize()
    table = dev_to_host(ck)[:R * sel].reshape(R, sel)
    assert np.array_equal(table, oracle.records(out_h, RM, RN, h.mask))
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0
    # corrupt ~15% of the regions (one random word each, every second one also a stale record)
    bad = rng.choice(R, max(1, R * 15 // 100), replace=False)
    Q = N // RN
    words = out_h.view(np.uint32) if dt == "f32" else out_h.view(np.uint16)
    ck_h = dev_to_host(ck).copy()
    for j, r in enumerate(sorted(bad.tolist())):
        p, q = divmod(r, Q)
        i = int(rng.integers(RM))
        c = int(rng.integers(RN))
        words[p * RM + i, q * RN + c] ^= 1 << int(rng.integers(16))
        if j % 2:
            ck_h[r * sel] ^= 0x10
    out.copy_(host_to_dev(out_h, dt))
    ck.copy_(torch.from_numpy(ck_h.view(np.int32)).cuda())
    for _ in range(2):                              # the fused path's ticket is back at zero after each call
        failed.fill_(-1)
        h.validate(wl, out, ck, failed, d_n, ws)
        torch.cuda.synchronize()
        n = int(d_n.item())
        got = failed[:n].cpu().numpy()
        exp = oracle_validate(out_h, ck_h, "array", RM, RN, h.mask)
        assert np.array_equal(got, exp)
    assert set(exp.tolist()) == set(bad.tolist())   # a single bit flip always changes MOD, XOR and Adler


def test_validate_graph_replay_and_large_table():
    """lp_validate captured in a CUDA graph and replayed (the fused ticket resets itself), and a table
    above the fused limit (R = 65536: two-launch path) -- both against the oracle."""
    for M, N, reg in [(2048, 2048, 32), (8192, 8192, 32)]:
        rng = np.random.default_rng(M + reg)
        out_h = _random_out(rng, M, N, "bf16")
        h = lp.LP(reg, reg, cksum="mod|xor")
        wl = lp.Workload.tmm(None, None, out_dtype="bf16", m=M, n=N, k=16)
        out = host_to_dev(out_h, "bf16")
        _, ck, failed, d_n, ws = h.alloc(wl)
        R = h.num_regions(wl)
        h.region_checksums(wl, out, ck)
        ck_h = dev_to_host(ck).copy()
        bad = np.sort(rng.choice(R, 37, replace=False))
        ck_h[bad * 2 + 1] ^= 0x1
        ck.copy_(torch.from_numpy(ck_h.view(np.int32)).cuda())
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            h.validate(wl, out, ck, failed, d_n, ws)          # warm-up outside capture
        torch.cuda.current_stream().wait_stream(s)
        with torch.cuda.graph(g):
            h.validate(wl, out, ck, failed, d_n, ws)
        for _ in range(3):
            failed.fill_(-1)
            d_n.fill_(-1)
            g.replay()
            torch.cuda.synchronize()
            n = int(d_n.item())
            assert n == 37 and np.array_equal(failed[:n].cpu().numpy(), bad), (M, reg)


@pytest.mark.parametrize("R_big", [False, True])
def test_nvls_count_single_gpu_emulation(R_big):
    """lp_attach_nvls_count in its single-GPU emulation (mc == uc, world 1): the CTA that finalises the failed
    count (fused last-CTA compaction for R <= 16384, the scatter launch above) publishes it into the counter
    buffer with the epoch / parity / arrival protocol of the NVLS path; slot 4 must equal the count of every
    successive validate, slot 3 the epoch.  (The multimem.red path itself needs >= 2 NVSwitch-connected GPUs:
    a 1-device multicast object cannot be created.)"""
    from lpsynth import device_fill
    M, N = (2048, 2048) if not R_big else (8192, 8192)
    reg = 32 if R_big else 128
    a = torch.empty((M, 64), dtype=torch.bfloat16, device="cuda")
    b = torch.empty((64, N), dtype=torch.bfloat16, device="cuda")
    device_fill(a, 1, "uniform", "bf16")
    device_fill(b, 2, "uniform", "bf16")
    h = lp.LP(reg, reg, cksum="mod|xor", nvls_count=True)
    wl = lp.Workload.tmm(a, b, out_dtype="bf16")
    out, ck, failed, d_n, ws = h.alloc(wl)
    cnt = torch.zeros(16, dtype=torch.int64, device="cuda")
    h.attach_nvls_count(cnt, cnt, 1)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    R = h.num_regions(wl)
    assert (R > 16384) == R_big
    stale = torch.zeros_like(out)
    for epoch, frac in enumerate([0.0, 0.05, 0.01, 0.2], start=1):
        if frac:
            inj = torch.from_numpy(lp.choose_regions(R, frac, 40 + epoch)).cuda()
            h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=epoch)
        h.validate(wl, out, ck, failed, d_n, ws)
        torch.cuda.synchronize()
        assert int(cnt[4].item()) == int(d_n.item()) and int(cnt[3].item()) == epoch
        h.recover(wl, out, ck, failed, d_n, ws)
    h.attach_nvls_count(None, None, 1)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(cnt[3].item()) == 4 and int(d_n.item()) == 0
