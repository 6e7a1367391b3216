"""GPU parity: lp_recover_revalidate -- recovery (a10) followed by the re-validation of the whole output (a11),
with the regions the previous validate did not flag re-validated on a side stream beside the recovery and the
failed list after it.  Final state and count must equal lp_recover + lp_validate; a clean region corrupted
after the first validate must be counted by the side path, and (test hook: no re-execution) every listed
region by the list path."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import lpsynth
from lpsynth import gen
from paper_conf_iiswc_yudhakzs20_b200 import lp
from tests.gpu_util import dev_to_host, host_to_dev, make_inputs, stale_image

pytestmark = pytest.mark.gpu


def _setup(kind, mask, reg, test_skip=False):
    h = lp.LP(reg, reg, cksum=mask, test_skip_reexec=test_skip)
    if kind == "stencil":
        H, W = 1024, 768
        x = host_to_dev(gen.generate(7, H, W, "uniform", "f32"), "f32")
        wl = lp.Workload.stencil(x)
        out_dt = "f32"
    else:
        M, N, K = (512, 768, 256)
        in_dt, out_dt, body = {"tmm_bf16": ("bf16", "bf16", "tcgen05"), "tmm_f32": ("f32", "f32", "tcgen05"),
                               "tmm_i32": ("i32", "i32", "simt")}[kind]
        h = lp.LP(reg, reg, cksum=mask, body=body, test_skip_reexec=test_skip)
        A, B = make_inputs(3, M, N, K, "int5" if in_dt != "i32" else "int17", in_dt)
        wl = lp.Workload.tmm(host_to_dev(A, in_dt), host_to_dev(B, in_dt), out_dtype=out_dt)
        H, W = M, N
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = host_to_dev(stale_image(5, H, W, out_dt), out_dt)
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    return h, wl, out, ck, failed, d_n, ws, stale


@pytest.mark.parametrize("kind,reg", [("stencil", 128), ("tmm_bf16", 128), ("tmm_i32", 32)])
@pytest.mark.parametrize("mask", ["mod|xor", "mod|xor|adler"])
@pytest.mark.parametrize("frac", [0.0, 0.2, 1.0])
def test_recover_revalidate_equals_sequential(kind, reg, mask, frac):
    h, wl, out, ck, failed, d_n, ws, stale = _setup(kind, mask, reg)
    golden, ck_golden = dev_to_host(out), dev_to_host(ck)
    R = h.num_regions(wl)
    inj = torch.from_numpy(lp.choose_regions(R, frac, 11)).cuda()
    h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=11)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    nf = int(d_n.item())
    assert nf == inj.numel()
    after = torch.full((1,), -1, dtype=torch.int64, device="cuda")
    rec = torch.zeros(1, dtype=torch.int64, device="cuda")
    h.recover_revalidate(wl, out, ck, failed, d_n, ws, after, d_n_recovered=rec)
    torch.cuda.synchronize()
    assert int(after.item()) == 0
    assert int(rec.item()) >= nf
    assert np.array_equal(dev_to_host(out).view(np.uint8), golden.view(np.uint8))
    assert np.array_equal(dev_to_host(ck), ck_golden)
    # the same state validates clean through the plain path
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0


@pytest.mark.parametrize("kind,reg", [("stencil", 128), ("tmm_bf16", 128), ("tmm_i32", 32)])
def test_side_path_counts_a_clean_region_corrupted_after_validate(kind, reg):
    h, wl, out, ck, failed, d_n, ws, stale = _setup(kind, "mod|xor", reg)
    R = h.num_regions(wl)
    inj = torch.from_numpy(lp.choose_regions(R, 0.2, 12)).cuda()
    h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=12)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    bad = sorted(set(range(R)) - set(inj.cpu().tolist()))[:2]      # two regions the validate found clean
    h.inject(wl, out, ck, stale, torch.tensor(bad, dtype=torch.int64, device="cuda"), mode="bitflip", seed=13)
    after = torch.zeros(1, dtype=torch.int64, device="cuda")
    h.recover_revalidate(wl, out, ck, failed, d_n, ws, after)
    torch.cuda.synchronize()
    assert int(after.item()) == 2


def test_list_path_counts_every_unrecovered_region():
    h, wl, out, ck, failed, d_n, ws, stale = _setup("stencil", "mod|xor|adler", 128, test_skip=True)
    R = h.num_regions(wl)
    inj = torch.from_numpy(lp.choose_regions(R, 0.3, 14)).cuda()
    h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=14)
    h.validate(wl, out, ck, failed, d_n, ws)
    after = torch.zeros(1, dtype=torch.int64, device="cuda")
    h.recover_revalidate(wl, out, ck, failed, d_n, ws, after)   # test hook: no re-execution
    torch.cuda.synchronize()
    assert int(after.item()) == inj.numel() > 0


@pytest.mark.parametrize("kind,reg", [("tmm_bf16", 32), ("tmm_f32", 128)])
def test_tile_rewriting_bodies_are_refused(kind, reg):
    """tcgen05 bodies whose recovery rewrites whole tiles (32x32 bf16 regions in 128x64 slices, 3xTF32 in 256x256
    tiles) would race a re-validation running beside the recovery: refused (use recover + validate)."""
    h, wl, out, ck, failed, d_n, ws, stale = _setup(kind, "mod|xor", reg)
    h.validate(wl, out, ck, failed, d_n, ws)
    after = torch.zeros(1, dtype=torch.int64, device="cuda")
    with pytest.raises(lp.LPError):
        h.recover_revalidate(wl, out, ck, failed, d_n, ws, after)


def test_hash_store_is_refused():
    h = lp.LP(128, 128, cksum="mod|xor", store="quad_cas")
    x = torch.zeros((256, 256), dtype=torch.float32, device="cuda")
    wl = lp.Workload.stencil(x)
    out, ck, failed, d_n, ws = h.alloc(wl)
    after = torch.zeros(1, dtype=torch.int64, device="cuda")
    with pytest.raises(lp.LPError):
        h.recover_revalidate(wl, out, ck, failed, d_n, ws, after)


def test_recover_revalidate_in_a_cuda_graph():
    """The side stream is forked from and joined into the caller's stream with events, so the call can be captured
    into a CUDA graph (bench.py replays its step segments as graphs): replay on a freshly crashed state."""
    h, wl, out, ck, failed, d_n, ws, stale = _setup("stencil", "mod|xor", 128)
    golden = dev_to_host(out)
    R = h.num_regions(wl)
    inj = torch.from_numpy(lp.choose_regions(R, 0.25, 15)).cuda()
    after = torch.full((1,), -1, dtype=torch.int64, device="cuda")
    h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=15)
    h.validate(wl, out, ck, failed, d_n, ws)
    h.recover_revalidate(wl, out, ck, failed, d_n, ws, after)        # eager warm-up (creates the side stream)
    torch.cuda.synchronize()
    assert int(after.item()) == 0
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s, capture_error_mode="thread_local"):
            h.validate(wl, out, ck, failed, d_n, ws)
            h.recover_revalidate(wl, out, ck, failed, d_n, ws, after)
    torch.cuda.synchronize()
    for _ in range(2):
        after.fill_(-1)
        h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=15)
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        assert int(d_n.item()) == inj.numel() and int(after.item()) == 0
        assert np.array_equal(dev_to_host(out).view(np.uint32), golden.view(np.uint32))
