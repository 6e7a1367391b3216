"""GPU parity: LP-protected 5-point stencil (config C4 shape family) vs the CPU oracle."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
from lpsynth import gen
from paper_conf_iiswc_yudhakzs20_b200 import lp
from tests.gpu_util import check_store_table, dev_to_host, host_to_dev, oracle_validate

pytestmark = pytest.mark.gpu


def stencil_cycle(H, W, kind, mask, mode, frac, seed=2, store="array"):
    h = lp.LP(128, 128, cksum=mask, store=store)
    X = gen.generate(seed, H, W, kind, "f32")
    x = host_to_dev(X, "f32")
    wl = lp.Workload.stencil(x)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = host_to_dev(gen.generate(seed + 500, H, W, "bits", "f32"), "f32")
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    R = h.num_regions(wl)
    sel = oracle.selem(h.mask)
    golden = dev_to_host(out)
    ck_golden = dev_to_host(ck)
    # values: bit-exact against the exact-order fp32 oracle (Reading R19)
    assert np.array_equal(golden.view(np.uint32), oracle.stencil5(X).view(np.uint32))
    if store == "array":
        assert np.array_equal(ck_golden[:R * sel].reshape(R, sel), oracle.records(golden, 128, 128, h.mask))
    else:
        check_store_table(ck_golden, store, R, sel, oracle.records(golden, 128, 128, h.mask))
    h.validate(wl, out, ck, failed, d_n, ws)
    assert int(d_n.item()) == 0
    inj = torch.from_numpy(lp.choose_regions(R, frac, 1000 + seed)).cuda()
    h.inject(wl, out, ck, stale, inj, mode=mode, seed=1000 + seed)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    nf = int(d_n.item())
    got = failed[:nf].cpu().numpy()
    exp = oracle_validate(dev_to_host(out), dev_to_host(ck), store, 128, 128, h.mask)
    assert np.array_equal(got, exp)
    assert set(got.tolist()) <= set(inj.cpu().numpy().tolist())
    if mode == "stale_region":
        assert nf == inj.numel()
    h.recover(wl, out, ck, failed, d_n, ws)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0
    assert np.array_equal(dev_to_host(out).view(np.uint32), golden.view(np.uint32))
    return nf


@pytest.mark.parametrize("kind", ["uniform", "int17"])
@pytest.mark.parametrize("frac", [0.01, 0.10, 0.50])
def test_stencil_inject_recover(kind, frac):
    stencil_cycle(1024, 768, kind, "mod|xor", "stale_region", frac)


@pytest.mark.parametrize("mask", ["mod", "xor", "adler", "mod|xor|adler"])
@pytest.mark.parametrize("mode", ["stale_words", "bitflip", "stale_record"])
def test_stencil_checksums_and_modes(mask, mode):
    stencil_cycle(512, 640, "uniform", mask, mode, 0.2)


@pytest.mark.parametrize("store", ["quad_cas", "cuckoo", "cuckoo_lock"])
def test_stencil_hash_stores(store):
    stencil_cycle(512, 512, "uniform", "mod|xor", "stale_words", 0.25, store=store)



@pytest.mark.parametrize("frac", [0.01, 0.10, 0.50])
@pytest.mark.parametrize("store", ["array", "quad_cas", "cuckoo"])
def test_same_grid_check_and_recover(frac, store):
    """Listing 7 (N2): one kernel validates every region and re-executes the failed ones in place;
    the result equals the golden output and the count equals the oracle's failed set."""
    H, W = 1024, 768
    h = lp.LP(128, 128, cksum="mod|xor", store=store)
    X = gen.generate(3, H, W, "uniform", "f32")
    x = host_to_dev(X, "f32")
    wl = lp.Workload.stencil(x)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = host_to_dev(gen.generate(503, H, W, "bits", "f32"), "f32")
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    golden = dev_to_host(out)
    R = h.num_regions(wl)
    inj = torch.from_numpy(lp.choose_regions(R, frac, 1003)).cuda()
    h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=1003)
    torch.cuda.synchronize()
    exp = oracle_validate(dev_to_host(out), dev_to_host(ck), store, 128, 128, 3)
    d_rec = torch.zeros(1, dtype=torch.int64, device="cuda")
    h.check_recover(wl, out, ck, d_rec)
    torch.cuda.synchronize()
    assert int(d_rec.item()) == len(exp) == inj.numel()
    assert np.array_equal(dev_to_host(out).view(np.uint32), golden.view(np.uint32))
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0


@pytest.mark.parametrize("shard", [0, 1, 2, 3])
def test_stencil_row_shard(shard):
    """Row shard s of 4 (SURVEY §8e for the stencil): the shard's input view keeps the neighbouring rows
    readable as its halo; its output rows, records (GLOBAL rids) and the failed set after injection equal the
    oracle's on the full domain's rows [s*H/4, (s+1)*H/4); recovery restores the golden bytes."""
    H, W, G = 1024, 512, 4
    m = H // G
    r0 = shard * m
    X = gen.generate(9, H, W, "uniform", "f32")
    full_in = host_to_dev(X, "f32")
    x = full_in[r0:r0 + m]                                  # view into the full input: halo rows readable
    h = lp.LP(128, 128, cksum="mod|xor")
    wl = lp.Workload.stencil(x, row_offset=r0, global_m=H)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = host_to_dev(gen.generate(509, m, W, "bits", "f32"), "f32")
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    golden = dev_to_host(out)
    exp_out = oracle.stencil5_block(X, r0, 0, m, W)
    assert np.array_equal(golden.view(np.uint32), exp_out.view(np.uint32))
    R = h.num_regions(wl)
    assert np.array_equal(dev_to_host(ck)[:R * 2].reshape(R, 2), oracle.records(exp_out, 128, 128, 3))
    rid0 = (r0 // 128) * (W // 128)
    inj = torch.from_numpy(lp.choose_regions(R, 0.3, 77 + shard) + rid0).cuda()   # global rids
    h.inject(wl, out, ck, stale, inj, mode="stale_words", seed=77)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    nf = int(d_n.item())
    exp = oracle.validate_array(dev_to_host(out), dev_to_host(ck)[:R * 2], 128, 128, 3, rid_offset=rid0)
    assert nf > 0 and np.array_equal(failed[:nf].cpu().numpy(), exp)
    h.recover(wl, out, ck, failed, d_n, ws)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0
    assert np.array_equal(dev_to_host(out).view(np.uint32), golden.view(np.uint32))


@pytest.mark.parametrize("frac", [0.0, 1.0])
def test_stencil_recover_none_and_all(frac):
    """Degenerate crash sets for the TMA-fed list-mode recovery: no failed region (an empty list: every
    persistent CTA exits at once) and every region failed (the list is the whole table)."""
    nf = stencil_cycle(640, 512, "uniform", "mod|xor", "stale_region", frac)
    assert nf == round(frac * (640 // 128) * (512 // 128))


def test_stencil_tma_list_more_regions_than_ctas_per_sm_ring():
    """More failed regions than 3 ring stages x #SM, with a region count not a multiple of the grid: every CTA
    wraps its stage ring several times and the last CTAs take one region fewer."""
    nf = stencil_cycle(128 * 30, 128 * 23, "int17", "mod|xor|adler", "stale_region", 0.9)
    assert nf == round(0.9 * 30 * 23)


@pytest.mark.parametrize("case", range(12))
def test_stencil_fuzz_shapes(case):
    """Seeded random shapes (1..9 region rows, 1..7 region columns, incl. single-region domains), checksum sets,
    stores, crash modes and fractions through the full-run body and the TMA-fed list recovery."""
    rng = np.random.default_rng(1000 + case)
    H, W = 128 * int(rng.integers(1, 10)), 128 * int(rng.integers(1, 8))
    store = str(rng.choice(["array", "array", "quad_cas", "cuckoo"]))
    mask = str(rng.choice(["mod", "xor", "mod|xor", "adler", "mod|xor|adler"])) if store == "array" else "mod|xor"
    mode = str(rng.choice(["stale_words", "stale_region", "bitflip"]))
    frac = float(rng.choice([0.0, 0.3, 1.0]))
    kind = str(rng.choice(["uniform", "int17"]))
    stencil_cycle(H, W, kind, mask, mode, frac, seed=3 + case, store=store)
