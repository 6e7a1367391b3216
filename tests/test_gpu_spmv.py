"""GPU parity: LP-protected SpMV region body (CSR, NEXT row N4) through the C ABI vs the CPU oracle.

Same bar as the TMM / stencil bodies: records of the stored y words ==
oracle records (bit-exact), y values == fp64 oracle (integer-valued inputs bit-exact, uniform
inputs within 1e-5 normwise), validate after injection == oracle failed set, recovery restores
the golden bytes and records, re-validation finds nothing.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import lpsynth
import oracle
from lpsynth import csr, gen
from paper_conf_iiswc_yudhakzs20_b200 import lp
from tests.gpu_util import check_store_table, dev_to_host, oracle_validate

pytestmark = pytest.mark.gpu


def synth(rows, ncols, kind="uniform", seed=11):
    rp = csr.row_ptr(seed, rows)
    cols = csr.columns(seed + 1, rp, ncols)
    vals = gen.values_f32(seed + 2, 1, int(rp[-1]), kind)[0]
    x = gen.values_f32(seed + 3, 1, ncols, kind)[0]
    return rp, cols, vals, x


def run_spmv_cycle(mat, RN, kind, mask="mod|xor", store="array", mode="stale_words", frac=0.1, seed=1,
                   shuffle=True, row0=0, rows=None):
    rp, cols, vals, x = mat
    m_all = len(rp) - 1
    rows = m_all - row0 if rows is None else rows
    rp_d = torch.from_numpy(np.ascontiguousarray(rp[row0:row0 + rows + 1])).cuda()
    cols_d = torch.from_numpy(cols).cuda()
    vals_d = torch.from_numpy(vals).cuda()
    x_d = torch.from_numpy(x).cuda()
    h = lp.LP(1, RN, cksum=mask, store=store, shuffle=shuffle)
    wl = lp.Workload.spmv(vals_d, x_d, rp_d, cols_d, row_offset=row0, global_m=m_all)
    out, ck, failed, d_n, ws = h.alloc(wl)
    R = h.num_regions(wl)
    assert R == rows // RN and tuple(out.shape) == (R, RN)
    stale = torch.from_numpy(gen.generate(seed + 500, R, RN, "bits", "f32")).cuda()
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    sel = oracle.selem(h.mask)
    golden = dev_to_host(out)
    ck_golden = dev_to_host(ck)
    recs = oracle.records(golden, 1, RN, h.mask)
    if store == "array":
        assert np.array_equal(ck_golden[:R * sel].reshape(R, sel), recs)
    else:
        check_store_table(ck_golden, store, R, sel, recs, rid0=row0 // RN)
    y_ref = oracle.spmv_rows(rp, cols, vals, x, row0=row0, rows=rows)
    if kind == "int5":
        assert np.array_equal(golden.reshape(-1), y_ref.astype(np.float32))
    else:
        assert oracle.rel_err(golden.reshape(-1), y_ref) <= 1e-5
    h.validate(wl, out, ck, failed, d_n, ws)
    assert int(d_n.item()) == 0
    inj = torch.from_numpy(lp.choose_regions(R, frac, 1000 + seed) + row0 // RN).cuda()
    h.inject(wl, out, ck, stale, inj, mode=mode, seed=1000 + seed)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    nf = int(d_n.item())
    got = failed[:nf].cpu().numpy()
    exp = oracle_validate(dev_to_host(out), dev_to_host(ck), store, 1, RN, h.mask, rid_offset=row0 // RN)
    assert np.array_equal(got, exp)
    assert set(got.tolist()) <= set(inj.cpu().numpy().tolist())
    h.recover(wl, out, ck, failed, d_n, ws)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0
    assert np.array_equal(dev_to_host(out).view(np.uint32), golden.view(np.uint32))
    if store == "array":
        assert np.array_equal(dev_to_host(ck)[:R * sel], ck_golden[:R * sel])
    return nf


@pytest.mark.parametrize("kind", ["uniform", "int5"])
@pytest.mark.parametrize("mode", ["stale_words", "stale_region", "bitflip", "stale_record"])
def test_spmv_cycle(kind, mode):
    nf = run_spmv_cycle(synth(65536, 65536, kind), 1024, kind, mode=mode, frac=0.1)
    assert nf >= 1


@pytest.mark.parametrize("mask", ["mod", "xor", "adler", "mod|xor|adler"])
def test_spmv_checksum_types(mask):
    run_spmv_cycle(synth(16384, 20000), 512, "uniform", mask=mask, mode="stale_words", frac=0.2)


@pytest.mark.parametrize("RN", [4, 64, 256, 4096])
def test_spmv_region_sizes(RN):
    """4 rows per region: one row per warp and 4 idle warps; 64: 8 rows per warp (warp-uniform trip counts)."""
    run_spmv_cycle(synth(max(RN * 24, 4 * 4096), 30000, "int5"), RN, "int5", frac=0.25)


@pytest.mark.parametrize("length", [2, 40, 1500])
def test_spmv_row_length_mixes(length):
    """Short rows with empty ones (a 2048-element chunk spans > 256 rows), long rows, and rows longer than a
    chunk (each row is still summed in CSR order across chunk boundaries)."""
    rows = 8192 if length < 1000 else 1024
    lens = (np.arange(rows) * 7919) % (2 * length + 1)
    rp = np.zeros(rows + 1, dtype=np.int64)
    np.cumsum(lens, out=rp[1:])
    ncols = max(9000, 2 * length * csr.BAND_STRIDE)
    cols = csr.columns(2, rp, ncols)
    vals = gen.values_f32(3, 1, int(rp[-1]), "int5")[0]
    x = gen.values_f32(4, 1, ncols, "int5")[0]
    run_spmv_cycle((rp, cols, vals, x), 512 if length < 1000 else 64, "int5", mode="stale_region", frac=0.3)


def test_spmv_nnz_not_multiple_of_4_and_unaligned_regions():
    """Region nnz ranges start at arbitrary offsets and the array ends in a partial 16-byte vector."""
    rows = 4096
    lens = 1 + (np.arange(rows) * 31) % 7
    rp = np.zeros(rows + 1, dtype=np.int64)
    np.cumsum(lens, out=rp[1:])
    if rp[-1] % 4 == 0:
        rp[-1] += 1
    cols = csr.columns(5, rp, 5000)
    vals = gen.values_f32(6, 1, int(rp[-1]), "uniform")[0]
    x = gen.values_f32(7, 1, 5000, "uniform")[0]
    run_spmv_cycle((rp, cols, vals, x), 256, "uniform", frac=0.3)


@pytest.mark.parametrize("store", ["quad_cas", "quad_lock", "cuckoo"])
def test_spmv_hash_stores(store):
    run_spmv_cycle(synth(32768, 32768), 256, "uniform", store=store, frac=0.1)


def test_spmv_no_shuffle_ablation_same_records():
    """The paper's no-shuffle reduction (L343) stores the same records as the shuffle reduction."""
    run_spmv_cycle(synth(32768, 32768, "int5"), 1024, "int5", shuffle=False, frac=0.1)


def test_spmv_row_shard():
    """Rows [4096, 4096 + 16384) of a 32768-row matrix: global rids, absolute row_ptr offsets."""
    run_spmv_cycle(synth(32768, 32768), 1024, "uniform", row0=4096, rows=16384, frac=0.2)


def test_spmv_device_twin_matches_host_recipe():
    rows, ncols = 100000, 120000
    rp_d, cols_d, vals_d = lpsynth.device_csr(21, 22, 23, rows, ncols, "uniform")
    rp = csr.row_ptr(21, rows)
    assert np.array_equal(rp_d.cpu().numpy(), rp)
    assert np.array_equal(cols_d.cpu().numpy(), csr.columns(22, rp, ncols))
    assert np.array_equal(vals_d.cpu().numpy(), gen.values_f32(23, 1, int(rp[-1]), "uniform")[0])


@pytest.mark.parametrize("RM,RN", [(2, 64), (1, 96), (1, 2)])
def test_spmv_invalid_region_shape(RM, RN):
    x = torch.zeros(64, device="cuda")
    h = lp.LP(RM, RN)
    wl = lp.Workload.spmv(None, x, None, None, m=RN * 8)
    with pytest.raises(lp.LPError):
        h.num_regions(wl)


@pytest.mark.parametrize("row0_regions", [1, 3])
def test_spmv_row_band_shard_bit_identical(row0_regions):
    """SpMV row-band shard (bench --gpus N): the rank's value / column arrays start at the 4-aligned global nnz
    index below its first row (shard.csr_band), so the shard's y words and records are bit-identical to the
    same rows of the unsharded run (the 2048-nnz chunk grid and 16-B vectors sit where they sit globally)."""
    from paper_conf_iiswc_yudhakzs20_b200 import shard

    RN, rows_all = 256, 256 * 6
    rp, cols, vals, x = synth(rows_all, rows_all)
    h = lp.LP(1, RN, cksum="mod|xor|adler")
    # full matrix
    wl = lp.Workload.spmv(torch.from_numpy(vals).cuda(), torch.from_numpy(x).cuda(), torch.from_numpy(rp).cuda(),
                          torch.from_numpy(cols).cuda())
    y_full, ck_full, *_ = h.alloc(wl)
    h.cksum_init(wl, ck_full)
    h.run_protected(wl, y_full, ck_full)
    # the band of rows [row0, row0 + 2 regions) with rebased, 4-aligned arrays
    row0, rows = RN * row0_regions, 2 * RN
    g0, rp_l, nnz_l, pad = shard.csr_band(rp, row0, rows)
    assert g0 % 4 == 0 and 0 <= pad < 4 and rp_l[0] == pad
    wls = lp.Workload.spmv(torch.from_numpy(vals[g0:g0 + nnz_l].copy()).cuda(), torch.from_numpy(x).cuda(),
                           torch.from_numpy(rp_l).cuda(), torch.from_numpy(cols[g0:g0 + nnz_l].copy()).cuda(),
                           row_offset=row0, global_m=rows_all)
    y_s, ck_s, *_ = h.alloc(wls)
    h.cksum_init(wls, ck_s)
    h.run_protected(wls, y_s, ck_s)
    torch.cuda.synchronize()
    yf = dev_to_host(y_full).reshape(-1).view(np.uint32)
    ys = dev_to_host(y_s).reshape(-1).view(np.uint32)
    assert np.array_equal(ys, yf[row0:row0 + rows])
    sel = oracle.selem(h.mask)
    cf = dev_to_host(ck_full)[:(rows_all // RN) * sel].reshape(-1, sel)
    cs = dev_to_host(ck_s)[:(rows // RN) * sel].reshape(-1, sel)
    assert np.array_equal(cs, cf[row0 // RN:(row0 + rows) // RN])
