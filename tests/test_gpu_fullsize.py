"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

Every stored record is checked bit-exactly against the oracle's recomputation
from the GPU's own output (all regions); region values are checked on sampled
regions against the fp64 / exact-order oracle; the failed set after injection is
checked bit-exactly against the oracle's validation of the corrupted state; the
recovered output must equal the golden output byte for byte.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import lpsynth
import oracle
from paper_conf_iiswc_yudhakzs20_b200 import lp, shard
from tests.gpu_util import check_store_table, dev_to_host, oracle_validate

pytestmark = pytest.mark.gpu


def _tmm_full(M, N, K, region, mask, store, kind, out_dt, nsample, row0=0, global_m=None, frac=0.05, seed=1,
              in_dt="bf16"):
    global_m = global_m or M
    tdt = torch.bfloat16 if in_dt == "bf16" else torch.float32
    a = torch.empty((M, K), dtype=tdt, device="cuda")
    b = torch.empty((K, N), dtype=tdt, device="cuda")
    lpsynth.device_fill(a, seed, kind, in_dt, row0=row0, ncols_global=K)
    lpsynth.device_fill(b, seed + 1, kind, in_dt)
    h = lp.LP(region, region, cksum=mask, store=store)                 # body AUTO = tcgen05, as in bench.py
    wl = lp.Workload.tmm(a, b, out_dtype=out_dt, row_offset=row0, global_m=global_m)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = torch.empty_like(out)
    if out.element_size() == 2:
        lpsynth.device_fill(stale, 3, "bits", "bf16", row0=row0, ncols_global=N)
    else:
        lpsynth.device_fill(stale.view(torch.int32), 3, "bits", "u32", row0=row0, ncols_global=N)
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    R = h.num_regions(wl)
    sel = oracle.selem(h.mask)
    rid0 = (row0 // region) * (N // region)
    golden_dev = out.clone()
    gold = dev_to_host(out)
    ckh = dev_to_host(ck)
    recs = oracle.records(gold, region, region, h.mask)
    if store == "array":
        assert np.array_equal(ckh[:R * sel].reshape(R, sel), recs)
    else:
        check_store_table(ckh, store, R, sel, recs, rid0)
    # sampled values vs the fp64 oracle (inputs regenerated on the host by the shared generator)
    from lpsynth import gen
    Q = N // region
    rng = np.random.default_rng(seed)
    for rid in rng.choice(R, nsample, replace=False):
        p, q = divmod(int(rid), Q)
        A_rows = gen.generate(seed, region, K, kind, in_dt, row0=row0 + p * region, ncols_global=K)
        B_cols = gen.generate(seed + 1, K, region, kind, in_dt, ncols_global=N, col0=q * region)
        ref = oracle.gemm_block_f64(A_rows, B_cols, 0, 0, region, region)
        got = gold[p * region:(p + 1) * region, q * region:(q + 1) * region]
        if kind != "uniform":
            exp = oracle.round_bf16(ref) if out_dt == "bf16" else ref.astype(np.float32)
            assert np.array_equal(got, exp), rid
        else:
            g32 = oracle.bf16_bits_to_f32(got) if out_dt == "bf16" else got
            assert oracle.rel_err(g32, ref) <= (2e-2 if out_dt == "bf16" else 1e-5), rid
    # crash -> validate (== oracle) -> recover (== golden) -> re-validate (0)
    inj = torch.from_numpy(lp.choose_regions(R, frac, 1000 + seed) + rid0).cuda()
    h.inject(wl, out, ck, stale, inj, mode="stale_words", seed=1000 + seed)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    nf = int(d_n.item())
    got_failed = failed[:nf].cpu().numpy()
    bad, badck = dev_to_host(out), dev_to_host(ck)
    exp_failed = oracle_validate(bad, badck, store, region, region, h.mask, rid_offset=rid0)
    assert np.array_equal(got_failed, exp_failed)
    assert set(got_failed.tolist()) <= set(inj.cpu().numpy().tolist()) and nf > 0
    h.recover(wl, out, ck, failed, d_n, ws)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0
    assert torch.equal(out.view(torch.int16) if out.element_size() == 2 else out.view(torch.int32),
                       golden_dev.view(torch.int16) if out.element_size() == 2 else golden_dev.view(torch.int32))


def test_c2_tmm8192_bf16_full():
    """configs[1]: 8192^3 bf16 -> bf16, 128x128 regions, MOD|XOR (the default bench workload)."""
    _tmm_full(8192, 8192, 8192, 128, "mod|xor", "array", "uniform", "bf16", nsample=6)


def test_c2_tmm8192_integer_valued_bit_exact():
    _tmm_full(8192, 8192, 8192, 128, "mod|xor|adler", "array", "int5", "bf16", nsample=6, seed=7)


def test_c2_tmm8192_f32_out():
    _tmm_full(8192, 8192, 8192, 128, "mod|xor", "array", "uniform", "f32", nsample=4, seed=11)


def test_c2_tmm8192_fp32_3xtf32_full():
    """configs[1] fp32 -> fp32 on the tensor cores (3xTF32): max rel. error <= 1e-5 on sampled regions."""
    _tmm_full(8192, 8192, 8192, 128, "mod|xor", "array", "uniform", "f32", nsample=4, seed=13, in_dt="f32")


def test_c2_tmm8192_fp32_integer_valued_bit_exact():
    _tmm_full(8192, 8192, 8192, 128, "mod|xor", "array", "int5", "f32", nsample=4, seed=17, in_dt="f32")


def test_c3_tmm16384_quad_cas_full():
    """configs[2]: 16384^3, lock-free quadratic-probing store; every rid looked up in the GPU's table."""
    _tmm_full(16384, 16384, 16384, 128, "mod|xor", "quad_cas", "int5", "bf16", nsample=2, seed=5)


def test_c3_tmm16384_cuckoo_full():
    """configs[2] ablation extended to the paper's cuckoo table (N1)."""
    _tmm_full(16384, 16384, 16384, 128, "mod|xor", "cuckoo", "int5", "bf16", nsample=2, seed=19)


def test_c3_tmm16384_r32_array_full():
    """configs[2] with 32x32 regions (R = 262144): records of every region, de-duplicated tile recovery."""
    _tmm_full(16384, 16384, 16384, 32, "mod|xor", "array", "int5", "bf16", nsample=4, seed=9)


def test_tmm8192_r32_half_failed_slice_grouping():
    """8192^2 with 32x32 regions and half of them failed: ~8000 failed 128x64 slices, so the grouping kernel
    takes several 4096-entry passes (run starts and task counts carried across passes)."""
    _tmm_full(8192, 8192, 128, 32, "mod|xor", "array", "int5", "bf16", nsample=2, frac=0.5, seed=21)


def test_c5_tmm65536_rank3_of_8_shard():
    """configs[4]: one rank's shard of the 65536^3 region-sharded TMM (rank 3 of 8), exactly as bench.py launches it."""
    s = shard.plan(65536, 65536, 128, 128, 8, 3)
    _tmm_full(s.rows, 65536, 65536, 128, "mod|xor", "array", "int5", "bf16", nsample=2, row0=s.row_offset,
              global_m=65536, seed=3)


def test_c4_stencil32768_full():
    """configs[3]: stencil 32768^2 fp32, 128x128 regions, 1% / 10% / 50% injection."""
    H = W = 32768
    x = torch.empty((H, W), dtype=torch.float32, device="cuda")
    lpsynth.device_fill(x, 1, "uniform", "f32")
    h = lp.LP(128, 128, cksum="mod|xor")
    wl = lp.Workload.stencil(x)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = torch.empty_like(out)
    lpsynth.device_fill(stale.view(torch.int32), 3, "bits", "u32")
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    R = h.num_regions(wl)
    gold_dev = out.clone()
    gold = dev_to_host(out)
    assert np.array_equal(dev_to_host(ck)[:R * 2].reshape(R, 2), oracle.records(gold, 128, 128, 3))
    X = dev_to_host(x)
    rng = np.random.default_rng(0)
    Q = W // 128
    for rid in list(rng.choice(R, 12, replace=False)) + [0, Q - 1, R - Q, R - 1]:   # incl. the 4 corners
        p, q = divmod(int(rid), Q)
        exp = oracle.stencil5_block(X, p * 128, q * 128, 128, 128)
        assert np.array_equal(gold[p * 128:(p + 1) * 128, q * 128:(q + 1) * 128].view(np.uint32), exp.view(np.uint32))
    del X
    for frac in (0.01, 0.10, 0.50):
        inj = torch.from_numpy(lp.choose_regions(R, frac, 77)).cuda()
        h.inject(wl, out, ck, stale, inj, mode="stale_region", seed=77)
        h.validate(wl, out, ck, failed, d_n, ws)
        torch.cuda.synchronize()
        nf = int(d_n.item())
        exp_failed = oracle.validate_array(dev_to_host(out), dev_to_host(ck)[:R * 2], 128, 128, 3)
        assert np.array_equal(failed[:nf].cpu().numpy(), exp_failed)
        assert nf == inj.numel()
        h.recover(wl, out, ck, failed, d_n, ws)
        h.validate(wl, out, ck, failed, d_n, ws)
        torch.cuda.synchronize()
        assert int(d_n.item()) == 0 and torch.equal(out, gold_dev)
