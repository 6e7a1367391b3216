"""GPU parity: LP-protected TMM through the C ABI vs the CPU oracle.

Config C1 (BASELINE.json configs[0]): 256x256x256 fp32, 32x32 regions, MOD, 5% of
regions corrupted then recovered -- plus random/odd shapes, every checksum type
and every injection mode.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
from paper_conf_iiswc_yudhakzs20_b200 import lp
from tests.gpu_util import check_store_table, dev_to_host, host_to_dev, make_inputs, oracle_validate, stale_image

pytestmark = pytest.mark.gpu


def run_cycle(M, N, K, RM, RN, in_dt, out_dt, kind, mask, body, mode="stale_words", frac=0.05, seed=1,
              store="array", check_values=True, recover_ws=True, tc_pair=True, shuffle=True, pairing=True,
              recover_slices=True, cuckoo_short_chains=False, recover_slices128=False):
    h = lp.LP(RM, RN, cksum=mask, store=store, body=body, tc_pair=tc_pair, shuffle=shuffle, pairing=pairing,
              recover_slices=recover_slices, cuckoo_short_chains=cuckoo_short_chains,
              recover_slices128=recover_slices128)
    A, B = make_inputs(seed, M, N, K, kind, in_dt)
    a, b = host_to_dev(A, in_dt), host_to_dev(B, in_dt)
    wl = lp.Workload.tmm(a, b, out_dtype=out_dt)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = host_to_dev(stale_image(seed, M, N, out_dt), out_dt)
    out.copy_(stale)                                   # the "persistent" array holds stale bits before the run
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    R = h.num_regions(wl)
    sel = oracle.selem(h.mask)
    golden = dev_to_host(out)
    ck_golden = dev_to_host(ck)

    # (4) clean-run check: records stored by the kernel == oracle records of the stored bits
    recs = oracle.records(golden, RM, RN, h.mask)
    if store == "array":
        assert np.array_equal(ck_golden[:R * sel].reshape(R, sel), recs)
    else:
        check_store_table(ck_golden, store, R, sel, recs)
    # (5) values vs fp64 oracle
    if check_values:
        to32 = (lambda x: x) if out_dt == "f32" else oracle.bf16_bits_to_f32
        Q = N // RN
        rids = range(R) if R <= 64 else np.random.default_rng(seed).choice(R, 16, replace=False)
        for rid in rids:
            p, q = divmod(int(rid), Q)
            ref = oracle.gemm_block_f64(A, B, p * RM, q * RN, RM, RN)
            got = golden[p * RM:(p + 1) * RM, q * RN:(q + 1) * RN]
            if out_dt == "i32":                         # the paper's int TMM (Listing 2): exact
                assert np.array_equal(got.view(np.int32), ref.astype(np.int64).astype(np.int32)), rid
            elif kind != "uniform":                     # integer-valued: bit-exact (Reading R18)
                exp = ref.astype(np.float32) if out_dt == "f32" else oracle.round_bf16(ref)
                assert np.array_equal(got, exp), rid
            else:
                tol = 1e-5 if (out_dt == "f32" and in_dt == "f32") else 2e-2
                if in_dt == "bf16" and out_dt == "f32":
                    tol = 1e-5
                assert oracle.rel_err(to32(got), ref) <= tol, rid
    # clean validate -> 0 failed
    if store.startswith("cuckoo"):
        d_stats = torch.zeros(2, dtype=torch.int64, device=out.device)
        h.stats(wl, ck, d_stats)
        assert d_stats[1].item() == 0 and ck_golden[6] == 0        # nothing lost, stash empty after the rehash
        run_cycle.last_rehashes = int(ck_golden[7])
    h.validate(wl, out, ck, failed, d_n, ws)
    assert int(d_n.item()) == 0

    # (6)(7) inject, validate == oracle on the corrupted state
    inj = torch.from_numpy(lp.choose_regions(R, frac, 1000 + seed)).cuda()
    h.inject(wl, out, ck, stale, inj, mode=mode, seed=1000 + seed)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    nf = int(d_n.item())
    got_failed = failed[:nf].cpu().numpy()
    bad_out, bad_ck = dev_to_host(out), dev_to_host(ck)
    exp_failed = oracle_validate(bad_out, bad_ck, store, RM, RN, h.mask)
    assert np.array_equal(got_failed, exp_failed)
    injected = set(inj.cpu().numpy().tolist())
    assert set(got_failed.tolist()) <= injected
    if mode in ("bitflip",):
        assert set(got_failed.tolist()) == injected          # a bit flip always changes MOD and XOR
    # (8) recover -> out == golden byte-for-byte, records == golden, re-validate == 0
    d_rec = torch.full((1,), -1, dtype=torch.int64, device=out.device)
    h.recover(wl, out, ck, failed, d_n, ws if recover_ws else None, d_n_recovered=d_rec)
    torch.cuda.synchronize()
    # regions rewritten (lp_recover_count): failed regions, or whole de-duplicated tiles / slices
    tc = body == "tcgen05" or (body == "auto" and in_dt != "i32")
    if not tc or (RM == 128 and in_dt == "bf16" and not (recover_slices128 and pairing and recover_ws)):
        exp_rec = nf
    else:
        EM = 128 if in_dt == "bf16" else 256
        EN = 64 if (in_dt == "bf16" and pairing and ((RM == 32 and recover_slices) or
                                                       (RM == 128 and recover_slices128))) else EM
        if not recover_ws:
            exp_rec = nf * (EM // RM) * (EM // RN)
        else:
            Q = N // RN
            tiles = {((r // Q) * RM // EM, c) for r in got_failed.tolist()
                     for c in range((r % Q) * RN // EN, ((r % Q) * RN + RN - 1) // EN + 1)}
            exp_rec = len(tiles) * EM * EN // (RM * RN)
    assert int(d_rec.item()) == exp_rec, (int(d_rec.item()), exp_rec, nf)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0
    assert np.array_equal(dev_to_host(out).view(np.uint8), golden.view(np.uint8))
    if store == "array":
        assert np.array_equal(dev_to_host(ck)[:R * sel], ck_golden[:R * sel])
    else:
        check_store_table(dev_to_host(ck), store, R, sel, recs)
    return h, nf


@pytest.mark.parametrize("kind", ["uniform", "int5"])
@pytest.mark.parametrize("mode", ["stale_words", "stale_region", "bitflip", "stale_record"])
def test_c1_simt_fp32_mod(kind, mode):
    """BASELINE configs[0]: 256^3 fp32, 32x32 regions, modular checksum, 5% corrupted then recovered."""
    _, nf = run_cycle(256, 256, 256, 32, 32, "f32", "f32", kind, "mod", "simt", mode=mode)
    assert nf >= 1


@pytest.mark.parametrize("mask", ["mod", "xor", "adler", "mod|xor", "mod|xor|adler", "xor|adler"])
def test_simt_checksum_types(mask):
    run_cycle(256, 192, 96, 32, 32, "f32", "f32", "uniform", mask, "simt", mode="stale_words", frac=0.1)


@pytest.mark.parametrize("in_dt,out_dt", [("bf16", "bf16"), ("bf16", "f32"), ("f32", "bf16")])
def test_simt_dtypes(in_dt, out_dt):
    run_cycle(128, 256, 64, 32, 32, in_dt, out_dt, "int5", "mod|xor|adler", "simt", frac=0.2)


@pytest.mark.parametrize("RM", [64, 128])
def test_simt_larger_regions(RM):
    run_cycle(256, 384, 160, RM, RM, "f32", "f32", "uniform", "mod|xor", "simt", frac=0.3)


@pytest.mark.parametrize("store", ["quad_cas", "quad_lock", "cuckoo", "cuckoo_lock"])
def test_simt_hash_stores(store):
    h, _ = run_cycle(256, 256, 64, 32, 32, "f32", "f32", "int5", "mod|xor", "simt", store=store, frac=0.1)


# ----------------------------------------------------------------------------- tcgen05 body (bf16 in)
@pytest.mark.parametrize("kind", ["int5", "uniform"])
@pytest.mark.parametrize("out_dt", ["bf16", "f32"])
@pytest.mark.parametrize("reg", [128, 32])
@pytest.mark.parametrize("tc_pair", [True, False])
def test_tc_cycle(kind, out_dt, reg, tc_pair):
    """M, N multiples of 256: the CTA-pair kernel (tc_pair) or the 1-SM kernel; recovery = 1-SM list mode."""
    run_cycle(256, 512, 256, reg, reg, "bf16", out_dt, kind, "mod|xor", "tcgen05", mode="stale_words", frac=0.2,
              tc_pair=tc_pair)


@pytest.mark.parametrize("recover_ws", [True, False])
def test_tc_r32_recovery_tile_dedup(recover_ws):
    """32x32 regions: many failed regions share a 128x128 tile; with the workspace each tile is recomputed once."""
    run_cycle(512, 768, 128, 32, 32, "bf16", "bf16", "uniform", "mod|xor", "tcgen05", mode="stale_region",
              frac=0.3, recover_ws=recover_ws)


@pytest.mark.parametrize("mask", ["mod", "xor", "adler", "mod|xor|adler"])
def test_tc_checksum_types(mask):
    run_cycle(384, 768, 192, 128, 128, "bf16", "bf16", "uniform", mask, "tcgen05", mode="bitflip", frac=0.3)


def test_tc_n_not_multiple_of_256():
    run_cycle(256, 384, 128, 128, 128, "bf16", "bf16", "int5", "mod|xor", "tcgen05", mode="stale_region", frac=0.5)


@pytest.mark.parametrize("tc_pair", [True, False])
def test_tc_many_tiles_persistent(tc_pair):
    # more tiles than SMs: persistent scheduling + TMEM double buffering across tiles
    run_cycle(2048, 2048, 512, 128, 128, "bf16", "bf16", "int5", "mod|xor", "tcgen05", mode="stale_words",
              frac=0.05, check_values=True, tc_pair=tc_pair)


@pytest.mark.parametrize("pairing", [True, False])
@pytest.mark.parametrize("reg,N,frac", [(128, 2176, 0.7), (32, 2048, 0.1)])
@pytest.mark.parametrize("out_dt", ["bf16", "f32"])
def test_tc_paired_recovery(pairing, reg, N, frac, out_dt):
    """More failed 128x128 tiles than SMs: failed tiles of one row band are re-executed in pairs on a 128x256
    tcgen05 tile with B gathered from two column panels (odd runs leave single tiles; N = 2176 has 17 tile
    columns).  Recovered bytes and records must equal the golden run either way."""
    _, nf = run_cycle(2048, N, 256, reg, reg, "bf16", out_dt, "uniform", "mod|xor", "tcgen05", mode="stale_words",
                      frac=frac, pairing=pairing)
    assert nf > 148


@pytest.mark.parametrize("slices", [True, False])
@pytest.mark.parametrize("N,frac", [(2048, 0.01), (2176, 0.1), (2048, 0.5), (1152, 1.0)])
@pytest.mark.parametrize("out_dt", ["bf16", "f32"])
def test_tc_slice_recovery(slices, N, frac, out_dt):
    """32x32 regions recovered as de-duplicated 128x64 slices (up to four slices of a row band per tcgen05
    task, N = 64 x slices, B gathered from up to four 64-column panels) vs the 128x128-tile path
    (LP_FLAG_RECOVER_TILE128).  frac 0.01: fewer slices than SMs (one slice per task, N = 64); N = 2176: 34
    slice columns per row band, runs of every length mod 4 (N = 64, 128, 192, 256 tasks); frac 1.0: every
    region.  Recovered bytes and records must equal the golden run."""
    _, nf = run_cycle(2048, N, 256, 32, 32, "bf16", out_dt, "uniform", "mod|xor", "tcgen05", mode="stale_words",
                      frac=frac, recover_slices=slices)
    assert nf > 0


@pytest.mark.parametrize("store", ["quad_cas", "cuckoo"])
def test_tc_paired_recovery_hash_store(store):
    run_cycle(2048, 2048, 128, 128, 128, "bf16", "bf16", "int5", "mod|xor", "tcgen05", store=store, frac=0.75)


@pytest.mark.parametrize("store", ["quad_cas", "quad_lock", "cuckoo", "cuckoo_lock"])
def test_tc_hash_stores(store):
    run_cycle(512, 512, 128, 128, 128, "bf16", "bf16", "int5", "mod|xor", "tcgen05", store=store, frac=0.1)


@pytest.mark.parametrize("store", ["quad_cas", "cuckoo"])
@pytest.mark.parametrize("mode", ["stale_record", "stale_region"])
def test_hash_store_recovery_modes(store, mode):
    """Recovery re-inserts records for keys that already exist (sentinel or intact records)."""
    run_cycle(512, 512, 128, 32, 32, "bf16", "bf16", "int5", "mod|xor", "tcgen05", store=store, mode=mode, frac=0.3)


def test_tc_unprotected_twin_same_bits():
    """cksum=0 builds the same body without the epilogue checksum: identical output bits."""
    import numpy as np
    from tests.gpu_util import make_inputs
    A, B = make_inputs(3, 512, 512, 256, "uniform", "bf16")
    a, b = host_to_dev(A, "bf16"), host_to_dev(B, "bf16")
    outs = []
    for mask in [0, 3]:
        h = lp.LP(128, 128, cksum=mask, body="tcgen05")
        wl = lp.Workload.tmm(a, b, out_dtype="bf16")
        out, ck, *_ = h.alloc(wl)
        if mask:
            h.cksum_init(wl, ck)
        h.run_protected(wl, out, ck if mask else None)
        torch.cuda.synchronize()
        outs.append(dev_to_host(out))
    assert np.array_equal(outs[0], outs[1])


def test_tc_matches_simt_integer_valued():
    """Both bodies are exact on integer-valued inputs: same bits (cross-check of two independent kernels)."""
    import numpy as np
    from tests.gpu_util import make_inputs
    A, B = make_inputs(4, 256, 256, 128, "int5", "bf16")
    a, b = host_to_dev(A, "bf16"), host_to_dev(B, "bf16")
    res = []
    for body in ["simt", "tcgen05"]:
        h = lp.LP(128, 128, cksum="mod|xor", body=body)
        wl = lp.Workload.tmm(a, b, out_dtype="bf16")
        out, ck, *_ = h.alloc(wl)
        h.cksum_init(wl, ck)
        h.run_protected(wl, out, ck)
        torch.cuda.synchronize()
        res.append((dev_to_host(out), dev_to_host(ck)))
    assert np.array_equal(res[0][0], res[1][0]) and np.array_equal(res[0][1], res[1][1])


# ----------------------------------------------------------------------------- fp32 via 3xTF32 (CTA pair)
@pytest.mark.parametrize("kind", ["int5", "uniform"])
@pytest.mark.parametrize("reg", [128, 32])
@pytest.mark.parametrize("recover_ws", [True, False])
def test_tf32x3_cycle(kind, reg, recover_ws):
    run_cycle(512, 768, 256, reg, reg, "f32", "f32", kind, "mod|xor", "tcgen05", mode="stale_words", frac=0.1,
              recover_ws=recover_ws)


def test_tf32x3_matches_simt_integer_valued():
    """3xTF32 tensor-core body and the SIMT FFMA body are both exact on integer-valued fp32 inputs: same bits."""
    import numpy as np
    from tests.gpu_util import make_inputs
    A, B = make_inputs(6, 512, 512, 512, "int5", "f32")
    a, b = host_to_dev(A, "f32"), host_to_dev(B, "f32")
    res = []
    for body in ["simt", "tcgen05"]:
        h = lp.LP(128, 128, cksum="mod|xor|adler", body=body)
        wl = lp.Workload.tmm(a, b, out_dtype="f32")
        out, ck, *_ = h.alloc(wl)
        h.cksum_init(wl, ck)
        h.run_protected(wl, out, ck)
        torch.cuda.synchronize()
        res.append((dev_to_host(out), dev_to_host(ck)))
    assert np.array_equal(res[0][0], res[1][0]) and np.array_equal(res[0][1], res[1][1])



# ----------------------------------------------------------------------------- int32 (the paper's TMM type)
@pytest.mark.parametrize("mask", ["mod|xor", "mod|xor|adler"])
@pytest.mark.parametrize("mode", ["stale_words", "bitflip"])
def test_int32_tmm_paper_shape(mask, mode):
    """Listing 2's int TMM with 32x32 thread-block regions (Table III: TMM = 32x32 blocks)."""
    run_cycle(256, 320, 192, 32, 32, "i32", "i32", "int17", mask, "simt", mode=mode, frac=0.1)


@pytest.mark.parametrize("in_dt,out_dt,kind", [("i32", "i32", "int17"), ("f32", "f32", "uniform"),
                                                ("bf16", "bf16", "uniform"), ("bf16", "f32", "int5")])
@pytest.mark.parametrize("mask", ["mod", "mod|xor", "xor|adler", "mod|xor|adler"])
def test_simt_multi_region_tile(in_dt, out_dt, kind, mask):
    """32x32 regions on the SIMT body with M, N % 128 == 0: 16 regions per 128x128 CTA tile (8x8 micro-tiles,
    segmented butterfly + two-warp combine, Reading c10); recovery re-executes single regions with the
    one-CTA-per-region kernel, which must reproduce the same bytes and records."""
    run_cycle(256, 384, 96, 32, 32, in_dt, out_dt, kind, mask, "simt", frac=0.15)


@pytest.mark.parametrize("store", ["quad_cas", "quad_lock", "cuckoo"])
def test_simt_multi_region_tile_hash_stores(store):
    run_cycle(384, 256, 64, 32, 32, "i32", "i32", "int17", "mod|xor", "simt", store=store, frac=0.1)


def test_int32_tmm_paper_4096_tile_forms_agree():
    """The paper's 4096^2 int TMM: the 128x128-tile body and the one-CTA-per-region body (LP_SIMT_MULTI=0 in a
    subprocess) store the same bytes and records."""
    import subprocess, sys, os
    code = (
        "import sys, hashlib; sys.path.insert(0, %r)\n"
        "import torch; from tests.gpu_util import *\n"
        "from paper_conf_iiswc_yudhakzs20_b200 import lp\n"
        "A, B = make_inputs(3, 4096, 4096, 4096, 'int17', 'i32')\n"
        "h = lp.LP(32, 32, cksum='mod|xor|adler', body='simt')\n"
        "wl = lp.Workload.tmm(host_to_dev(A, 'i32'), host_to_dev(B, 'i32'), out_dtype='i32')\n"
        "out, ck, *_ = h.alloc(wl); h.cksum_init(wl, ck); h.run_protected(wl, out, ck); torch.cuda.synchronize()\n"
        "print(hashlib.sha256(dev_to_host(out).tobytes() + dev_to_host(ck).tobytes()).hexdigest())\n"
    ) % os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    digests = []
    for multi in ("1", "0"):
        env = dict(os.environ, LP_SIMT_MULTI=multi)
        r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-2000:]
        digests.append(r.stdout.strip().splitlines()[-1])
    assert digests[0] == digests[1]


@pytest.mark.parametrize("store", ["quad_cas", "cuckoo", "cuckoo_lock"])
def test_tf32x3_hash_stores(store):
    run_cycle(512, 512, 128, 128, 128, "f32", "f32", "int5", "mod|xor", "tcgen05", store=store, frac=0.2)



@pytest.mark.parametrize("store", ["array", "quad_cas", "cuckoo"])
def test_simt_no_shuffle_ablation(store):
    """The paper's "without parallel reduction" variant (L343): same records, sequential fold."""
    run_cycle(256, 256, 128, 32, 32, "i32", "i32", "int17", "mod|xor", "simt", store=store, frac=0.1, shuffle=False)


# ----------------------------------------------------------------------------- cuckoo rehash (L270)
def test_cuckoo_rehash_after_short_chains():
    """L270 "When a cycle is detected, the cuckoo hash table performs hash tables rehashing": with the body's
    eviction bound cut to 16 (test hook), walks at 43% load end in the stash (~20 of 65536 inserts); the rehash
    kernel rebuilds T1/T2 under a new seed.  Afterwards every rid is found by the oracle's lookup (with the
    header's new seed) with its oracle record, the stash is empty and the error flag is 0 -- and recovery
    (which re-inserts) leaves the same state."""
    run_cycle.last_rehashes = 0
    run_cycle(8192, 8192, 64, 32, 32, "bf16", "bf16", "int5", "mod|xor", "tcgen05", store="cuckoo", frac=0.05,
              cuckoo_short_chains=True, check_values=False)
    assert run_cycle.last_rehashes >= 1


@pytest.mark.parametrize("store", ["cuckoo", "cuckoo_lock"])
def test_cuckoo_full_r262144(store):
    """at R = 262144 (16384^2 output, 32x32 regions) the 50%-load sizing lost records; with 1.15 R
    per table + rehash every rid must be found with its oracle record and lp_stats must report no error."""
    h = lp.LP(32, 32, cksum="mod|xor", store=store)
    A, B = make_inputs(41, 16384, 16384, 64, "int5", "bf16")
    a, b = host_to_dev(A, "bf16"), host_to_dev(B, "bf16")
    wl = lp.Workload.tmm(a, b, out_dtype="bf16")
    out, ck, failed, d_n, ws = h.alloc(wl)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    d_stats = torch.zeros(2, dtype=torch.int64, device=out.device)
    h.stats(wl, ck, d_stats)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert d_stats[1].item() == 0
    assert int(d_n.item()) == 0
    R = h.num_regions(wl)
    ck_h = dev_to_host(ck)
    assert ck_h[6] == 0
    check_store_table(ck_h, store, R, 2, oracle.records(dev_to_host(out), 32, 32, 3))


# ----------------------------------------------------------------------------- Listing 7 on the TMM (N2)
@pytest.mark.parametrize("reg,out_dt,store", [(128, "bf16", "array"), (32, "bf16", "array"), (128, "f32", "array"),
                                              (32, "f32", "quad_cas"), (128, "bf16", "cuckoo")])
@pytest.mark.parametrize("frac", [0.01, 0.10, 0.50])
@pytest.mark.parametrize("balanced", [False, True])
def test_tmm_same_grid_check_and_recover(reg, out_dt, store, frac, balanced):
    """Listing 7 (L565-578) on the tcgen05 CTA-pair TMM: one kernel validates every region of its tiles and
    recomputes in place only the tiles holding a failed region.  The count equals the oracle's failed set on
    the corrupted image, the recovered bytes equal the golden run, and a re-validate finds nothing."""
    M, N, K = 1024, 1536, 128          # 24 tiles of 256x256 over the CTA pairs; ragged per-pair counts
    h = lp.LP(reg, reg, cksum="mod|xor", store=store)
    A, B = make_inputs(13, M, N, K, "uniform", "bf16")
    a, b = host_to_dev(A, "bf16"), host_to_dev(B, "bf16")
    wl = lp.Workload.tmm(a, b, out_dtype=out_dt)
    out, ck, failed, d_n, ws = h.alloc(wl)
    stale = host_to_dev(stale_image(13, M, N, out_dt), out_dt)
    out.copy_(stale)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    torch.cuda.synchronize()
    golden = dev_to_host(out)
    R = h.num_regions(wl)
    # clean image: nothing fails, nothing is recomputed
    d_rec = torch.zeros(1, dtype=torch.int64, device="cuda")
    wsb = ws if balanced else None
    h.check_recover(wl, out, ck, d_rec, workspace=wsb)
    torch.cuda.synchronize()
    assert int(d_rec.item()) == 0
    inj = torch.from_numpy(lp.choose_regions(R, frac, 500 + reg)).cuda()
    h.inject(wl, out, ck, stale, inj, mode="stale_words", seed=501)
    torch.cuda.synchronize()
    exp = oracle_validate(dev_to_host(out), dev_to_host(ck), store, reg, reg, h.mask)
    assert len(exp) > 0
    h.check_recover(wl, out, ck, d_rec, workspace=wsb)
    torch.cuda.synchronize()
    assert int(d_rec.item()) == len(exp)
    assert np.array_equal(dev_to_host(out).view(np.uint8), golden.view(np.uint8))
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0


def test_tmm_check_and_recover_full_8192():
    """BASELINE configs[1] shape: 8192^3 bf16, 128x128 regions, 5% STALE_WORDS: check-and-recover restores the
    golden bytes; the count equals the oracle's failed set recomputed from the corrupted image."""
    from lpsynth import device_fill
    M = N = K = 8192
    a = torch.empty((M, K), dtype=torch.bfloat16, device="cuda")
    b = torch.empty((K, N), dtype=torch.bfloat16, device="cuda")
    device_fill(a, 1, "uniform", "bf16")
    device_fill(b, 2, "uniform", "bf16")
    h = lp.LP(128, 128, cksum="mod|xor")
    wl = lp.Workload.tmm(a, b, out_dtype="bf16")
    out, ck, failed, d_n, ws = h.alloc(wl)
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    golden = out.clone()
    stale = torch.zeros_like(out)
    R = h.num_regions(wl)
    inj = torch.from_numpy(lp.choose_regions(R, 0.05, 1001)).cuda()
    h.inject(wl, out, ck, stale, inj, mode="stale_words", seed=1001)
    torch.cuda.synchronize()
    exp = oracle_validate(dev_to_host(out), dev_to_host(ck), "array", 128, 128, h.mask)
    d_rec = torch.zeros(1, dtype=torch.int64, device="cuda")
    for wsb in (None, ws):                     # static, then balanced (re-corrupted in between)
        h.inject(wl, out, ck, stale, inj, mode="stale_words", seed=1001)
        h.check_recover(wl, out, ck, d_rec, workspace=wsb)
        torch.cuda.synchronize()
        assert int(d_rec.item()) == len(exp) > 0
        assert torch.equal(out.view(torch.int16), golden.view(torch.int16))


@pytest.mark.parametrize("frac", [0.02, 0.3, 1.0])
@pytest.mark.parametrize("out_dt", ["bf16", "f32"])
@pytest.mark.parametrize("store", ["array", "quad_cas"])
def test_tc_recovery_slices128(frac, out_dt, store):
    """LP_FLAG_RECOVER_SLICES128 (A/B switch): failed 128x128 regions re-executed as two 128x64 slices grouped
    1-4 per task in size-sorted snake order; each region's record is combined from its two slice partials,
    possibly computed by different CTAs.  Recovered bytes and records must equal the golden run."""
    _, nf = run_cycle(2048, 2560, 256, 128, 128, "bf16", out_dt, "uniform", "mod|xor|adler" if store == "array"
                      else "mod|xor", "tcgen05", mode="stale_words", frac=frac, store=store, recover_slices128=True)
    assert nf > 0


@pytest.mark.parametrize("reg", [128, 32])
@pytest.mark.parametrize("out_dt", ["bf16", "f32"])
@pytest.mark.parametrize("kind", ["int5", "uniform"])
def test_tc4_256row_pair_kernel(reg, out_dt, kind):
    """M % 512 == 0: the CTA-pair kernel with 256 rows per CTA (two M = 256 MMAs per k-step into the whole TMEM);
    values, records, validate and recovery against the oracle (N = 768: 3 column tiles, 2 x 3 pair tiles)."""
    run_cycle(1024, 768, 256, reg, reg, "bf16", out_dt, kind, "mod|xor|adler", "tcgen05", mode="stale_words",
              frac=0.2)


@pytest.mark.parametrize("store", ["quad_cas", "cuckoo"])
def test_tc4_hash_stores(store):
    run_cycle(1024, 1024, 128, 128, 128, "bf16", "bf16", "int5", "mod|xor", "tcgen05", store=store, frac=0.1)


def test_tc4_matches_tc2_bits():
    """The 256-row pair kernel (M = 1024) and the 128-row pair kernel (the same rows as M = 768 + M = 256
    problems, which it cannot take) produce identical bits: the same K order per output element."""
    from lpsynth import device_fill
    a = torch.empty((1024, 512), dtype=torch.bfloat16, device="cuda")
    b = torch.empty((512, 768), dtype=torch.bfloat16, device="cuda")
    device_fill(a, 1, "uniform", "bf16")
    device_fill(b, 2, "uniform", "bf16")
    outs = []
    for rows in ((0, 1024), (0, 768), (768, 1024)):
        h = lp.LP(128, 128, cksum="mod|xor")
        wl = lp.Workload.tmm(a[rows[0]:rows[1]], b, out_dtype="f32")
        out, ck, failed, d_n, ws = h.alloc(wl)
        h.cksum_init(wl, ck)
        h.run_protected(wl, out, ck)
        outs.append(out)
    torch.cuda.synchronize()
    assert torch.equal(outs[0].view(torch.int32), torch.cat([outs[1], outs[2]]).view(torch.int32))


@pytest.mark.parametrize("case", range(8))
def test_simt_fuzz_shapes(case):
    """Seeded random SIMT shapes with 32x32 regions: M, N multiples of 128 (16-region tiles) or of 32 only (one CTA
    per region), int32 / fp32 / bf16, checksum sets and stores, through body, validate and per-region recovery."""
    rng = np.random.default_rng(2000 + case)
    tile = bool(rng.integers(0, 2))
    M = int(rng.integers(1, 4)) * (128 if tile else 96)
    N = int(rng.integers(1, 4)) * (128 if tile else 160)
    K = 16 * int(rng.integers(1, 9))
    in_dt, out_dt, kind = [("i32", "i32", "int17"), ("f32", "f32", "uniform"), ("bf16", "f32", "int5")][case % 3]
    store = str(rng.choice(["array", "array", "quad_cas", "cuckoo"]))
    mask = str(rng.choice(["mod", "mod|xor", "xor|adler", "mod|xor|adler"])) if store == "array" else "mod|xor"
    run_cycle(M, N, K, 32, 32, in_dt, out_dt, kind, mask, "simt", store=store, frac=float(rng.choice([0.1, 0.5])),
              seed=5 + case)


@pytest.mark.parametrize("case", range(6))
def test_tf32x3_fuzz_shapes(case):
    """Seeded random 3xTF32 shapes (M, N multiples of 256, K multiples of 32 across the 512-K chunk boundaries):
    A's hi operand read raw from the TMA stage must stay within 1e-5 of the fp64 oracle (it would not if the tensor
    core rounded instead of truncating the low mantissa bits) and integer-valued inputs bit-exact."""
    rng = np.random.default_rng(3000 + case)
    M, N = 256 * int(rng.integers(1, 4)), 256 * int(rng.integers(1, 4))
    K = 32 * int(rng.integers(1, 40))
    kind = "uniform" if case % 2 == 0 else "int5"
    run_cycle(M, N, K, 128, 128, "f32", "f32", kind, "mod|xor", "tcgen05", frac=0.25, seed=7 + case)
