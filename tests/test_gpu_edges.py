"""GPU parity at the degenerate ends of the method: a single region (R = 1),
every region corrupted (k = R), the smallest K the tcgen05 bodies take (one 64-deep k-block), a clean
run followed by recovery of an empty failed list (a no-op), and a re-run of the protected kernel over
an already-recovered state (idempotence, L183: the TB is re-executable)."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
from paper_conf_iiswc_yudhakzs20_b200 import lp
from tests.gpu_util import dev_to_host, host_to_dev, make_inputs, stale_image
from tests.test_gpu_tmm import run_cycle

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("mode", ["stale_words", "stale_region", "bitflip", "stale_record"])
@pytest.mark.parametrize("body,in_dt,out_dt", [("tcgen05", "bf16", "bf16"), ("simt", "f32", "f32")])
def test_single_region(mode, body, in_dt, out_dt):
    """R = 1: one 128x128 region, corrupted (k = floor(1 * 1 + 0.5) = 1), validated, recovered."""
    _, nf = run_cycle(128, 128, 64, 128, 128, in_dt, out_dt, "int5", "mod|xor", body, mode=mode, frac=1.0)
    assert nf == 1


@pytest.mark.parametrize("reg,N", [(128, 512), (32, 256)])
@pytest.mark.parametrize("mode", ["stale_region", "bitflip"])
def test_every_region_corrupted(reg, N, mode):
    """k = R: the failed list is the whole table, recovery re-executes everything (tile de-dup / pairing
    over a full list)."""
    M = 512
    _, nf = run_cycle(M, N, 128, reg, reg, "bf16", "bf16", "int5", "mod|xor", "tcgen05", mode=mode, frac=1.0)
    assert nf == (M // reg) * (N // reg)


@pytest.mark.parametrize("tc_pair", [True, False])
def test_minimal_k(tc_pair):
    """K = 64: one k-block (one TMA stage) per tile."""
    run_cycle(256, 256, 64, 128, 128, "bf16", "f32", "uniform", "mod|xor|adler", "tcgen05", tc_pair=tc_pair)


def test_empty_recovery_and_reexecution_idempotent():
    """Recover with 0 failed regions leaves out and the table untouched; re-running the protected kernel
    over the recovered state rewrites the same bits (the region body is idempotent)."""
    M = N = 256
    K = 128
    A, B = make_inputs(3, M, N, K, "uniform", "bf16")
    a, b = host_to_dev(A, "bf16"), host_to_dev(B, "bf16")
    h = lp.LP(128, 128, cksum="mod|xor")
    wl = lp.Workload.tmm(a, b, out_dtype="bf16")
    out, ck, failed, d_n, ws = h.alloc(wl)
    out.copy_(host_to_dev(stale_image(3, M, N, "bf16"), "bf16"))
    h.cksum_init(wl, ck)
    h.run_protected(wl, out, ck)
    h.validate(wl, out, ck, failed, d_n, ws)
    torch.cuda.synchronize()
    assert int(d_n.item()) == 0
    gold, ckg = dev_to_host(out).copy(), dev_to_host(ck).copy()
    h.recover(wl, out, ck, failed, d_n, ws)           # empty list: nothing to do
    torch.cuda.synchronize()
    assert np.array_equal(dev_to_host(out), gold) and np.array_equal(dev_to_host(ck), ckg)
    h.run_protected(wl, out, ck)                       # re-execute every region over the golden state
    torch.cuda.synchronize()
    assert np.array_equal(dev_to_host(out), gold) and np.array_equal(dev_to_host(ck), ckg)
    R = h.num_regions(wl)
    assert np.array_equal(ckg[:R * 2].reshape(R, 2), oracle.records(gold, 128, 128, h.mask))
