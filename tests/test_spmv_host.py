"""CPU pins of the SpMV oracle (oracle.spmv_rows, NEXT row N4) and of the synthetic CSR recipe
(lpsynth/csr.py).  The oracle is pinned to things other than itself: scipy.sparse's CSR product
(a library routine), the identity matrix, integer-valued inputs against an exact int64 dense
product, empty rows and row-slab consistency."""
from __future__ import annotations

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
from lpsynth import csr, gen


def _matrix(rows, ncols, kind="uniform", seed=5):
    rp = csr.row_ptr(seed, rows)
    cols = csr.columns(seed + 1, rp, ncols)
    vals = gen.values_f32(seed + 2, 1, int(rp[-1]), kind)[0]
    x = gen.values_f32(seed + 3, 1, ncols, kind)[0]
    return rp, cols, vals, x


def test_spmv_matches_scipy_csr():
    rp, cols, vals, x = _matrix(3000, 2500)
    A = sp.csr_matrix((vals.astype(np.float64), cols, rp), shape=(3000, 2500))
    ref = A @ x.astype(np.float64)
    y = oracle.spmv_rows(rp, cols, vals, x)
    assert np.allclose(y, ref, rtol=0, atol=1e-12)


def test_spmv_identity_and_empty_rows():
    n = 257
    rp = np.arange(n + 1, dtype=np.int64)
    rp[100:] -= 1                      # row 99 is empty
    cols = np.delete(np.arange(n, dtype=np.int32), 99)
    vals = np.ones(n - 1, dtype=np.float32)
    x = gen.values_f32(9, 1, n)[0]
    y = oracle.spmv_rows(rp, cols, vals, x)
    exp = x.astype(np.float64)
    exp[99] = 0.0
    assert np.array_equal(y, exp)


def test_spmv_integer_valued_exact():
    rp, cols, vals, x = _matrix(2000, 2000, kind="int5")
    dense = np.zeros((2000, 2000), dtype=np.int64)
    for i in range(2000):
        for k in range(rp[i], rp[i + 1]):
            dense[i, cols[k]] += int(vals[k])
    exp = dense @ x.astype(np.int64)
    assert np.array_equal(oracle.spmv_rows(rp, cols, vals, x), exp.astype(np.float64))


def test_spmv_row_slab():
    rp, cols, vals, x = _matrix(1000, 1000)
    full = oracle.spmv_rows(rp, cols, vals, x)
    assert np.array_equal(oracle.spmv_rows(rp, cols, vals, x, row0=300, rows=200), full[300:500])


def test_csr_recipe_shape():
    rows = 200000
    lens = csr.row_lengths(7, rows)
    assert lens.min() >= 8 and lens.max() <= 8 + 16 + 255
    assert 20.0 < lens.mean() < 28.0                      # mean 8 + 8 + 127.5/16 ~= 24
    assert (lens > 24).mean() > 0.03                      # the heavy tail exists
    rp = csr.row_ptr(7, rows)
    assert rp[0] == 0 and np.array_equal(np.diff(rp), lens)


def test_csr_columns_banded_distinct_and_shard_consistent():
    rows, ncols = 5000, 5000
    rp = csr.row_ptr(3, rows)
    cols = csr.columns(4, rp, ncols)
    assert cols.min() >= 0 and cols.max() < ncols
    for i in range(0, rows, 97):
        c = cols[rp[i]:rp[i + 1]]
        assert len(set(c.tolist())) == len(c)
        if 300 < i < rows - 300:                          # away from the wrap: strictly increasing, banded
            assert np.all(np.diff(c) > 0)
            assert np.abs(c.astype(np.int64) - i).max() <= (len(c) * csr.BAND_STRIDE) // 2 + csr.BAND_STRIDE
    a, b = 1234, 2345                                     # a row slab regenerates identically
    assert np.array_equal(csr.columns(4, rp[a:b + 1], ncols, row0=a), cols[rp[a]:rp[b]])


@pytest.mark.parametrize("seed", [1, 2])
def test_csr_deterministic(seed):
    rp1, c1, v1, x1 = _matrix(700, 900, seed=seed)
    rp2, c2, v2, x2 = _matrix(700, 900, seed=seed)
    assert np.array_equal(rp1, rp2) and np.array_equal(c1, c2) and np.array_equal(v1, v2) and np.array_equal(x1, x2)


def test_csr_band_alignment_and_rebase():
    """shard.csr_band: 4-aligned global start, rebased row_ptr with the same row lengths, pad < 4."""
    from paper_conf_iiswc_yudhakzs20_b200 import shard

    rp = csr.row_ptr(31, 5000)
    for row0, rows in [(0, 5000), (1024, 2048), (1, 7), (4999, 1)]:
        g0, local, nnz, pad = shard.csr_band(rp, row0, rows)
        assert g0 % 4 == 0 and 0 <= pad < 4 and g0 + pad == rp[row0]
        assert np.array_equal(np.diff(local), np.diff(rp[row0:row0 + rows + 1]))
        assert local[0] == pad and nnz == rp[row0 + rows] - g0
        # the chunk grid of every row's region start: (K0 & ~3) relative to the array is the same globally
        assert all(((int(rp[r]) & ~3) - g0) == (int(local[r - row0]) & ~3) for r in range(row0, row0 + rows))
