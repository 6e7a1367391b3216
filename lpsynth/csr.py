"""Seeded synthetic sparse matrices (CSR) for the SpMV region body (NEXT row N4).

Like gen.py this holds NONE of the method's arithmetic: it only turns seeds and
counters into a matrix structure and values, identically on the host (numpy,
here) and on the device (``lpsynth/synth.cu`` ``synth_csr_cols``).  Recipe
(SpMV):

  row length   x_r = splitmix64(seed_len * GOLDEN + r)
               len = 8 + (x_r mod 17) + [((x_r >> 8) mod 16) == 0] * ((x_r >> 16) mod 256)
               -> 8..24 for 15/16 of the rows, a heavy tail up to 279 (mean ~24), like the
                  FEM-style matrices of Parboil's SpMV inputs (Table I)
  row_ptr      exclusive prefix sum of the lengths (int64, m + 1 entries)
  column k     banded: c = r - (len * S) / 2 + k * S + (splitmix64(seed_col * GOLDEN + row_ptr[r] + k) mod S),
               S = 8, taken mod ncols (non-negative) -> strictly increasing inside a row unless the
               band wraps the matrix edge; always distinct within a row when len * S <= ncols
  values       gen.values_f32(seed_val, 1, nnz) (counter = global nnz index), kinds uniform / int5
  x            gen.values_f32(seed_x, 1, ncols)
"""
from __future__ import annotations

import numpy as np

from .gen import GOLDEN, splitmix64

BAND_STRIDE = 8


def row_lengths(seed: int, rows: int, row0: int = 0) -> np.ndarray:
    r = np.arange(row0, row0 + rows, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = splitmix64(np.uint64(seed) * GOLDEN + r)
    tail = ((x >> np.uint64(8)) % np.uint64(16) == 0).astype(np.uint64) * ((x >> np.uint64(16)) % np.uint64(256))
    return (np.uint64(8) + x % np.uint64(17) + tail).astype(np.int64)


def row_ptr(seed: int, rows: int) -> np.ndarray:
    rp = np.zeros(rows + 1, dtype=np.int64)
    np.cumsum(row_lengths(seed, rows), out=rp[1:])
    return rp


def columns(seed: int, rp: np.ndarray, ncols: int, row0: int = 0) -> np.ndarray:
    """int32 column indices of rows [row0, row0 + len(rp) - 1) given their row_ptr slice rp."""
    rows = len(rp) - 1
    lens = np.diff(rp)
    nnz = int(rp[-1] - rp[0])
    r = np.repeat(np.arange(row0, row0 + rows, dtype=np.int64), lens)
    k = np.arange(nnz, dtype=np.int64) - np.repeat(rp[:-1] - rp[0], lens)
    gidx = (np.repeat(rp[:-1], lens) + k).astype(np.uint64)
    with np.errstate(over="ignore"):
        h = splitmix64(np.uint64(seed) * GOLDEN + gidx)
    jit = (h % np.uint64(BAND_STRIDE)).astype(np.int64)
    ln = np.repeat(lens, lens)
    c = r - (ln * BAND_STRIDE) // 2 + k * BAND_STRIDE + jit
    return np.mod(c, ncols).astype(np.int32)
