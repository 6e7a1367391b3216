"""Seeded, counter-based synthetic inputs shared by the oracle and the CUDA path.

This module holds NONE of the method's arithmetic (no checksum, no GEMM, no
stencil). It only turns (seed, global element index) into input values, so that
the oracle side (numpy, here) and the device side (``lpsynth/synth.cu``) can
produce the same inputs independently. The recipe is DESIGN.md "Input recipe"
(SURVEY.md §8d "Synthetic inputs").

    x   = splitmix64(seed * GOLDEN + global_index)
    uniform : v = (x >> 40) * 2^-23 - 1        in [-1, 1), exact in fp32
    int5    : v = (x mod 5) - 2                 TMM integer-valued inputs
    int17   : v = (x mod 17) - 8                stencil integer-valued inputs
    bits    : u32 = low 32 bits of x            "stale" pre-image of the output
    int32 ("i32") inputs take the integer-valued kinds as int32 (the paper's TMM, Listing 2)

global_index = row * ncols_global + col over the *global* matrix, so a row shard
sees the same values it would see inside the unsharded matrix.
bf16 values are the round-to-nearest-even of the fp32 value.
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

KINDS = {"uniform": 0, "int5": 1, "int17": 2, "bits": 3}
DTYPES = {"f32": 0, "bf16": 1, "u32": 2, "i32": 3}


def splitmix64(z: np.ndarray) -> np.ndarray:
    """Vigna's splitmix64 output function applied to state z + GOLDEN (uint64, wrapping)."""
    with np.errstate(over="ignore"):
        z = z.astype(np.uint64) + GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def raw(seed: int, rows: int, cols: int, row0: int = 0, ncols_global: int | None = None,
        col0: int = 0) -> np.ndarray:
    """uint64 x for rows [row0, row0+rows) x cols [col0, col0+cols) of a matrix with ncols_global columns."""
    ncg = cols if ncols_global is None else ncols_global
    r = np.arange(row0, row0 + rows, dtype=np.uint64)[:, None]
    c = np.arange(col0, col0 + cols, dtype=np.uint64)[None, :]
    with np.errstate(over="ignore"):
        state = np.uint64(seed) * GOLDEN + r * np.uint64(ncg) + c
    return splitmix64(state)


def values_f32(seed: int, rows: int, cols: int, kind: str = "uniform", row0: int = 0,
               ncols_global: int | None = None, col0: int = 0) -> np.ndarray:
    x = raw(seed, rows, cols, row0, ncols_global, col0)
    if kind == "uniform":
        return ((x >> np.uint64(40)).astype(np.float64) * 2.0 ** -23 - 1.0).astype(np.float32)
    if kind == "int5":
        return ((x % np.uint64(5)).astype(np.int64) - 2).astype(np.float32)
    if kind == "int17":
        return ((x % np.uint64(17)).astype(np.int64) - 8).astype(np.float32)
    raise ValueError(kind)


def f32_to_bf16_bits(v: np.ndarray) -> np.ndarray:
    """Round-to-nearest-even fp32 -> bf16 bit patterns (uint16). Inputs here are finite."""
    b = np.ascontiguousarray(v, dtype=np.float32).view(np.uint32).astype(np.uint64)
    b = b + np.uint64(0x7FFF) + ((b >> np.uint64(16)) & np.uint64(1))
    return (b >> np.uint64(16)).astype(np.uint16)


def generate(seed: int, rows: int, cols: int, kind: str, dtype: str, row0: int = 0,
             ncols_global: int | None = None, col0: int = 0) -> np.ndarray:
    """Host copy of the synthetic matrix (block at row0/col0 of a matrix with ncols_global columns).
    f32 -> float32, bf16 -> uint16 bits, u32 -> uint32."""
    if kind == "bits":
        x = raw(seed, rows, cols, row0, ncols_global, col0)
        bits = (x & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        if dtype in ("u32", "f32", "i32"):
            return {"u32": bits, "f32": bits.view(np.float32), "i32": bits.view(np.int32)}[dtype]
        if dtype == "bf16":
            return (bits & np.uint32(0xFFFF)).astype(np.uint16)
        raise ValueError(dtype)
    v = values_f32(seed, rows, cols, kind, row0, ncols_global, col0)
    if dtype == "f32":
        return v
    if dtype == "i32":
        if kind == "uniform":
            raise ValueError("int32 inputs are integer-valued kinds (int5, int17)")
        return v.astype(np.int32)
    if dtype == "bf16":
        return f32_to_bf16_bits(v)
    raise ValueError(dtype)
