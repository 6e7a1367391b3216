"""CPU oracle for the Lazy Persistency hot path (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package. It shares no code with the
CUDA path (``paper_conf_iiswc_yudhakzs20_b200``) and never imports it.

Thin ctypes wrapper over ``oracle/lp_oracle.c`` (plain single-threaded C); each
wrapped function cites the PAPER.md passage it follows in the C source. Arrays
are numpy: fp32 outputs as float32, bf16 outputs as uint16 bit patterns.

Parity status: every function here is pinned by tests/test_oracle_pins.py
(paper worked example, zlib, brute force, closed forms); none is "parity
unpinned" except the hash-collision *counts*, which the oracle does not model
(DESIGN.md "Unpinned").
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

MOD, XOR, ADLER = 1, 2, 4
EMPTY_KEY = 0xFFFFFFFF
SENTINEL = 0xFFFFFFFF

_p = ctypes.c_void_p
_i64 = ctypes.c_int64
_u32 = ctypes.c_uint32
_i = ctypes.c_int


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C, no contraction)."""
    import subprocess

    so = os.path.join(_HERE, "liboracle.so")
    src = os.path.join(_HERE, "lp_oracle.c")
    if force or not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-shared", "-fPIC",
                               "-o", so, src])
    return so


def lib():
    global _LIB
    if _LIB is None:
        L = ctypes.CDLL(build())
        L.lpo_float_word.restype = _u32
        L.lpo_float_word.argtypes = [ctypes.c_float]
        L.lpo_adler32.restype = _u32
        L.lpo_adler32.argtypes = [_p, _i64]
        L.lpo_selem.restype = _i
        L.lpo_selem.argtypes = [_u32]
        L.lpo_region_record.restype = None
        L.lpo_region_record.argtypes = [_p, _i64, _i, _i64, _i64, _i, _i, _u32, _p]
        L.lpo_records.restype = None
        L.lpo_records.argtypes = [_p, _i64, _i64, _i64, _i, _i, _i, _u32, _p]
        L.lpo_validate_array.restype = _i64
        L.lpo_validate_array.argtypes = [_p, _p, _i64, _i64, _i64, _i, _i, _i, _u32, _i64, _p]
        L.lpo_quad_hash.restype = _u32
        L.lpo_quad_hash.argtypes = [_u32, _u32, _u32]
        L.lpo_quad_probe.restype = _u32
        L.lpo_quad_probe.argtypes = [_u32, _u32, _u32, _u32]
        L.lpo_quad_lookup.restype = _i
        L.lpo_quad_lookup.argtypes = [_p, _u32, _i, _u32, _u32, _p]
        L.lpo_quad_insert.restype = _u32
        L.lpo_quad_insert.argtypes = [_p, _u32, _i, _u32, _u32, _p]
        L.lpo_validate_quad.restype = _i64
        L.lpo_validate_quad.argtypes = [_p, _p, _u32, _u32, _i64, _i64, _i64, _i, _i, _i, _u32, _i64, _p]
        L.lpo_cuckoo_hash.restype = _u32
        L.lpo_cuckoo_hash.argtypes = [_i, _u32, _u32, _u32]
        L.lpo_cuckoo_lookup.restype = _i
        L.lpo_cuckoo_lookup.argtypes = [_p, _u32, _i, _u32, _u32, _p]
        L.lpo_cuckoo_insert.restype = _u32
        L.lpo_cuckoo_insert.argtypes = [_p, _u32, _i, _u32, _u32, _p, _i]
        L.lpo_validate_cuckoo.restype = _i64
        L.lpo_validate_cuckoo.argtypes = [_p, _p, _u32, _u32, _i64, _i64, _i64, _i, _i, _i, _u32, _i64, _p]
        L.lpo_gemm_block_f64.restype = None
        L.lpo_gemm_block_f64.argtypes = [_p, _i64, _p, _i64, _i, _i64, _i64, _i64, _i64, _i64, _p]
        L.lpo_round_bf16.restype = None
        L.lpo_round_bf16.argtypes = [_p, _i64, _p]
        L.lpo_stencil5_block.restype = None
        L.lpo_stencil5_block.argtypes = [_p, _i64, _i64, _i64, _i64, _i64, _i64, _i64, _p]
        L.lpo_spmv_rows.restype = None
        L.lpo_spmv_rows.argtypes = [_p, _p, _p, _p, _i64, _i64, _p]
        _LIB = L
    return _LIB


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _es(out: np.ndarray) -> int:
    if out.dtype == np.float32 or out.dtype == np.uint32 or out.dtype == np.int32:
        return 4
    if out.dtype == np.uint16:
        return 2
    raise TypeError(f"output dtype {out.dtype}: expected float32 (fp32) or uint16 (bf16 bits)")


def selem(mask: int) -> int:
    return bin(mask & 7).count("1")


def float_word(v: float) -> int:
    """Fig. 2 (L260-261) float -> 'ordered integer'."""
    return int(lib().lpo_float_word(ctypes.c_float(v)))


def adler32(data: bytes) -> int:
    buf = np.frombuffer(data, dtype=np.uint8)
    return int(lib().lpo_adler32(_ptr(np.ascontiguousarray(buf)), len(buf)))


def region_record(out: np.ndarray, p: int, q: int, RM: int, RN: int, mask: int) -> np.ndarray:
    out = np.ascontiguousarray(out)
    rec = np.zeros(selem(mask), dtype=np.uint32)
    lib().lpo_region_record(_ptr(out), out.shape[1], _es(out), p, q, RM, RN, mask, _ptr(rec))
    return rec


def records(out: np.ndarray, RM: int, RN: int, mask: int) -> np.ndarray:
    """[R, selem] uint32 records of every region, rid = p*(N/RN)+q."""
    out = np.ascontiguousarray(out)
    M, N = out.shape
    assert M % RM == 0 and N % RN == 0
    recs = np.zeros(((M // RM) * (N // RN), selem(mask)), dtype=np.uint32)
    lib().lpo_records(_ptr(out), M, N, N, _es(out), RM, RN, mask, _ptr(recs))
    return recs


def validate_array(out: np.ndarray, table: np.ndarray, RM: int, RN: int, mask: int, rid_offset: int = 0) -> np.ndarray:
    """Ascending failed global rids for a hash-table-less record array."""
    out = np.ascontiguousarray(out)
    table = np.ascontiguousarray(table, dtype=np.uint32).reshape(-1)
    M, N = out.shape
    R = (M // RM) * (N // RN)
    assert table.size >= R * selem(mask)
    failed = np.zeros(R, dtype=np.int64)
    nf = lib().lpo_validate_array(_ptr(out), _ptr(table), M, N, N, _es(out), RM, RN, mask, rid_offset, _ptr(failed))
    return failed[:nf].copy()


def quad_hash(key: int, seed: int, cap: int) -> int:
    return int(lib().lpo_quad_hash(key, seed, cap))


def quad_probe(key: int, seed: int, cap: int, i: int) -> int:
    return int(lib().lpo_quad_probe(key, seed, cap, i))


def quad_lookup(table: np.ndarray, cap: int, sel: int, key: int, seed: int):
    table = np.ascontiguousarray(table, dtype=np.uint32).reshape(-1)
    rec = np.zeros(max(sel, 1), dtype=np.uint32)
    ok = lib().lpo_quad_lookup(_ptr(table), cap, sel, key, seed, _ptr(rec))
    return (rec[:sel].copy() if ok else None)


def quad_insert(table: np.ndarray, cap: int, sel: int, key: int, seed: int, rec) -> int:
    assert table.flags.c_contiguous and table.dtype == np.uint32
    r = np.ascontiguousarray(np.asarray(rec, dtype=np.uint32).reshape(-1))
    if r.size == 0:
        r = np.zeros(1, dtype=np.uint32)
    return int(lib().lpo_quad_insert(_ptr(table), cap, sel, key, seed, _ptr(r)))


def validate_quad(out: np.ndarray, table: np.ndarray, cap: int, seed: int, RM: int, RN: int, mask: int,
                  rid_offset: int = 0) -> np.ndarray:
    out = np.ascontiguousarray(out)
    table = np.ascontiguousarray(table, dtype=np.uint32).reshape(-1)
    M, N = out.shape
    R = (M // RM) * (N // RN)
    failed = np.zeros(R, dtype=np.int64)
    nf = lib().lpo_validate_quad(_ptr(out), _ptr(table), cap, seed, M, N, N, _es(out), RM, RN, mask, rid_offset,
                                 _ptr(failed))
    return failed[:nf].copy()


def cuckoo_hash(t: int, key: int, seed: int, cap: int) -> int:
    return int(lib().lpo_cuckoo_hash(t, key, seed, cap))


def cuckoo_lookup(table: np.ndarray, cap: int, sel: int, key: int, seed: int):
    """table: uint32 [2*cap*4] (T1 then T2, 16-byte entries {key, rec0, rec1, rec2})."""
    table = np.ascontiguousarray(table, dtype=np.uint32).reshape(-1)
    rec = np.zeros(max(sel, 1), dtype=np.uint32)
    ok = lib().lpo_cuckoo_lookup(_ptr(table), cap, sel, key, seed, _ptr(rec))
    return rec[:sel].copy() if ok else None


def cuckoo_insert(table: np.ndarray, cap: int, sel: int, key: int, seed: int, rec, max_evict: int = 128) -> int:
    assert table.flags.c_contiguous and table.dtype == np.uint32
    r = np.ascontiguousarray(np.asarray(rec, dtype=np.uint32).reshape(-1))
    if r.size == 0:
        r = np.zeros(1, dtype=np.uint32)
    return int(lib().lpo_cuckoo_insert(_ptr(table), cap, sel, key, seed, _ptr(r), max_evict))


def validate_cuckoo(out: np.ndarray, table: np.ndarray, cap: int, seed: int, RM: int, RN: int, mask: int,
                    rid_offset: int = 0) -> np.ndarray:
    out = np.ascontiguousarray(out)
    table = np.ascontiguousarray(table, dtype=np.uint32).reshape(-1)
    M, N = out.shape
    R = (M // RM) * (N // RN)
    failed = np.zeros(R, dtype=np.int64)
    nf = lib().lpo_validate_cuckoo(_ptr(out), _ptr(table), cap, seed, M, N, N, _es(out), RM, RN, mask, rid_offset,
                                   _ptr(failed))
    return failed[:nf].copy()


def gemm_block_f64(A: np.ndarray, B: np.ndarray, row0: int, col0: int, rows: int, cols: int) -> np.ndarray:
    """fp64 C[row0:row0+rows, col0:col0+cols] of A @ B (A, B float32, bf16-bits uint16 or int32)."""
    A = np.ascontiguousarray(A)
    B = np.ascontiguousarray(B)
    assert A.dtype == B.dtype and A.shape[1] == B.shape[0]
    is_bf16 = {np.dtype(np.uint16): 1, np.dtype(np.float32): 0, np.dtype(np.int32): 2}[A.dtype]
    C = np.zeros((rows, cols), dtype=np.float64)
    lib().lpo_gemm_block_f64(_ptr(A), A.shape[1], _ptr(B), B.shape[1], is_bf16, A.shape[1], row0, col0, rows, cols,
                             _ptr(C))
    return C


def round_bf16(x: np.ndarray) -> np.ndarray:
    x = np.ascontiguousarray(x, dtype=np.float64)
    out = np.zeros(x.shape, dtype=np.uint16)
    lib().lpo_round_bf16(_ptr(x), x.size, _ptr(out))
    return out


def stencil5_block(inp: np.ndarray, row0: int, col0: int, rows: int, cols: int) -> np.ndarray:
    inp = np.ascontiguousarray(inp, dtype=np.float32)
    H, W = inp.shape
    out = np.zeros((rows, cols), dtype=np.float32)
    lib().lpo_stencil5_block(_ptr(inp), H, W, W, row0, col0, rows, cols, _ptr(out))
    return out


def stencil5(inp: np.ndarray) -> np.ndarray:
    H, W = inp.shape
    return stencil5_block(inp, 0, 0, H, W)


def spmv_rows(row_ptr: np.ndarray, col: np.ndarray, val: np.ndarray, x: np.ndarray, row0: int = 0,
              rows: int | None = None) -> np.ndarray:
    """fp64 y[row0:row0+rows] of the CSR product A @ x (lpo_spmv_rows; row_ptr absolute offsets)."""
    row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
    col = np.ascontiguousarray(col, dtype=np.int32)
    val = np.ascontiguousarray(val, dtype=np.float32)
    x = np.ascontiguousarray(x, dtype=np.float32)
    if rows is None:
        rows = len(row_ptr) - 1 - row0
    y = np.zeros(rows, dtype=np.float64)
    lib().lpo_spmv_rows(_ptr(row_ptr), _ptr(col), _ptr(val), _ptr(x), row0, rows, _ptr(y))
    return y


def rel_err(got: np.ndarray, ref: np.ndarray) -> float:
    """Normwise relative error max|got-ref| / max|ref| (Reading R16)."""
    ref = np.asarray(ref, dtype=np.float64)
    d = np.abs(np.asarray(got, dtype=np.float64) - ref).max() if ref.size else 0.0
    m = np.abs(ref).max() if ref.size else 0.0
    return float(d / m) if m > 0 else float(d)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (np.asarray(b, dtype=np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32)
