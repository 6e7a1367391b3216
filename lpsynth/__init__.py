"""Seeded synthetic workload inputs shared by the oracle and the CUDA path.

No Lazy-Persistency arithmetic lives here (see gen.py). ``device_fill`` is the
CUDA twin used for large operands; it requires lpsynth/libsynth.so (built by
``__graft_entry__.build()``) and a GPU.
"""
from __future__ import annotations

import ctypes
import os

from .gen import DTYPES, KINDS, generate, raw, splitmix64, values_f32, f32_to_bf16_bits  # noqa: F401
from . import csr  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libsynth.so")
        if not os.path.exists(path):
            raise RuntimeError("lpsynth/libsynth.so is not built; run __graft_entry__.build()")
        L = ctypes.CDLL(path)
        L.synth_fill.restype = ctypes.c_int
        L.synth_fill.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
                                 ctypes.c_int64, ctypes.c_int64, ctypes.c_uint64, ctypes.c_int,
                                 ctypes.c_int, ctypes.c_void_p]
        L.synth_csr_cols.restype = ctypes.c_int
        L.synth_csr_cols.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
                                     ctypes.c_uint64, ctypes.c_void_p, ctypes.c_void_p]
        _LIB = L
    return _LIB


def device_fill(tensor, seed: int, kind: str, dtype: str, row0: int = 0, ncols_global: int | None = None,
                stream=None) -> None:
    """Fill a 2-D CUDA tensor (rows x cols, row pitch = stride(0)) on `stream` (torch stream or None)."""
    import torch

    assert tensor.is_cuda and tensor.dim() == 2 and tensor.stride(1) == 1
    rows, cols = tensor.shape
    s = (stream or torch.cuda.current_stream()).cuda_stream
    rc = lib().synth_fill(tensor.data_ptr(), rows, cols, tensor.stride(0), row0,
                          cols if ncols_global is None else ncols_global, seed, KINDS[kind], DTYPES[dtype], s)
    if rc != 0:
        raise RuntimeError(f"synth_fill failed rc={rc}")


def device_csr(seed_len: int, seed_col: int, seed_val: int, rows: int, ncols: int, kind: str = "uniform",
               device="cuda", stream=None):
    """The synthetic CSR matrix of csr.py on the device: (row_ptr int64 [rows+1], col_idx int32 [nnz],
    values f32 [nnz]).  Row lengths / row_ptr are computed on the host (rows int64s); columns and
    values are generated in HBM by the device twins."""
    import torch

    rp_h = csr.row_ptr(seed_len, rows)
    nnz = int(rp_h[-1])
    rp = torch.from_numpy(rp_h).to(device)
    cols = torch.empty(nnz, dtype=torch.int32, device=device)
    vals = torch.empty((1, nnz), dtype=torch.float32, device=device)
    s = (stream or torch.cuda.current_stream()).cuda_stream
    rc = lib().synth_csr_cols(rp.data_ptr(), rows, 0, ncols, seed_col, cols.data_ptr(), s)
    if rc != 0:
        raise RuntimeError(f"synth_csr_cols failed rc={rc}")
    device_fill(vals, seed_val, kind, "f32", stream=stream)
    return rp, cols, vals.view(-1)
