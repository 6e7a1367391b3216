"""Seeded synthetic workload inputs shared by the oracle and the CUDA path.

No Lazy-Persistency arithmetic lives here (see gen.py). ``device_fill`` is the
CUDA twin used for large operands; it requires lpsynth/libsynth.so (built by
``__graft_entry__.build()``) and a GPU.
"""
from __future__ import annotations

import ctypes
import os

from .gen import DTYPES, KINDS, generate, raw, splitmix64, values_f32, f32_to_bf16_bits  # noqa: F401

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
