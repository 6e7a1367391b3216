"""Shared helpers for the -m gpu parity tests (inputs from lpsynth, expectations from oracle)."""
from __future__ import annotations

import numpy as np
import torch

from lpsynth import gen


def host_to_dev(arr: np.ndarray, dtype: str, device="cuda"):
    """numpy (float32 or bf16-bits uint16) -> torch CUDA tensor of the right dtype."""
    if dtype == "bf16":
        t = torch.from_numpy(np.ascontiguousarray(arr).view(np.int16)).view(torch.bfloat16)
    elif dtype == "f32":
        t = torch.from_numpy(np.ascontiguousarray(arr, dtype=np.float32))
    elif dtype == "i32":
        t = torch.from_numpy(np.ascontiguousarray(arr, dtype=np.int32))
    else:
        raise ValueError(dtype)
    return t.to(device)


def dev_to_host(t) -> np.ndarray:
    """torch CUDA tensor -> numpy: float32 stays float32, bf16 becomes uint16 bits, int32 -> uint32."""
    t = t.detach().contiguous().cpu()
    if t.dtype == torch.bfloat16:
        return t.view(torch.int16).numpy().view(np.uint16)
    if t.dtype == torch.int32:
        return t.numpy().view(np.uint32)
    return t.numpy()


def make_inputs(seed: int, m: int, n: int, k: int, kind: str, dtype: str):
    A = gen.generate(seed, m, k, kind, dtype)
    B = gen.generate(seed + 100, k, n, kind, dtype)
    return A, B


def stale_image(seed: int, m: int, n: int, out_dtype: str):
    return gen.generate(seed + 500, m, n, "bits", out_dtype)
