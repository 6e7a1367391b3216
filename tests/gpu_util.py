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


def oracle_validate(out_h, ck_h, store, RM, RN, mask, rid_offset=0):
    """The oracle's failed set for any store kind, from host copies of out and the cksum buffer."""
    import oracle
    sel = oracle.selem(mask)
    R = (out_h.shape[0] // RM) * (out_h.shape[1] // RN)
    if store == "array":
        return oracle.validate_array(out_h, ck_h[:R * sel], RM, RN, mask, rid_offset=rid_offset)
    cap, seed = int(ck_h[0]), int(ck_h[1])
    if store.startswith("cuckoo"):
        return oracle.validate_cuckoo(out_h, ck_h[16:16 + 2 * cap * 4], cap, seed, RM, RN, mask, rid_offset=rid_offset)
    return oracle.validate_quad(out_h, ck_h[16:16 + cap * (1 + sel)], cap, seed, RM, RN, mask, rid_offset=rid_offset)


def check_store_table(ck_h, store, R, sel, recs, rid0=0):
    """Every rid is found exactly once by the oracle's lookup with its oracle record; an absent rid misses."""
    import oracle
    cap, seed = int(ck_h[0]), int(ck_h[1])
    if store.startswith("cuckoo"):
        table = ck_h[16:16 + 2 * cap * 4]
        keys = table.reshape(2 * cap, 4)[:, 0]
        lookup = lambda k: oracle.cuckoo_lookup(table, cap, sel, k, seed)  # noqa: E731
    else:
        table = ck_h[16:16 + cap * (1 + sel)]
        keys = table.reshape(cap, 1 + sel)[:, 0]
        lookup = lambda k: oracle.quad_lookup(table, cap, sel, k, seed)  # noqa: E731
    present = keys[keys != oracle.EMPTY_KEY]
    assert len(present) == R and len(set(present.tolist())) == R
    for rid in range(R):
        assert list(lookup(rid0 + rid)) == list(recs[rid]), rid
    assert lookup(rid0 + R + 7) is None
