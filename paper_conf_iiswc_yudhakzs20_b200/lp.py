"""Thin Python binding of liblp (include/liblp.h) -- argument marshalling only.

Every step of the Lazy Persistency hot path runs in liblp's CUDA kernels; this
module only converts torch tensors / ints into the C ABI's pointers and sizes.
torch provides device memory and streams (plumbing). There is no CPU fallback:
if liblp.so is missing the import of the handle fails loudly.

Names follow the paper: a *region* is the LP unit of recovery (L51, L181), the
*record* is the region's checksum entry (L192, L349), ``lp_config`` ~
``#pragma nvm lpcuda_init`` (L357, L528).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import Optional

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liblp.so")

# ---- enums (mirror include/liblp.h)
LP_OK, LP_ERR_INVALID_ARG, LP_ERR_UNSUPPORTED, LP_ERR_CUDA, LP_ERR_CAPACITY, LP_ERR_STATE = range(6)
CK_NONE, CK_MOD, CK_XOR, CK_ADLER32 = 0, 1, 2, 4
STORE_ARRAY, STORE_QUAD_CAS, STORE_QUAD_LOCK, STORE_CUCKOO, STORE_CUCKOO_LOCK = 0, 1, 2, 3, 4
F32, BF16, I32 = 0, 1, 2
WL_TMM, WL_STENCIL5, WL_SPMV = 0, 1, 2
BODY_AUTO, BODY_SIMT, BODY_TCGEN05 = 0, 1, 2
FLAG_TC_1CTA = 1
FLAG_NO_SHUFFLE = 2
FLAG_NO_PAIRING = 4
FLAG_NO_FUSED_COMPACT = 8
FLAG_RECOVER_TILE128 = 16
FLAG_CUCKOO_SHORT_CHAINS = 32
FLAG_NVLS_COUNT = 64
FLAG_RECOVER_SLICES128 = 128
FLAG_TEST_SKIP_REEXEC = 256
INJ_STALE_WORDS, INJ_STALE_REGION, INJ_BITFLIP, INJ_STALE_RECORD = 0, 1, 2, 3

CK_NAMES = {"none": 0, "mod": 1, "xor": 2, "adler": 4, "adler32": 4}
STORE_NAMES = {"array": 0, "quad_cas": 1, "quad": 1, "quad_lock": 2, "cuckoo": 3, "cuckoo_lock": 4}
BODY_NAMES = {"auto": 0, "simt": 1, "tcgen05": 2}
INJ_NAMES = {"stale_words": 0, "stale_region": 1, "bitflip": 2, "stale_record": 3}
EXPORTED = ["lp_config", "lp_destroy", "lp_num_regions", "lp_cksum_bytes", "lp_workspace_bytes", "lp_cksum_init",
            "lp_run_protected", "lp_validate", "lp_recover", "lp_region_checksums", "lp_inject", "lp_stats",
            "lp_device_sm_count", "lp_last_error", "lp_abi_version", "lp_fn_study", "lp_check_recover",
            "lp_attach_nvls_count", "lp_recover_count", "lp_check_recover_ws",
            "lp_recover_revalidate"]


def parse_cksum(spec) -> int:
    if isinstance(spec, int):
        return spec
    m = 0
    for part in str(spec).lower().replace("+", "|").split("|"):
        part = part.strip()
        if part:
            m |= CK_NAMES[part]
    return m


def selem(mask: int) -> int:
    return bin(mask & 7).count("1")


class LPError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"liblp status {status}: {msg}")
        self.status = status


class Config(ctypes.Structure):
    _fields_ = [("region_m", ctypes.c_int32), ("region_n", ctypes.c_int32), ("cksum", ctypes.c_uint32),
                ("store", ctypes.c_int32), ("device", ctypes.c_int32), ("body", ctypes.c_int32),
                ("hash_seed", ctypes.c_uint32), ("flags", ctypes.c_uint32)]


class CWorkload(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("in_dtype", ctypes.c_int32), ("out_dtype", ctypes.c_int32),
                ("reserved", ctypes.c_int32), ("m", ctypes.c_int64), ("n", ctypes.c_int64), ("k", ctypes.c_int64),
                ("a", ctypes.c_void_p), ("lda", ctypes.c_int64), ("b", ctypes.c_void_p), ("ldb", ctypes.c_int64),
                ("ldc", ctypes.c_int64), ("row_offset", ctypes.c_int64), ("global_m", ctypes.c_int64),
                ("row_ptr", ctypes.c_void_p), ("col_idx", ctypes.c_void_p), ("nnz", ctypes.c_int64)]


_LIB = None


def lib():
    """Load liblp.so (raises if it has not been built -- there is no fallback)."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(LIB_PATH)
        P, I64, U32, U64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint32, ctypes.c_uint64
        pw = ctypes.POINTER(CWorkload)
        sig = {
            "lp_config": [ctypes.POINTER(Config), ctypes.POINTER(ctypes.c_void_p)],
            "lp_destroy": [P],
            "lp_num_regions": [P, pw, ctypes.POINTER(I64)],
            "lp_cksum_bytes": [P, pw, ctypes.POINTER(ctypes.c_size_t)],
            "lp_workspace_bytes": [P, pw, ctypes.POINTER(ctypes.c_size_t)],
            "lp_cksum_init": [P, pw, P, P],
            "lp_run_protected": [P, pw, P, P, P],
            "lp_validate": [P, pw, P, P, P, I64, P, P, P],
            "lp_recover": [P, pw, P, P, P, P, P, P],
            "lp_recover_count": [P, pw, P, P, P, P, P, P, P],
            "lp_recover_revalidate": [P, pw, P, P, P, P, P, P, P, P],
            "lp_region_checksums": [P, pw, P, P, P],
            "lp_inject": [P, pw, P, P, P, P, I64, U32, U64, P],
            "lp_stats": [P, pw, P, P, P],
            "lp_fn_study": [P, U32, ctypes.c_int32, I64, U64, I64, P, P, I64, P],
            "lp_check_recover": [P, pw, P, P, P, P],
            "lp_check_recover_ws": [P, pw, P, P, P, P, P],
            "lp_attach_nvls_count": [P, P, P, ctypes.c_int32],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.lp_device_sm_count.argtypes = [P]
        L.lp_device_sm_count.restype = ctypes.c_int32
        L.lp_last_error.argtypes = []
        L.lp_last_error.restype = ctypes.c_char_p
        L.lp_abi_version.argtypes = []
        L.lp_abi_version.restype = ctypes.c_int32
        _LIB = L
    return _LIB


def _check(status: int):
    if status != LP_OK:
        raise LPError(status, lib().lp_last_error().decode())


def _ptr(t) -> Optional[int]:
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


def _stream(stream) -> Optional[int]:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


_DT = {"f32": F32, "fp32": F32, "float32": F32, "bf16": BF16, "bfloat16": BF16, "i32": I32, "int32": I32}


def _dt_of(x) -> int:
    if isinstance(x, int):
        return x
    if isinstance(x, str):
        return _DT[x]
    import torch
    return {torch.float32: F32, torch.bfloat16: BF16, torch.int32: I32}[x]


@dataclass
class Workload:
    """A region body's problem (mirrors lp_workload_t). Tensors stay owned by the caller."""
    kind: int
    m: int
    n: int
    k: int = 0
    a: object = None
    b: object = None
    in_dtype: int = F32
    out_dtype: int = F32
    lda: int = 0
    ldb: int = 0
    ldc: int = 0
    row_offset: int = 0
    global_m: int = 0
    row_ptr: object = None
    col_idx: object = None
    nnz: int = 0

    @staticmethod
    def tmm(a, b, out_dtype="bf16", m=None, n=None, k=None, row_offset=0, global_m=None, ldc=None) -> "Workload":
        """C[m,n] = A[m,k] B[k,n] (Listing 2 / Listing 6); a, b torch tensors (or None for sizing only)."""
        if a is not None:
            m, k = a.shape
            n = b.shape[1]
            ind = _dt_of(a.dtype)
            lda, ldb = a.stride(0), b.stride(0)
        else:
            ind, lda, ldb = _dt_of(out_dtype), k, n
        return Workload(WL_TMM, m, n, k, a, b, ind, _dt_of(out_dtype), lda, ldb, ldc or n, row_offset,
                        global_m if global_m is not None else row_offset + m)

    @staticmethod
    def stencil(inp, H=None, W=None, row_offset=0, global_m=None) -> "Workload":
        """out = 5-point stencil of inp (Reading R19).  Row shard: inp = rows [row_offset, row_offset + H) of a
        global_m-row input, as a view whose neighbouring rows (the halo) are readable where the domain continues."""
        if inp is not None:
            H, W = inp.shape
            lda = inp.stride(0)
        else:
            lda = W
        return Workload(WL_STENCIL5, H, W, 0, inp, None, F32, F32, lda, 0, W, row_offset,
                        global_m if global_m is not None else row_offset + H)

    @staticmethod
    def spmv(values, x, row_ptr, col_idx, m=None, row_offset=0, global_m=None) -> "Workload":
        """y[m] = A x for the CSR matrix (row_ptr int64 [m+1], col_idx int32 [nnz], values f32 [nnz]) and
        x f32 [n] (the paper's SPMV, Table I; N4).  Regions = region_n consecutive rows of y (region_m = 1);
        out is allocated as [m / region_n, region_n] by LP.alloc.  Tensors None -> sizing only (give m, n=len(x))."""
        if row_ptr is not None:
            m = row_ptr.numel() - 1
        n = x.numel() if x is not None else 1
        nnz = values.numel() if values is not None else 0
        w = Workload(WL_SPMV, m, n, 0, values, x, F32, F32, 0, 0, 0, row_offset,
                     global_m if global_m is not None else row_offset + m)
        w.row_ptr, w.col_idx, w.nnz = row_ptr, col_idx, nnz
        return w

    def c(self) -> CWorkload:
        return CWorkload(self.kind, self.in_dtype, self.out_dtype, 0, self.m, self.n, self.k, _ptr(self.a), self.lda,
                         _ptr(self.b), self.ldb, self.ldc, self.row_offset, self.global_m or self.row_offset + self.m,
                         _ptr(self.row_ptr), _ptr(self.col_idx), self.nnz)


class LP:
    """One liblp handle: region shape + checksum type + store (lp_config)."""

    def __init__(self, region_m: int, region_n: int, cksum="mod|xor", store="array", device: int = 0,
                 body="auto", hash_seed: int = 0x9747B28C,
                 tc_pair: bool = True, shuffle: bool = True, pairing: bool = True, fused_compact: bool = True,
                 recover_slices: bool = True, cuckoo_short_chains: bool = False, nvls_count: bool = False,
                 recover_slices128: bool = False, test_skip_reexec: bool = False):
        self.mask = parse_cksum(cksum)
        self.store = STORE_NAMES[store] if isinstance(store, str) else int(store)
        self.body = BODY_NAMES[body] if isinstance(body, str) else int(body)
        self.region = (region_m, region_n)
        self.device = device
        self.cfg = Config(region_m, region_n, self.mask, self.store, device, self.body, hash_seed,
                          (0 if tc_pair else FLAG_TC_1CTA) | (0 if shuffle else FLAG_NO_SHUFFLE) |
                          (0 if pairing else FLAG_NO_PAIRING) | (0 if fused_compact else FLAG_NO_FUSED_COMPACT) |
                          (0 if recover_slices else FLAG_RECOVER_TILE128) |
                          (FLAG_CUCKOO_SHORT_CHAINS if cuckoo_short_chains else 0) |
                          (FLAG_NVLS_COUNT if nvls_count else 0) |
                          (FLAG_RECOVER_SLICES128 if recover_slices128 else 0) |
                          (FLAG_TEST_SKIP_REEXEC if test_skip_reexec else 0))
        h = ctypes.c_void_p()
        _check(lib().lp_config(ctypes.byref(self.cfg), ctypes.byref(h)))
        self._h = h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and _LIB is not None:
            _LIB.lp_destroy(h)
            self._h = None

    @property
    def selem(self) -> int:
        return selem(self.mask)

    # ---- sizing (host only)
    def num_regions(self, wl: Workload) -> int:
        r = ctypes.c_int64()
        _check(lib().lp_num_regions(self._h, ctypes.byref(wl.c()), ctypes.byref(r)))
        return r.value

    def cksum_bytes(self, wl: Workload) -> int:
        b = ctypes.c_size_t()
        _check(lib().lp_cksum_bytes(self._h, ctypes.byref(wl.c()), ctypes.byref(b)))
        return b.value

    def workspace_bytes(self, wl: Workload) -> int:
        b = ctypes.c_size_t()
        _check(lib().lp_workspace_bytes(self._h, ctypes.byref(wl.c()), ctypes.byref(b)))
        return b.value

    def sm_count(self) -> int:
        return int(lib().lp_device_sm_count(self._h))

    # ---- device calls (enqueue on `stream`, no sync)
    def cksum_init(self, wl, ck, stream=None):
        _check(lib().lp_cksum_init(self._h, ctypes.byref(wl.c()), _ptr(ck), _stream(stream)))

    def run_protected(self, wl, out, ck, stream=None):
        _check(lib().lp_run_protected(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(ck), _stream(stream)))

    def validate(self, wl, out, ck, failed, d_n, workspace, stream=None):
        _check(lib().lp_validate(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(ck), _ptr(failed), failed.numel(),
                                 _ptr(d_n), _ptr(workspace), _stream(stream)))

    def recover(self, wl, out, ck, failed, d_n, workspace=None, stream=None, d_n_recovered=None):
        """lp_recover; with d_n_recovered (device int64[1]) lp_recover_count: regions rewritten."""
        if d_n_recovered is None:
            _check(lib().lp_recover(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(ck), _ptr(failed), _ptr(d_n),
                                    _ptr(workspace), _stream(stream)))
        else:
            _check(lib().lp_recover_count(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(ck), _ptr(failed),
                                          _ptr(d_n), _ptr(workspace), _ptr(d_n_recovered), _stream(stream)))

    def recover_revalidate(self, wl, out, ck, failed, d_n, workspace, d_n_after, d_n_recovered=None, stream=None):
        """lp_recover_revalidate: recover the failed list and re-validate the whole output, the unflagged regions
        on a side stream beside the recovery; *d_n_after (device int64[1]) = regions still mismatching."""
        _check(lib().lp_recover_revalidate(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(ck), _ptr(failed), _ptr(d_n),
                                           _ptr(workspace), _ptr(d_n_after), _ptr(d_n_recovered), _stream(stream)))

    def check_recover(self, wl, out, ck, d_n_recovered, workspace=None, stream=None):
        """Listing 7's same-grid check-and-recover (N2): validate + in-place re-execution in one kernel; with a
        workspace the TMM form deals the failed tiles over all CTA pairs (lp_check_recover_ws)."""
        if workspace is None:
            _check(lib().lp_check_recover(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(ck), _ptr(d_n_recovered),
                                          _stream(stream)))
        else:
            _check(lib().lp_check_recover_ws(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(ck),
                                             _ptr(d_n_recovered), _ptr(workspace), _stream(stream)))

    def attach_nvls_count(self, mc_ptr, uc_ptr, world_size: int):
        """NVLS-fused all-rank failed count (lp_attach_nvls_count); pointers are ints or tensors (None, None: off)."""
        _check(lib().lp_attach_nvls_count(self._h, _ptr(mc_ptr), _ptr(uc_ptr), int(world_size)))

    def region_checksums(self, wl, out, records, stream=None):
        _check(lib().lp_region_checksums(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(records), _stream(stream)))

    def inject(self, wl, out, ck, stale, rids, mode="stale_words", seed: int = 0, stream=None):
        m = INJ_NAMES[mode] if isinstance(mode, str) else int(mode)
        _check(lib().lp_inject(self._h, ctypes.byref(wl.c()), _ptr(out), _ptr(ck), _ptr(stale), _ptr(rids),
                               rids.numel(), m, seed, _stream(stream)))

    def stats(self, wl, ck, d_stats, stream=None):
        _check(lib().lp_stats(self._h, ctypes.byref(wl.c()), _ptr(ck), _ptr(d_stats), _stream(stream)))

    def fn_study(self, model, kmax, region_words, seed, trials, d_counts, dump=None, dump_trials=0, stream=None):
        """False-negative study (N3): see lp_fn_study in include/liblp.h."""
        m = {"random_words": 0, "bitflips": 1, "adversarial": 2, "zeroed": 3}[model] if isinstance(model, str) \
            else int(model)
        _check(lib().lp_fn_study(self._h, m, kmax, region_words, seed, trials, _ptr(d_counts), _ptr(dump),
                                 dump_trials, _stream(stream)))

    # ---- buffer helper (torch allocations; the caller owns them)
    def alloc(self, wl: Workload, device=None):
        """Allocate out, cksum, failed list, d_n (int64[1]) and workspace on the device."""
        import torch
        dev = torch.device("cuda", self.device if device is None else device)
        dt = {BF16: torch.bfloat16, F32: torch.float32, I32: torch.int32}[wl.out_dtype]
        R = self.num_regions(wl)
        if wl.kind == WL_SPMV:   # y viewed as [m / region_n][region_n]
            out = torch.empty((wl.m // self.region[1], self.region[1]), dtype=dt, device=dev)
        else:
            out = torch.empty((wl.m, wl.ldc), dtype=dt, device=dev)[:, :wl.n]
        ckb = max(self.cksum_bytes(wl), 16)
        ck = torch.empty((ckb + 3) // 4, dtype=torch.int32, device=dev)
        failed = torch.empty(max(R, 1), dtype=torch.int64, device=dev)
        d_n = torch.zeros(1, dtype=torch.int64, device=dev)
        ws = torch.zeros(self.workspace_bytes(wl), dtype=torch.uint8, device=dev)   # zero-filled once (ABI contract)
        return out, ck, failed, d_n, ws


def choose_regions(R: int, frac: float, seed: int):
    """k = floor(frac*R + 0.5) distinct region ids, seeded (harness; Reading R11). numpy, host."""
    import numpy as np
    k = int(frac * R + 0.5)
    rng = np.random.default_rng(seed)
    return np.sort(rng.choice(R, size=k, replace=False)).astype(np.int64)
