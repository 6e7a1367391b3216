"""CPU tests of the host logic and of the C-ABI boundary (no GPU, no kernel launches)."""
from __future__ import annotations

import os
import re

import numpy as np
import pytest

from paper_conf_iiswc_yudhakzs20_b200 import lp, report

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")


def _golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


# --------------------------------------------------------------------------- the paper's averaging convention
def test_geomean_reproduces_table_v():
    rows = _golden("table_v_overheads.txt")
    vals = [float(v) for name, v in rows if name != "GEOMEAN"]
    printed = float([v for name, v in rows if name == "GEOMEAN"][0])
    assert round(report.geomean_overhead_pct(vals), 1) == printed


def test_geomean_reproduces_table_iv():
    rows = _golden("table_iv_overheads.txt")
    body = [r for r in rows if r[0] != "GEOMEAN"]
    printed = [float(x) for x in [r for r in rows if r[0] == "GEOMEAN"][0][1:]]
    for col in range(4):
        g = report.geomean_overhead_pct([float(r[1 + col]) for r in body])
        # the paper prints 29.4 / 63.3 / 31.7 / 65.8; the convention gives 29.31 / 63.26 / 31.66 / 65.83
        assert abs(g - printed[col]) < 0.1, (col, g)


def test_overhead_and_space_helpers():
    assert report.overhead_pct(1.062, 1.0) == pytest.approx(6.2)
    assert report.space_overhead_pct(8, 4096) == pytest.approx(0.1953125)


# --------------------------------------------------------------------------- the C ABI (loads on a CPU box)
def _header_symbols():
    with open(os.path.join(ROOT, "include", "liblp.h")) as f:
        text = f.read()
    return sorted(set(re.findall(r"LP_API\s+[\w\s\*]+?\b(lp_\w+)\s*\(", text)))


def test_library_exports_every_declared_symbol():
    L = lp.lib()
    syms = _header_symbols()
    assert len(syms) >= 15
    for s in syms:
        assert hasattr(L, s), s
    assert set(syms) == set(lp.EXPORTED)
    assert L.lp_abi_version() == 100


def test_config_argument_errors():
    with pytest.raises(lp.LPError) as e:
        lp.LP(0, 32)
    assert e.value.status == lp.LP_ERR_INVALID_ARG
    with pytest.raises(lp.LPError):
        lp.LP(32, 32, cksum=8)
    with pytest.raises(lp.LPError):
        lp.LP(32, 32, cksum=0, store="quad_cas")


def test_region_count_matches_table_iii_and_space_matches_table_v():
    (M, N, rm, rn, regions, space), = _golden("tmm_regions.txt")
    h = lp.LP(int(rm), int(rn), cksum="mod|xor")
    wl = lp.Workload.tmm(None, None, out_dtype="f32", m=int(M), n=int(N), k=int(M))
    assert h.num_regions(wl) == int(regions)
    ck = h.cksum_bytes(wl)
    assert ck == int(regions) * 8
    assert round(report.space_overhead_pct(ck, int(M) * int(N) * 4), 1) == float(space)


def test_cksum_bytes_hash_store_sizing():
    h = lp.LP(128, 128, cksum="mod|xor", store="quad_cas")
    wl = lp.Workload.tmm(None, None, out_dtype="bf16", m=16384, n=16384, k=16384)
    R = h.num_regions(wl)
    assert R == 16384
    b = h.cksum_bytes(wl)
    cap = (b - 64) // 12
    assert (b - 64) % 12 == 0
    assert cap >= R / 0.7 and all(cap % d for d in range(2, int(cap ** 0.5) + 1))  # smallest prime >= R/0.7
    assert not any(all(c % d for d in range(2, int(c ** 0.5) + 1)) for c in range(int(np.ceil(R / 0.7)), cap))


def test_workload_divisibility_errors():
    h = lp.LP(32, 32, cksum="mod")
    with pytest.raises(lp.LPError) as e:
        h.num_regions(lp.Workload.tmm(None, None, out_dtype="f32", m=100, n=64, k=64))
    assert e.value.status == lp.LP_ERR_INVALID_ARG
    with pytest.raises(lp.LPError):
        h.num_regions(lp.Workload.tmm(None, None, out_dtype="f32", m=64, n=64, k=64, row_offset=16, global_m=128))
    # shard: global rid offset = (row_offset/RM) * (N/RN)
    assert h.num_regions(lp.Workload.tmm(None, None, out_dtype="f32", m=64, n=64, k=64, row_offset=64,
                                         global_m=128)) == 4


def test_device_calls_fail_loudly_without_gpu():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    h = lp.LP(32, 32, cksum="mod")
    wl = lp.Workload.tmm(None, None, out_dtype="f32", m=64, n=64, k=64)
    wl.a, wl.b = 256, 512  # fake (aligned) addresses: must be refused before any launch
    with pytest.raises(lp.LPError) as e:
        h.run_protected(wl, 1024, 2048, stream=0)
    assert e.value.status == lp.LP_ERR_UNSUPPORTED


def test_choose_regions_is_seeded_and_rounded():
    a = lp.choose_regions(64, 0.05, 7)
    assert len(a) == 3 and np.all(np.diff(a) > 0)          # k = floor(0.05*64 + 0.5) = 3
    assert np.array_equal(a, lp.choose_regions(64, 0.05, 7))
    assert len(lp.choose_regions(65536, 0.01, 1)) == 655 and len(lp.choose_regions(65536, 0.10, 1)) == 6554
    assert len(lp.choose_regions(65536, 0.50, 1)) == 32768


class _Fake:
    """A fake device buffer: an address (aligned or not) and an element count -- argument checks run
    before any device access, so these never reach a kernel."""

    def __init__(self, addr, n=1 << 20):
        self.addr, self.n = addr, n

    def data_ptr(self):
        return self.addr

    def numel(self):
        return self.n


def _status(fn):
    with pytest.raises(lp.LPError) as e:
        fn()
    return e.value.status


def test_validate_recover_inject_argument_errors():
    """The boundary's synchronous argument errors (liblp.h conventions): every one is refused before a
    launch, on a machine with or without a GPU."""
    h = lp.LP(32, 32, cksum="mod|xor")
    wl = lp.Workload.tmm(None, None, out_dtype="f32", m=64, n=64, k=64)      # R = 4
    A = _Fake(1 << 20)
    assert _status(lambda: h.validate(wl, A, A, _Fake(1 << 20, 3), A, A, stream=0)) == lp.LP_ERR_INVALID_ARG   # cap < R
    assert _status(lambda: h.validate(wl, None, A, A, A, A, stream=0)) == lp.LP_ERR_INVALID_ARG               # null out
    assert _status(lambda: h.validate(wl, _Fake((1 << 20) + 4), A, A, A, A, stream=0)) == lp.LP_ERR_INVALID_ARG  # misaligned
    assert _status(lambda: h.validate(wl, A, A, A, A, None, stream=0)) == lp.LP_ERR_INVALID_ARG               # no workspace
    h0 = lp.LP(32, 32, cksum=0)
    assert _status(lambda: h0.validate(wl, A, A, A, A, A, stream=0)) == lp.LP_ERR_STATE                       # unprotected
    assert _status(lambda: h.recover(wl, A, A, None, A, stream=0)) == lp.LP_ERR_INVALID_ARG                   # no list
    assert _status(lambda: h.inject(wl, A, A, A, _Fake(1 << 20, 5), stream=0)) == lp.LP_ERR_INVALID_ARG       # n > R
    assert _status(lambda: h.inject(wl, A, A, None, _Fake(1 << 20, 2), mode="stale_region", stream=0)) == lp.LP_ERR_INVALID_ARG
    assert _status(lambda: h.inject(wl, A, A, A, _Fake(1 << 20, 2), mode=9, stream=0)) == lp.LP_ERR_INVALID_ARG
    empty = lp.Workload.tmm(None, None, out_dtype="f32", m=0, n=64, k=64)
    assert _status(lambda: h.num_regions(empty)) == lp.LP_ERR_INVALID_ARG                          # m = 0
    bad_ld = lp.Workload.tmm(None, None, out_dtype="f32", m=64, n=64, k=64)
    bad_ld.ldc = 32
    assert _status(lambda: h.num_regions(bad_ld)) == lp.LP_ERR_INVALID_ARG                         # ldc < n
    assert "ldc" in lp.lib().lp_last_error().decode()


def test_spmv_and_stencil_shape_errors():
    hs = lp.LP(1, 1000, cksum="mod")                                        # not a power of two
    wl = lp.Workload.spmv(None, None, None, None, m=4000)
    assert _status(lambda: hs.num_regions(wl)) == lp.LP_ERR_UNSUPPORTED
    h2 = lp.LP(2, 1024, cksum="mod")                                        # SPMV regions are 1 x region_n
    assert _status(lambda: h2.num_regions(lp.Workload.spmv(None, None, None, None, m=4096))) == lp.LP_ERR_INVALID_ARG
    h3 = lp.LP(1, 1024, cksum="mod")
    assert _status(lambda: h3.num_regions(lp.Workload.spmv(None, None, None, None, m=1000))) == lp.LP_ERR_INVALID_ARG
    assert h3.num_regions(lp.Workload.spmv(None, None, None, None, m=4096)) == 4


def test_quantile_matches_numpy():
    import numpy as np
    rng = np.random.default_rng(3)
    for n in [1, 2, 5, 40]:
        xs = rng.standard_normal(n).tolist()
        for q in [0.0, 0.25, 0.5, 0.75, 1.0]:
            assert report.quantile(xs, q) == pytest.approx(float(np.quantile(xs, q)))


def test_bench_self_launch_reference_two_ranks():
    """`bench.py --impl reference --gpus 2` outside torchrun re-launches itself with 2 ranks; rank 0 alone runs the
    oracle and prints one line, the other rank exits 0 (no GPU needed)."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--steps", "1",
                        "--warmup", "0", "--workload", "tmm8192_bf16"], cwd=root, capture_output=True, text=True,
                       timeout=300, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["value"] > 0


def test_nvls_attach_argument_errors():
    """lp_attach_nvls_count is host-checked (no GPU needed): the config flag is required, both addresses are
    needed, 64-B alignment, the single-GPU emulation only with world 1; NULL, NULL detaches."""
    from paper_conf_iiswc_yudhakzs20_b200 import lp
    h = lp.LP(128, 128, cksum="mod|xor")
    with pytest.raises(lp.LPError):
        h.attach_nvls_count(4096, 4096, 1)                 # flag missing
    h2 = lp.LP(128, 128, cksum="mod|xor", nvls_count=True)
    for args in [(4096, None, 2), (4096, 8192 + 8, 2), (4096, 4096, 2), (4096, 8192, 0)]:
        with pytest.raises(lp.LPError):
            h2.attach_nvls_count(*args)
    h2.attach_nvls_count(4096, 8192, 8)                    # accepted (no device access at attach time)
    h2.attach_nvls_count(None, None, 1)
