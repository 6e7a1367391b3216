"""Reporting helpers (host logic).

The paper averages overheads as geomean(1 + o_i) - 1: that convention
reproduces Table V's 2.1% (L643-645) and Table IV's geomean row (L517-522)
from the per-benchmark entries (pinned in tests/test_host_logic.py).
"""
from __future__ import annotations

import math
from typing import Iterable


def overhead_pct(t_protected: float, t_unprotected: float) -> float:
    """LP overhead = slowdown of the protected kernel vs the same kernel without LP (L585)."""
    return 100.0 * (t_protected / t_unprotected - 1.0)


def geomean_overhead_pct(overheads_pct: Iterable[float]) -> float:
    """geomean(1 + o_i) - 1, in percent (the paper's averaging, L517-522 / L643-645)."""
    xs = [1.0 + o / 100.0 for o in overheads_pct]
    return 100.0 * (math.exp(sum(math.log(x) for x in xs) / len(xs)) - 1.0)


def space_overhead_pct(record_bytes: int, data_bytes: int) -> float:
    """Checksum-table bytes over protected data bytes (Table V 'Space overhead', L598)."""
    return 100.0 * record_bytes / data_bytes


def median(xs):
    s = sorted(xs)
    n = len(s)
    return s[n // 2] if n % 2 else 0.5 * (s[n // 2 - 1] + s[n // 2])


def quantile(xs, q: float) -> float:
    """Linear-interpolation quantile (numpy's default 'linear' method), q in [0, 1]."""
    s = sorted(xs)
    if not s:
        raise ValueError("empty sample")
    pos = q * (len(s) - 1)
    lo = int(math.floor(pos))
    hi = min(lo + 1, len(s) - 1)
    return s[lo] + (s[hi] - s[lo]) * (pos - lo)
