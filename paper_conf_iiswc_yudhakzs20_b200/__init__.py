"""B200-native Lazy Persistency (LP) hot path -- Yudha et al., IISWC 2020.

liblp (C ABI, include/liblp.h) + a thin ctypes binding (lp.py); host helpers for
reporting (report.py) and region sharding across GPUs (shard.py).
"""
from . import lp  # noqa: F401
from .lp import LP, Workload, choose_regions, parse_cksum  # noqa: F401
