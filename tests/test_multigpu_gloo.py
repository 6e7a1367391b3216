"""World-size-2 gloo tests of the multi-GPU host logic on CPU.

The device kernels cannot run here; what is exercised is the sharding plan, the
global region-id arithmetic, the count all-reduce and the union of per-rank
failed lists -- checked against the oracle's validation of the unsharded output.
"""
from __future__ import annotations

import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from lpsynth import gen
from paper_conf_iiswc_yudhakzs20_b200 import shard


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_plan_covers_rows_disjointly():
    for world in [1, 2, 3, 4, 8]:
        shards = [shard.plan(65536, 65536, 128, 128, world, r) for r in range(world)]
        assert shards[0].row_offset == 0
        for a, b in zip(shards, shards[1:]):
            assert a.row_offset + a.rows == b.row_offset and a.rid_offset + a.regions == b.rid_offset
        assert sum(s.regions for s in shards) == (65536 // 128) ** 2
        # global rid = (row_offset/RM + p) * Q + q  (include/liblp.h "Region ids are GLOBAL")
        for s in shards:
            assert s.rid_offset == (s.row_offset // 128) * (65536 // 128)


def test_plan_rejects_bad_splits():
    with pytest.raises(ValueError):
        shard.plan(100, 128, 32, 32, 1, 0)
    with pytest.raises(ValueError):
        shard.plan(128, 128, 128, 128, 2, 0)


def _worker(rank, world, port, tmp):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    M, N, RM, RN, mask = 256, 192, 32, 32, 3
    out = gen.generate(1, M, N, "uniform", "f32")                 # the global "persistent" output
    table = oracle.records(out, RM, RN, mask)                     # a clean record table
    bad = out.copy()
    R = (M // RM) * (N // RN)
    inj = np.random.default_rng(5).choice(R, 9, replace=False)
    Q = N // RN
    for rid in inj:                                               # corrupt one word per injected region
        p, q = divmod(int(rid), Q)
        bad.view(np.uint32)[p * RM + 3, q * RN + 5] ^= np.uint32(1 << 7)
    s = shard.plan(M, N, RM, RN, world, rank)
    # each rank validates only its band, producing GLOBAL rids
    local = oracle.validate_array(bad[s.row_offset:s.row_offset + s.rows], table[s.rid_offset:s.rid_offset + s.regions],
                                  RM, RN, mask, rid_offset=s.rid_offset)
    counts = torch.tensor([len(local), len(local), 0], dtype=torch.int64)
    shard.allreduce_counts(counts)
    union = shard.gather_failed(torch.from_numpy(local))
    np.save(os.path.join(tmp, f"r{rank}.npy"), np.array([counts.tolist(), sorted(union.tolist())], dtype=object),
            allow_pickle=True)
    dist.destroy_process_group()


def test_two_rank_count_allreduce_and_union_match_oracle():
    world = 2
    with tempfile.TemporaryDirectory() as tmp:
        mp.spawn(_worker, args=(world, _free_port(), tmp), nprocs=world, join=True)
        res = [np.load(os.path.join(tmp, f"r{r}.npy"), allow_pickle=True) for r in range(world)]
    M, N, RM, RN = 256, 192, 32, 32
    R = (M // RM) * (N // RN)
    inj = sorted(np.random.default_rng(5).choice(R, 9, replace=False).tolist())
    for counts, union in res:
        assert counts[0] == 9 and counts[1] == 9 and counts[2] == 0
        assert union == inj
