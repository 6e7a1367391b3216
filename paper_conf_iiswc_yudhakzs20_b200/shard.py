"""Region sharding across GPUs (host logic).

LP regions are associative and independent (L51, L181) and the record array is
indexed by region id (L349), so each GPU owns a disjoint contiguous band of
region rows: rank g owns output rows [g*M/G, (g+1)*M/G) -- i.e. global rids
[g*R/G, (g+1)*R/G) -- together with its A row panel, a full B, its C shard and
its slice of the record table.  Protected run, validation, compaction and
recovery are all local; the only exchange is an all-reduce(SUM) of the int64
counts {n_failed, n_recovered, n_failed_after} (16-24 bytes, latency-bound),
issued straight from device memory on the compute stream.
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class Shard:
    rank: int
    world: int
    row_offset: int   # first global output row of this shard
    rows: int         # rows of this shard
    rid_offset: int   # first global region id
    regions: int      # regions of this shard


def plan(global_m: int, n: int, region_m: int, region_n: int, world: int, rank: int) -> Shard:
    """Contiguous row-band shard of a global_m x n output, in whole region rows."""
    if global_m % region_m or n % region_n:
        raise ValueError("output must be a whole number of regions")
    P = global_m // region_m
    Q = n // region_n
    if P < world:
        raise ValueError(f"{P} region rows cannot be split over {world} ranks")
    lo = (P * rank) // world
    hi = (P * (rank + 1)) // world
    return Shard(rank, world, lo * region_m, (hi - lo) * region_m, lo * Q, (hi - lo) * Q)


def csr_band(rp_global, row0: int, rows: int):
    """A rank's slice of a CSR matrix for SpMV row-band shards: rows [row0, row0 + rows) with global row_ptr
    rp_global (int64, at least row0 + rows + 1 entries).  The rank's value / column arrays start at global nnz
    index g0 = rp_global[row0] rounded down to a multiple of 4 (up to 3 leading elements of the previous row,
    never summed), so every region's 16-B vector and 2048-nnz chunk grid (Reading R25) sit exactly where they
    sit in the unsharded matrix: the sharded product is bit-identical to the single-GPU one.
    Returns (g0, local row_ptr = rp_global[row0 : row0 + rows + 1] - g0, local nnz = rp[-1] - g0, pad)."""
    import numpy as np

    sl = np.asarray(rp_global[row0:row0 + rows + 1], dtype=np.int64)
    if len(sl) != rows + 1:
        raise ValueError("row_ptr too short for the band")
    g0 = int(sl[0]) & ~3
    local = sl - g0
    return g0, local, int(local[-1]), int(sl[0]) - g0


def allreduce_counts(counts, group=None):
    """SUM all-reduce of the device int64 count vector (the one collective of the path)."""
    import torch.distributed as dist

    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    return counts


def gather_failed(local_failed, group=None):
    """All-gather of the per-rank failed-rid lists (off the hot path; used by checks)."""
    import torch
    import torch.distributed as dist

    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return local_failed
    n = torch.tensor([local_failed.numel()], dtype=torch.int64, device=local_failed.device)
    sizes = [torch.zeros_like(n) for _ in range(dist.get_world_size(group))]
    dist.all_gather(sizes, n, group=group)
    mx = int(max(int(s.item()) for s in sizes))
    pad = torch.full((mx,), -1, dtype=torch.int64, device=local_failed.device)
    pad[:local_failed.numel()] = local_failed
    outs = [torch.empty_like(pad) for _ in sizes]
    dist.all_gather(outs, pad, group=group)
    return torch.cat([o[:int(s.item())] for o, s in zip(outs, sizes)])


def nvls_counter(device, group=None):
    """A 16 x int64 counter buffer in torch symmetric memory, bound to an NVSwitch multicast object on every
    rank (the NVLS-fused failed count, lp_attach_nvls_count).  Returns (multicast_ptr, local tensor) or
    (None, reason) when the fabric offers no multicast (e.g. one GPU, or no NVSwitch)."""
    import torch
    import torch.distributed as dist
    import torch.distributed._symmetric_memory as symm_mem

    try:
        t = symm_mem.empty(16, dtype=torch.int64, device=device)
        t.zero_()
        hdl = symm_mem.rendezvous(t, group if group is not None else dist.group.WORLD)
        if not getattr(hdl, "has_multicast_support", lambda: False)() or not hdl.multicast_ptr:
            return None, "symmetric memory without multicast support on this fabric"
        torch.cuda.synchronize(device)
        hdl.barrier()
        return int(hdl.multicast_ptr), t
    except Exception as e:  # noqa: BLE001 -- reported in the bench line, the NCCL all-reduce stays in place
        return None, f"{type(e).__name__}: {e}"
