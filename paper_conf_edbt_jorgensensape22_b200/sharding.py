"""Row sharding for one process per GPU (host-side logic only).

Points are independent units: rank r owns a contiguous row range and
every k x d partial sum of a pass (H increments, centroid sums, deviation
sums, counts) is combined by one NCCL allreduce of int64 fixed-point values
inside the library (include/proclus.h, options.world_size > 1).

The kernels quantise each sum per sub-chunk of SUB points at a fixed scale,
and integer addition is associative, so when every shard boundary is a
multiple of SUB the totals - hence labels, medoids, dimensions and cost -
are bit-identical for any number of GPUs.  shard_rows() produces such
boundaries.
"""
from __future__ import annotations

SUB = 1024  # lcm of every sub-chunk size the kernels use (32 * points per lane)


def shard_rows(n: int, world: int, rank: int, align: int = SUB) -> tuple[int, int]:
    """[lo, hi) rows of `rank` out of `world`: balanced in units of `align`
    rows, every boundary a multiple of `align` (the last shard takes the
    ragged tail).  Shards may be empty when n < world * align."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad world/rank")
    if n < 0 or align < 1:
        raise ValueError("bad n/align")
    units = (n + align - 1) // align
    lo_u = units * rank // world
    hi_u = units * (rank + 1) // world
    lo = min(n, lo_u * align)
    hi = min(n, hi_u * align)
    return lo, hi


def nccl_unique_id_bytes() -> bytes:
    """A fresh 128-byte ncclUniqueId (rank 0 creates it, the launcher
    broadcasts it, e.g. with torch.distributed.broadcast_object_list)."""
    import torch

    return bytes(torch.cuda.nccl.unique_id())
