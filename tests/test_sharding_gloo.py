"""Multi-process (world_size 2, gloo, CPU) tests of the row-sharded path's
host logic: shard planning and the exact combination of per-rank
fixed-point partial sums (the quantity the library allreduces over NCCL)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_edbt_jorgensensape22_b200.sharding import SUB, shard_rows
import synth

SUBCHUNK = 64  # points per warp sub-chunk of the assign / final passes (32 x 2)


def test_shard_rows_cover_and_align():
    for n in (1, 63, 1000, 1024, 4097, 1_000_000, 3 * SUB + 5):
        for world in (1, 2, 3, 4, 8):
            got = [shard_rows(n, world, r) for r in range(world)]
            assert got[0][0] == 0 and got[-1][1] == n
            for (lo, hi), (lo2, _) in zip(got, got[1:]):
                assert hi == lo2 and lo <= hi
            for lo, hi in got[:-1]:
                assert lo % SUB == 0 and (hi % SUB == 0 or hi == n)
            sizes = [hi - lo for lo, hi in got]
            assert max(sizes) - min(sizes) <= SUB + n % SUB or n < world * SUB
    with pytest.raises(ValueError):
        shard_rows(10, 2, 2)


def quantised_cell_sums(x, labels, k, centre, scale, lo, hi):
    """Model of one pass's cells on rows [lo, hi): per sub-chunk of SUBCHUNK
    points (global alignment), per cluster i and dimension j the fp64 sum of
    |x - c_ij| over the members, quantised to int64 at scale 2^e_j."""
    d = x.shape[1]
    acc = np.zeros((k, d), np.int64)
    for s0 in range(lo, hi, SUBCHUNK):
        s1 = min(hi, s0 + SUBCHUNK)
        xs, ls = x[s0:s1].astype(np.float64), labels[s0:s1]
        for i in range(k):
            m = ls == i
            if not m.any():
                continue
            part = np.abs(xs[m] - centre[i]).sum(axis=0)
            acc[i] += np.rint(part * scale).astype(np.int64)
    return acc


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    data = synth.generate(5000, 7, 3, 2, seed=11)
    rng = np.random.default_rng(0)
    labels = rng.integers(0, 4, size=len(data))
    centre = rng.random((4, 7))
    scale = 2.0 ** np.array([40, 41, 39, 40, 40, 38, 42], dtype=np.float64)
    lo, hi = shard_rows(len(data), world, rank)
    part = torch.from_numpy(quantised_cell_sums(data, labels, 4, centre, scale, lo, hi))
    cnt = torch.tensor(np.bincount(labels[lo:hi], minlength=4).astype(np.int64))
    dist.all_reduce(part)  # int64 sum: exact
    dist.all_reduce(cnt)
    if rank == 0:
        q.put((part.numpy(), cnt.numpy()))
    dist.barrier()
    dist.destroy_process_group()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("world", [2])
def test_two_rank_partials_equal_single_process(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    part, cnt = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    data = synth.generate(5000, 7, 3, 2, seed=11)
    rng = np.random.default_rng(0)
    labels = rng.integers(0, 4, size=len(data))
    centre = rng.random((4, 7))
    scale = 2.0 ** np.array([40, 41, 39, 40, 40, 38, 42], dtype=np.float64)
    want = quantised_cell_sums(data, labels, 4, centre, scale, 0, len(data))
    assert np.array_equal(part, want)  # bit-identical across GPU counts
    assert np.array_equal(cnt, np.bincount(labels, minlength=4))
    # and the fixed-point totals agree with plain fp64 to ~1e-12 relative
    full = np.stack([np.abs(data[labels == i].astype(np.float64) - centre[i]).sum(0)
                     for i in range(4)])
    np.testing.assert_allclose(want / scale, full, rtol=1e-11)
