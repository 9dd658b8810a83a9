"""Test layer F: the row-sharded multi-GPU schedule with G
logical shards on ONE GPU.  Each shard is a handle with world_size = G and
its own row range; the handles share an in-process communicator
(proclus_group_create) whose fixed-order host reduction stands in for the
NCCL allreduce, and each rank runs from its own host thread.  Everything
the N > 1 path does on the device runs here: the gathers of the sample rows
by global id with row_offset, the max-reduction of max |x_j| for the
fixed-point scales, every pass without its fused tail followed by the
reduction of all NCOPY int64 accumulator copies and the replicated
single-block tails, per-shard Dist caches, speculative iteration batches.

Contract (sharding.py): with shard boundaries on the
kernels' quantisation-group multiples the result is bit-identical to one
GPU -- labels (concatenated), medoids, dimensions, iterations and cost --
and hence to the oracle."""
import threading

import numpy as np
import pytest

import synth
from parity import assert_parity

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pk():
    import torch

    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    import paper_conf_edbt_jorgensensape22_b200 as pk

    pk.lib()
    return pk


def run_group(pk, data, G, k, l, *, seed=1, metric=0, align=1024, trace=False, **kw):
    from paper_conf_edbt_jorgensensape22_b200.sharding import shard_rows

    n = data.shape[0]
    g = pk.proclus_group_create(G)
    out, err = [None] * G, [None] * G

    def work(r):
        try:
            lo, hi = shard_rows(n, G, r, align)
            with pk.Proclus(data[lo:hi], world_size=G, rank=r, n_global=n, row_offset=lo,
                            group=g, metric=metric, trace=trace) as h:
                res = h.run(k, l, seed=seed, **kw)
                out[r] = (lo, hi, res, h.trace() if trace else None)
        except Exception as e:  # noqa: BLE001 - re-raised below
            err[r] = e

    ts = [threading.Thread(target=work, args=(r,)) for r in range(G)]
    for t in ts:
        t.start()
    for t in ts:
        t.join(timeout=600)
    pk.proclus_group_destroy(g)
    for e in err:
        if e is not None:
            raise e
    assert [o[0] for o in out] == sorted(o[0] for o in out) and out[-1][1] == n
    first = out[0][2]
    for lo, hi, res, _ in out[1:]:  # replicated tails: every rank decides the same
        assert np.array_equal(res.medoids, first.medoids)
        assert np.array_equal(res.dims, first.dims)
        assert res.iterations == first.iterations and res.cost == first.cost
    labels = np.concatenate([o[2].labels for o in out])
    merged = pk.Result(labels, first.medoids, first.dims, first.cost, first.iterations)
    return merged, out[0][3]


def assert_identical(a, b, what):
    assert a.iterations == b.iterations, what
    assert np.array_equal(a.medoids, b.medoids), what
    assert np.array_equal(a.dims, b.dims), what
    assert np.array_equal(np.asarray(a.labels), np.asarray(b.labels)), what
    assert a.cost == b.cost, f"{what}: cost {a.cost!r} vs {b.cost!r}"


CASES = [
    # config, seed, world sizes, shard alignment (rows)
    ("C1", 1, (2, 3, 4), 1024),
    ("C1", 2, (8,), 64),      # 4000 rows: 8 shards of 448-512 rows (64-point groups)
    ("C2", 1, (2, 3, 8), 1024),
    ("C3", 1, (2, 8), 1024),
]


@pytest.mark.parametrize("name,seed,worlds,align", CASES)
def test_group_shards_bit_identical(pk, orc, name, seed, worlds, align):
    data, cfg = synth.config_data(name, seed=seed)
    k, l = cfg["k"], cfg["l"]
    with pk.Proclus(data, trace=True) as h:
        one = h.run(k, l, seed=seed)
        one_tr = h.trace()
    for G in worlds:
        got, tr = run_group(pk, data, G, k, l, seed=seed, align=align, trace=True)
        assert_identical(got, one, f"{name} world {G}")
        np.testing.assert_array_equal(tr.X, one_tr.X)   # fixed-point sums: exact
        np.testing.assert_array_equal(tr.nL, one_tr.nL)
    if name in ("C1", "C2"):
        o = orc.proclus(data, k, l, seed=seed, trace=True)
        assert_parity(got, o, tr, o.trace, what=f"{name} world {worlds[-1]} vs oracle")


@pytest.mark.parametrize("metric", [0, 1])
def test_group_shards_ragged_and_L1(pk, orc, metric):
    """A ragged last shard, d > 16 (k_locality<32>), L1 and L2."""
    data = synth.generate(5000, 20, 6, 4, seed=19)
    with pk.Proclus(data, metric=metric) as h:
        one = h.run(6, 4, seed=2)
    got, _ = run_group(pk, data, 3, 6, 4, seed=2, metric=metric)
    assert_identical(got, one, f"ragged metric {metric}")
    assert_parity(got, orc.proclus(data, 6, 4, seed=2, metric=metric), what="ragged vs oracle")


def test_group_rejects_mismatched_world(pk):
    data = synth.generate(3000, 6, 3, 2, seed=3)
    g = pk.proclus_group_create(2)
    try:
        with pytest.raises(pk.ProclusError):
            pk.Proclus(data[:1024], world_size=3, rank=0, n_global=3000, row_offset=0, group=g)
    finally:
        pk.proclus_group_destroy(g)
