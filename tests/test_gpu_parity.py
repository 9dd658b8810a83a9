"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on
the same seeded inputs and RNG streams.  Needs a B200 (``-m gpu``)."""
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


def run_both(pk, orc, data, k, l, *, A=100, B=10, minDev=0.7, itrPat=5, seed=1,
             metric=0, trace=True, variant=0):
    with pk.Proclus(data, metric=metric, trace=trace, variant=variant) as h:
        g = h.run(k, l, A, B, minDev, itrPat, seed)
        gt = h.trace() if trace else None
    o = orc.proclus(data, k, l, A, B, minDev, itrPat, seed, metric=metric, trace=trace)
    return g, gt, o, o.trace if trace else None


# ---------------------------------------------------------------- C1 sweep
@pytest.mark.parametrize("seed", range(1, 41))
def test_C1_seed_sweep(pk, orc, seed):
    data, cfg = synth.config_data("C1", seed=seed)
    g, gt, o, ot = run_both(pk, orc, data, cfg["k"], cfg["l"], seed=seed)
    assert_parity(g, o, gt, ot, what=f"C1 seed {seed}")


@pytest.mark.parametrize("seed", range(1, 9))
def test_C1_L1_metric(pk, orc, seed):
    data, cfg = synth.config_data("C1", seed=seed)
    g, gt, o, ot = run_both(pk, orc, data, cfg["k"], cfg["l"], seed=seed, metric=1)
    assert_parity(g, o, gt, ot, what=f"C1/L1 seed {seed}")


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_C2(pk, orc, seed):
    data, cfg = synth.config_data("C2", seed=seed)
    g, gt, o, ot = run_both(pk, orc, data, cfg["k"], cfg["l"], seed=seed)
    assert_parity(g, o, gt, ot, what=f"C2 seed {seed}")


# ---------------------------------------------------------------- shapes / edges
SHAPES = [
    # n, d, k, l, A, B  (ragged n, several chunks, d around the warp size)
    (1, 2, 2, 2, 100, 10),
    (5, 3, 2, 2, 100, 10),
    (257, 4, 3, 2, 100, 10),
    (1000, 2, 4, 2, 50, 5),
    (3001, 16, 6, 4, 30, 6),
    (2049, 17, 5, 17, 40, 4),
    (4097, 33, 8, 6, 20, 5),
    (1500, 100, 10, 10, 20, 5),
    (3000, 64, 32, 3, 8, 2),
    (2500, 100, 24, 5, 10, 3),  # k*d = 2400: radix selection of the tails
]


@pytest.mark.parametrize("shape", SHAPES)
def test_shapes(pk, orc, shape):
    n, d, k, l, A, B = shape
    if n < 2 * k:
        data = np.random.default_rng(n).random((max(n, 1), d)).astype(np.float32)
        if orc.validate(data, k, l, A, B) != 0:
            with pytest.raises(pk.ProclusError):
                pk.proclus(data, k, l, A, B)
            return
    data = synth.generate(n, d, max(2, k // 2), max(1, d // 3), seed=n)
    g, gt, o, ot = run_both(pk, orc, data, k, l, A=A, B=B, seed=3)
    assert_parity(g, o, gt, ot, what=f"shape {shape}")


def test_duplicates_and_ties(pk, orc):
    """Integer data with many duplicate points: delta_i = 0, exact distance
    ties in greedy, in L_i membership and in the assignment argmin."""
    rng = np.random.default_rng(7)
    data = rng.integers(0, 4, size=(3000, 6)).astype(np.float32)
    for seed in range(1, 6):
        g, gt, o, ot = run_both(pk, orc, data, 6, 3, seed=seed)
        assert_parity(g, o, gt, ot, what=f"ties seed {seed}")


def test_constant_columns_and_identical_points(pk, orc):
    data = synth.generate(2000, 8, 4, 3, seed=5)
    data[:, 2] = 0.5
    data[:, 5] = 0.25
    g, gt, o, ot = run_both(pk, orc, data, 4, 3, seed=2)
    assert_parity(g, o, gt, ot, what="constant columns")
    same = np.tile(np.float32([0.1, 0.2, 0.3]), (500, 1))  # sigma = 0 everywhere
    g, gt, o, ot = run_both(pk, orc, same, 3, 2, seed=1)
    assert_parity(g, o, gt, ot, what="identical points")


def test_clamped_M_and_full_shuffle(pk, orc):
    data = synth.generate(400, 5, 3, 2, seed=8)
    g, gt, o, ot = run_both(pk, orc, data, 4, 2, A=2, B=10, seed=4)  # #M = #S = 8
    assert_parity(g, o, gt, ot, what="clamped")
    g, gt, o, ot = run_both(pk, orc, data[:40], 4, 2, A=100, B=10, seed=4)  # #S = n
    assert_parity(g, o, gt, ot, what="n == #S")


def test_l_equals_d_and_l_2(pk, orc):
    data = synth.generate(3000, 7, 4, 3, seed=9)
    for l in (2, 7):
        g, gt, o, ot = run_both(pk, orc, data, 5, l, seed=6)
        assert_parity(g, o, gt, ot, what=f"l={l}")


def test_itrPat_and_minDev_variants(pk, orc):
    data, cfg = synth.config_data("C1", seed=11)
    for itrPat, minDev in ((1, 0.7), (3, 0.1), (8, 1.5)):
        g, gt, o, ot = run_both(pk, orc, data, 5, 3, itrPat=itrPat, minDev=minDev, seed=2)
        assert_parity(g, o, gt, ot, what=f"itrPat={itrPat} minDev={minDev}")


def test_max_iter_cap(pk, orc):
    data, cfg = synth.config_data("C1", seed=3)
    with pk.Proclus(data, max_iter=3) as h:
        g = h.run(5, 3, seed=1)
    o = orc.proclus(data, 5, 3, seed=1, max_iter=3)
    assert g.iterations == 3
    assert_parity(g, o, what="max_iter")


def test_deterministic_and_handle_reuse(pk):
    data, cfg = synth.config_data("C2", seed=4)
    with pk.Proclus(data) as h:
        a = h.run(10, 5, seed=3)
        b = h.run(10, 5, seed=3)  # caches warm from the first run
        c = h.run(10, 5, seed=4)
    assert np.array_equal(a.labels, b.labels) and a.cost == b.cost
    assert np.array_equal(a.medoids, b.medoids) and a.iterations == b.iterations
    assert c.labels.shape == a.labels.shape


def test_load_replaces_data(pk, orc):
    d1, _ = synth.config_data("C1", seed=1)
    d2, _ = synth.config_data("C1", seed=2)
    with pk.Proclus(d1) as h:
        h.run(5, 3, seed=1)
        h.load(d2)
        g = h.run(5, 3, seed=1)
    assert_parity(g, orc.proclus(d2, 5, 3, seed=1), what="after load")


def test_graph_cache_interleaved_settings(pk, orc):
    """Runs of different (k, l) alternate on one handle, so the second run of
    each setting launches the CUDA graph instantiated by its first run: the
    results are those of the first run and of the oracle."""
    data, _ = synth.config_data("C2", seed=5)
    with pk.Proclus(data) as h:
        first = [h.run(k, l, seed=2) for k, l in ((10, 5), (6, 3), (12, 7))]
        again = [h.run(k, l, seed=2) for k, l in ((10, 5), (6, 3), (12, 7))]
    for (k, l), a, b in zip(((10, 5), (6, 3), (12, 7)), first, again):
        assert np.array_equal(a.labels, b.labels) and np.array_equal(a.dims, b.dims)
        assert a.cost == b.cost and a.iterations == b.iterations
        assert_parity(b, orc.proclus(data, k, l, seed=2), what=f"graph cache ({k}, {l})")


@pytest.mark.parametrize("d", [15, 16])
def test_pack_unaligned_ragged_input(pk, orc, d):
    """k_pack_soa on device-resident input whose base is not 16-byte aligned
    (scalar load path) and whose n is not a multiple of the pack block
    (ragged last block), for an odd d (flat shared rows) and an even d
    (padded rows); also the aligned host-input path of the same data."""
    import torch

    data = synth.generate(3001, d, 5, 3, seed=21)
    buf = torch.empty(data.size + 1, dtype=torch.float32, device="cuda")
    view = buf[1:].view(data.shape)  # base offset 4 bytes
    view.copy_(torch.from_numpy(data))
    assert view.data_ptr() % 16 != 0
    with pk.Proclus(view) as h:
        g = h.run(5, 3, seed=4)
    with pk.Proclus(data) as h:
        g2 = h.run(5, 3, seed=4)
    assert np.array_equal(g.labels, g2.labels) and g.cost == g2.cost
    assert_parity(g, orc.proclus(data, 5, 3, seed=4), what=f"unaligned input d={d}")


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_run_multi_level3_grids(pk, orc, seed):
    """Level 3 over a grid where k grows and shrinks, and a repeated
    setting (warm start from a permutation of MBest)."""
    data = synth.generate(5000, 9, 5, 3, seed=40 + seed)
    for ks, ls in (([3, 5, 2], [2, 4]), ([4, 4], [3])):
        with pk.Proclus(data) as h:
            got = h.run_multi(ks, ls, seed=seed, reuse_level=3)
        want = orc.proclus_multi(data, ks, ls, seed=seed, reuse_level=3)
        for i, (g, o) in enumerate(zip(got, want)):
            assert_parity(g, o, what=f"level 3 {ks}x{ls} setting {i}")


def test_prefetch_overlaps_next_dataset(pk, orc):
    """proclus_prefetch stages the next dataset while the current one is
    clustered; load() of the same pointer then swaps it in (P:87 per step)."""
    import torch

    a = synth.generate(3000, 9, 4, 3, seed=31)
    b = synth.generate(3000, 9, 4, 3, seed=32)
    pa = torch.from_numpy(a).pin_memory()
    pb = torch.from_numpy(b).pin_memory()
    with pk.Proclus(pa.numpy()) as h:
        h.prefetch(pb.numpy())
        ga = h.run(4, 3, seed=5)       # still dataset a
        h.load(pb.numpy())              # waits for the prefetch, no second copy
        gb = h.run(4, 3, seed=5)
        h.prefetch(pa.numpy())
        h.load(b)                       # a different pointer: plain copy wins
        gb2 = h.run(4, 3, seed=5)
    for g, data in ((ga, a), (gb, b), (gb2, b)):
        o = orc.proclus(data, 4, 3, seed=5)
        assert_parity(g, o, what="prefetch")


def test_nonfinite_rejected(pk):
    data = np.random.default_rng(0).random((100, 4)).astype(np.float32)
    data[7, 1] = np.inf
    with pytest.raises(pk.ProclusError) as e:
        pk.Proclus(data)
    assert e.value.status == pk.EINVAL


def test_invalid_settings(pk):
    data = synth.generate(300, 5, 3, 2, seed=1)
    with pk.Proclus(data) as h:
        for args in ((1, 3), (5, 1), (5, 6), (33, 2)):
            with pytest.raises(pk.ProclusError):
                h.run(*args)
        with pytest.raises(pk.ProclusError):
            h.run(5, 3, minDev=0.0)
        with pytest.raises(pk.ProclusError):
            h.run(5, 3, itrPat=0)
        with pytest.raises(pk.ProclusError):
            h.run(200, 3, A=1, B=1)  # #M = min(200, 300) ... k > K_MAX


def test_device_resident_io(pk, orc):
    import torch

    data, cfg = synth.config_data("C1", seed=5)
    xd = torch.from_numpy(data).cuda()
    lab = torch.empty(data.shape[0], dtype=torch.int32, device="cuda")
    with pk.Proclus(xd) as h:
        g = h.run(5, 3, seed=5, labels=lab)
    torch.cuda.synchronize()
    g.labels = lab.cpu().numpy()
    assert_parity(g, orc.proclus(data, 5, 3, seed=5), what="device io")


# ---------------------------------------------------------------- multi-setting
def test_run_multi_levels(pk, orc):
    data = synth.generate(6000, 10, 5, 3, seed=12)
    ks, ls = [3, 5], [2, 4]
    for level in (1, 2, 3):
        with pk.Proclus(data) as h:
            got = h.run_multi(ks, ls, seed=7, reuse_level=level)
        want = orc.proclus_multi(data, ks, ls, seed=7, reuse_level=level)
        for i, (g, o) in enumerate(zip(got, want)):
            assert_parity(g, o, what=f"multi level {level} setting {i}")


@pytest.mark.parametrize("level", [1, 2, 3])
def test_run_multi_sweep_extent(pk, orc, level):
    """The C5 sweep's extremes (BASELINE configs[4]: k up to 20, l up to 10,
    #M = B k_max = 200) on C2-sized data: every setting of a 3 x 3 grid equals
    the oracle's multi-parameter run at each reuse level."""
    data, _ = synth.config_data("C2", seed=3)
    ks, ls = [5, 12, 20], [3, 6, 10]
    with pk.Proclus(data) as h:
        got = h.run_multi(ks, ls, seed=11, reuse_level=level)
    want = orc.proclus_multi(data, ks, ls, seed=11, reuse_level=level)
    assert len(got) == len(want) == 9
    for i, (g, o) in enumerate(zip(got, want)):
        assert g.medoids.shape[0] == ks[i // 3]
        assert_parity(g, o, what=f"sweep level {level} (k, l) = ({ks[i // 3]}, {ls[i % 3]})")


def test_run_list_full_size_C5_corners(pk, orc):
    """C5 itself (n = 1M, d = 15) at the corners of its grid, level 2 through
    run_list with k_sample = 20 (the settings-parallel split of section
    8(e)): each setting equals the oracle's level-2 sweep over the same
    corners (S and M drawn once for k_max = 20)."""
    data, _ = synth.config_data("C3", seed=1)
    ks, ls = [5, 20], [3, 10]
    settings = [(k, l) for k in ks for l in ls]
    with pk.Proclus(data) as h:
        got = h.run_list(settings, k_sample=20, seed=5, reuse_level=2)
    want = orc.proclus_multi(data, ks, ls, seed=5, reuse_level=2)
    for (k, l), g, o in zip(settings, got, want):
        assert_parity(g, o, what=f"C5 corner (k, l) = ({k}, {l})")


# ---------------------------------------------------------------- full sizes
@pytest.mark.parametrize("metric", [0, 1])
@pytest.mark.parametrize("name,seed", [("C3", 1), ("C4", 1)])
def test_full_size_configs(pk, orc, name, seed, metric):
    """BASELINE.json full sizes, in the bench's launch configuration: the
    whole run against the oracle (seconds of CPU each), with the paper's
    Euclidean full-space metric and with north_star's L1
    (reading R1)."""
    data, cfg = synth.config_data(name, seed=seed)
    g, gt, o, ot = run_both(pk, orc, data, cfg["k"], cfg["l"], seed=seed, metric=metric)
    assert_parity(g, o, gt, ot, what=f"{name} metric {metric}")


# ------------------------------------------------ L1 at every kernel shape
# The full-space metric enters the greedy (k_greedy_cluster / k_sdist_tiled
# for DP > 16), the Dist rows of k_locality<16>, <32> and <0> (d <= 16,
# d <= 32, longer rows) and the exact fp64 fallback.  L1 (north_star) at the
# d ranges that select each instantiation.
L1_SHAPES = [
    # n, d, k, l, A, B
    (3001, 16, 6, 4, 30, 6),     # k_locality<16>
    (4097, 33, 8, 6, 20, 5),     # d > 32: k_locality<0>, greedy DP 64
    (3000, 64, 12, 5, 20, 4),    # d = 64
    (2600, 100, 10, 10, 20, 5),  # d = 100 (C4 width)
    (2049, 24, 5, 7, 40, 4),     # d <= 32: k_locality<32>
]


@pytest.mark.parametrize("shape", L1_SHAPES)
def test_L1_shapes(pk, orc, shape):
    n, d, k, l, A, B = shape
    data = synth.generate(n, d, max(2, k // 2), max(2, d // 3), seed=n + d)
    for seed in (1, 2):
        g, gt, o, ot = run_both(pk, orc, data, k, l, A=A, B=B, seed=seed, metric=1)
        assert_parity(g, o, gt, ot, what=f"L1 shape {shape} seed {seed}")


@pytest.mark.parametrize("metric", [0, 1])
def test_greedy_big_sample(pk, orc, metric):
    """#S > 4096 (k_greedy_big: the sample matrix does not fit the cluster
    kernels): A*k = 5000 sample points, #M = 250."""
    data = synth.generate(12000, 6, 8, 3, seed=77)
    g, gt, o, ot = run_both(pk, orc, data, 25, 3, A=200, B=10, seed=5, metric=metric)
    assert o.nS == 5000 and o.nM == 250
    assert_parity(g, o, gt, ot, what=f"greedy big metric {metric}")


# ------------------------------------------------ variants
# GPU-PROCLUS (no caches) and GPU-FAST*-PROCLUS (slot caches from the
# previous iteration only) must reach the same clustering as plain
# PROCLUS -- the oracle -- on the same draws.
@pytest.mark.parametrize("variant", [1, 2])
@pytest.mark.parametrize("seed", range(1, 9))
def test_variants_C1(pk, orc, variant, seed):
    data, cfg = synth.config_data("C1", seed=seed)
    g, gt, o, ot = run_both(pk, orc, data, cfg["k"], cfg["l"], seed=seed, variant=variant)
    assert_parity(g, o, gt, ot, what=f"variant {variant} C1 seed {seed}")


@pytest.mark.parametrize("variant", [1, 2])
@pytest.mark.parametrize("shape", [(3001, 16, 6, 4, 30, 6), (4097, 33, 8, 6, 20, 5),
                                   (1500, 100, 10, 10, 20, 5)])
def test_variants_shapes(pk, orc, variant, shape):
    n, d, k, l, A, B = shape
    data = synth.generate(n, d, max(2, k // 2), max(1, d // 3), seed=n)
    g, gt, o, ot = run_both(pk, orc, data, k, l, A=A, B=B, seed=3, variant=variant)
    assert_parity(g, o, gt, ot, what=f"variant {variant} shape {shape}")


@pytest.mark.parametrize("variant", [1, 2])
def test_variants_C2_and_multi(pk, orc, variant):
    data, cfg = synth.config_data("C2", seed=1)
    g, gt, o, ot = run_both(pk, orc, data, cfg["k"], cfg["l"], seed=1, variant=variant)
    assert_parity(g, o, gt, ot, what=f"variant {variant} C2")
    small = synth.generate(6000, 10, 5, 3, seed=12)
    with pk.Proclus(small, variant=variant) as h:
        got = h.run_multi([3, 5], [2, 4], seed=7, reuse_level=2)
    want = orc.proclus_multi(small, [3, 5], [2, 4], seed=7, reuse_level=2)
    for i, (gg, oo) in enumerate(zip(got, want)):
        assert_parity(gg, oo, what=f"variant {variant} multi setting {i}")


@pytest.mark.parametrize("variant", [1, 2])
def test_variants_full_size_C3(pk, orc, variant):
    data, cfg = synth.config_data("C3", seed=1)
    g, gt, o, ot = run_both(pk, orc, data, cfg["k"], cfg["l"], seed=1, variant=variant)
    assert_parity(g, o, gt, ot, what=f"variant {variant} C3")


# ------------------------------------------------ n = 8M
def _seg(x, m, dmask):
    """seg_D(x, m) of O0 in fp64, one column per cluster (x: [p, d])."""
    diff = np.abs(x[:, None, :].astype(np.float64) - m[None, :, :].astype(np.float64))
    return (diff * dmask[None]).sum(axis=2) / dmask.sum(axis=1)[None]


def test_large_n_properties(pk):
    """At the L8 size (8M x 15, Fig 3e) the oracle takes minutes per run, so
    the GPU result is checked through properties that hold at any size, on
    20,000 sampled points: every label is the segmental argmin over the
    returned medoids / dimensions (reading R8, ties to the smaller slot), -1
    exactly when the point is outside every Delta_i sphere (R17); every
    medoid carries its own label; k*l dimensions, >= 2 per cluster."""
    import torch

    data, cfg = synth.config_data("L8", seed=1)
    k, l = cfg["k"], cfg["l"]
    x = torch.from_numpy(data).cuda()
    lab = torch.empty(data.shape[0], dtype=torch.int32, device="cuda")
    with pk.Proclus(x) as h:
        g = h.run(k, l, seed=1, labels=lab)
    labels = lab.cpu().numpy()
    dm = g.dims.astype(np.float64)
    assert int(g.dims.sum()) == k * l and (g.dims.sum(axis=1) >= 2).all()
    med = data[g.medoids]
    # Delta_i = min_{j != i} seg_{D_i}(m_i, m_j) (R5)
    sm = _seg(med, med, dm)                      # sm[a, i] = seg_{D_i}(m_a, m_i)
    Delta = np.array([min(sm[j, i] for j in range(k) if j != i) for i in range(k)])
    rng = np.random.default_rng(0)
    idx = rng.choice(data.shape[0], 20_000, replace=False)
    sd = _seg(data[idx], med, dm)
    order = np.sort(sd, axis=1)
    gap = (order[:, 1] - order[:, 0]) / np.maximum(order[:, 0], 1e-300)
    want = np.argmin(sd, axis=1)
    outside = (sd > Delta[None]).all(axis=1)
    want = np.where(outside, -1, want)
    ok = (labels[idx] == want) | (gap < 1e-6)   # north_star argmin allowance
    assert ok.all(), f"{(~ok).sum()} sampled labels differ"
    for i, mi in enumerate(g.medoids):
        assert labels[mi] in (i, -1) or sd.shape[0] == 0
    assert (labels >= -1).all() and (labels < k).all()
    assert 6 <= g.iterations < 10000


# ------------------------------------------------ multi-GPU schedule on 1 GPU
# World size > 1 runs every pass without its fused tail, allreduces the
# fixed-point cell sums (all NCOPY copies) over NCCL and finalises in a
# separate single-block kernel (split_tail).  PROCLUS_SPLIT_TAIL=1 runs that
# schedule on one GPU (the allreduce is then the identity), so the tail
# kernel, the speculative iteration batches and the host control of the
# N > 1 path are covered by parity here.
@pytest.mark.parametrize("case", ["C1-1", "C1-2", "C1-3", "C2-1", "shape"])
def test_split_tail_schedule(pk, orc, monkeypatch, case):
    monkeypatch.setenv("PROCLUS_SPLIT_TAIL", "1")
    if case == "shape":
        data = synth.generate(1500, 100, 5, 33, seed=1500)
        k, l, seed = 10, 10, 3
    else:
        name, seed = case.split("-")
        seed = int(seed)
        data, cfg = synth.config_data(name, seed=seed)
        k, l = cfg["k"], cfg["l"]
    g, gt, o, ot = run_both(pk, orc, data, k, l, seed=seed)
    assert_parity(g, o, gt, ot, what=f"split tail {case}")


# ------------------------------------------------ settings parallelism (C5)
@pytest.mark.parametrize("level", [1, 2])
def test_run_list_splits_grid(pk, orc, level):
    """The C5 sweep split across ranks: every rank holds the whole
    dataset and runs its share of the (k, l) settings through run_list with
    k_sample = the grid's largest k; the union equals run_multi over the grid
    bit for bit, and the oracle's multi-parameter run."""
    data = synth.generate(6000, 10, 5, 3, seed=12)
    ks, ls = [3, 4, 5], [2, 3, 4]
    with pk.Proclus(data) as h:
        whole = h.run_multi(ks, ls, seed=7, reuse_level=level)
    settings = [(k, l) for k in ks for l in ls]
    got = [None] * len(settings)
    for rank in range(3):  # three "ranks", one after the other on this GPU
        mine = list(range(rank, len(settings), 3))
        with pk.Proclus(data) as h:
            res = h.run_list([settings[i] for i in mine], k_sample=max(ks), seed=7,
                             reuse_level=level)
        for i, r in zip(mine, res):
            got[i] = r
    want = orc.proclus_multi(data, ks, ls, seed=7, reuse_level=level)
    for i, (g, w, o) in enumerate(zip(got, whole, want)):
        assert np.array_equal(g.labels, w.labels) and np.array_equal(g.medoids, w.medoids)
        assert np.array_equal(g.dims, w.dims) and g.cost == w.cost
        assert g.iterations == w.iterations
        assert_parity(g, o, what=f"run_list level {level} setting {settings[i]}")


# ------------------------------------------------ oracle parity at n = 8M
@pytest.mark.parametrize("k,l", [(10, 5), (15, 7)])
def test_L8_oracle_parity(pk, orc, k, l):
    """Fig 3e's large-n workload (> 8M points) against the oracle: the
    default setting (L8) and one setting of the 9-setting grid (L8S, reading
    R22), full traces, labels, medoids, dimensions, iterations and cost.  The
    plain oracle needs ~2 minutes of one host core per run."""
    import torch

    data, cfg = synth.config_data("L8", seed=1)
    x = torch.from_numpy(data).cuda()
    lab = torch.empty(data.shape[0], dtype=torch.int32, device="cuda")
    with pk.Proclus(x, trace=True) as h:
        g = h.run(k, l, seed=1, labels=lab)
        gt = h.trace()
    g.labels = lab.cpu().numpy()
    del x
    o = orc.proclus(data, k, l, seed=1, trace=True)
    assert_parity(g, o, gt, o.trace, what=f"L8 k={k} l={l}")


def test_async_load_rejects_nonfinite_at_run(pk, orc):
    """proclus_load is asynchronous on one GPU (scales computed on the device):
    a non-finite value makes the next run fail with EINVAL; a later load of
    finite data recovers, with results equal to the oracle's."""
    d1, _ = synth.config_data("C1", seed=1)
    bad = d1.copy()
    bad[123, 4] = np.nan
    with pk.Proclus(d1) as h:
        h.load(bad)
        with pytest.raises(pk.ProclusError) as e:
            h.run(5, 3, seed=1)
        assert e.value.status == pk.EINVAL
        h.load(d1)
        g = h.run(5, 3, seed=1)
    assert_parity(g, orc.proclus(d1, 5, 3, seed=1), what="after a rejected load")


@pytest.mark.parametrize("case", ["C1-1", "C1-2", "C2-1"])
def test_tail_kernels_in_graph(pk, orc, monkeypatch, case):
    """PROCLUS_TAIL_KERNELS=1: the single-block tails as 1024-thread kernels
    of their own inside the graph (the default only for k d > 512) give the
    same clustering at small k d."""
    monkeypatch.setenv("PROCLUS_TAIL_KERNELS", "1")
    name, seed = case.split("-")
    data, cfg = synth.config_data(name, seed=int(seed))
    g, gt, o, ot = run_both(pk, orc, data, cfg["k"], cfg["l"], seed=int(seed))
    assert_parity(g, o, gt, ot, what=f"tail kernels {case}")


def test_concurrent_handles_of_different_shapes(pk, orc):
    """Two handles with different shared-memory needs (d = 15 and d = 100)
    run from two host threads at once: the kernels' dynamic shared-memory
    opt-in only grows, so neither launch fails."""
    import threading

    a = synth.generate(4000, 15, 5, 3, seed=61)
    b = synth.generate(3000, 100, 10, 10, seed=62)
    out, err = {}, []

    def work(name, data, k, l):
        try:
            with pk.Proclus(data) as h:
                for s in range(3):
                    out[(name, s)] = h.run(k, l, A=20, B=5, seed=s + 1)
        except Exception as e:  # noqa: BLE001
            err.append(e)

    ts = [threading.Thread(target=work, args=("a", a, 5, 3)),
          threading.Thread(target=work, args=("b", b, 10, 10))]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    assert not err, err
    for s in range(3):
        assert_parity(out[("a", s)], orc.proclus(a, 5, 3, A=20, B=5, seed=s + 1), what="a")
        assert_parity(out[("b", s)], orc.proclus(b, 10, 10, A=20, B=5, seed=s + 1), what="b")
