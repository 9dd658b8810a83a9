"""Pins of the CPU oracle against things other than itself (CPU only).

Each test names the PAPER.md passage (P:<line>) it checks and what pins it:
a worked example (tests/golden), a closed form, a library routine for a
special case, an invariant, or brute force on tiny inputs.  A plausible bug
in the oracle (dropped term, wrong sign/index, transposed operand, wrong tie
rule, wrong denominator) fails at least one of them.
"""
import itertools
import json
import os

import numpy as np
import pytest
from scipy.spatial.distance import cdist

import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ------------------------------------------------------------------ RNG
def test_splitmix_known_answers(orc):
    """Reading R2: SplitMix64 published test vectors."""
    for v in gold("splitmix64.json")["vectors"]:
        s = v["seed"]
        for want in v["outputs"]:
            got, s = orc.splitmix_next(s)
            assert got == int(want, 16)


def test_uniform_range_and_chi2(orc):
    """uniform(m) in [0,m) and flat (chi-square, 10 bins, 20k draws)."""
    s = 12345
    m = 10
    counts = np.zeros(m)
    for _ in range(20000):
        v, s = orc.uniform(s, m)
        assert 0 <= v < m
        counts[v] += 1
    chi2 = ((counts - 2000) ** 2 / 2000).sum()
    assert chi2 < 30.0  # 9 dof, p ~ 4e-4


def test_streams_keyed(orc):
    """SM depends on (seed,k) only; IT on (seed,k,l) (multi-param reuse)."""
    assert orc.stream_sm(7, 10) == orc.stream_sm(7, 10)
    assert orc.stream_sm(7, 10) != orc.stream_sm(7, 11)
    assert orc.stream_sm(7, 10) != orc.stream_sm(8, 10)
    assert orc.stream_it(7, 10, 5) != orc.stream_it(7, 10, 6)
    assert orc.stream_it(7, 10, 5) != orc.stream_sm(7, 10)


# ------------------------------------------------------------------ sample
def test_sample_without_replacement(orc):
    """Alg 1 l.2, reading R13: a sample without replacement."""
    S, _ = orc.sample(1000, 500, 99)
    assert len(set(S.tolist())) == 500 and S.min() >= 0 and S.max() < 1000
    P, _ = orc.sample(50, 50, 3)
    assert sorted(P.tolist()) == list(range(50))


def test_sample_first_element_uniform(orc):
    counts = np.zeros(8)
    for seed in range(4000):
        S, _ = orc.sample(8, 3, orc.stream_sm(seed, 3))
        counts[S[0]] += 1
    chi2 = ((counts - 500) ** 2 / 500).sum()
    assert chi2 < 25.0  # 7 dof


# ------------------------------------------------------------------ distances
def test_full_and_seg_vs_scipy(orc):
    """O0 distances against scipy on integer data (exact)."""
    rng = np.random.default_rng(0)
    a = rng.integers(-5, 6, size=(20, 7)).astype(np.float32)
    E = cdist(a, a, "euclidean")
    M = cdist(a, a, "cityblock")
    for i in range(20):
        for j in range(20):
            assert orc.full(a[i], a[j], orc.METRIC_L2) == E[i, j]
            assert orc.full(a[i], a[j], orc.METRIC_L1) == M[i, j]
    mask = np.array([1, 0, 1, 1, 0, 0, 1], bool)
    for i in range(5):
        want = np.abs(a[i] - a[i + 1])[mask].sum() / mask.sum()
        assert orc.seg(a[i], a[i + 1], mask) == want


# ------------------------------------------------------------------ greedy
def test_greedy_worked_example(orc):
    g = gold("greedy_collinear.json")
    data = np.array(g["points"], np.float32)[:, None]
    pos, pd = orc.greedy(data, np.arange(len(data)), g["nM"], g["q0"])
    assert pos.tolist() == g["picks"]
    assert pd[1:].tolist() == g["pickdist"][1:]


def _greedy_brute(pts, q0, nM):
    """Literal Alg 2: each pick recomputes min over picked from scratch."""
    D = cdist(pts, pts)
    picked = [q0]
    while len(picked) < nM:
        best, bestd = None, -1.0
        for q in range(len(pts)):
            if q in picked:
                continue
            md = min(D[q, m] for m in picked)
            if md > bestd:
                best, bestd = q, md
        picked.append(best)
    return picked


@pytest.mark.parametrize("seed", range(12))
def test_greedy_brute_force(orc, seed):
    """Alg 2 vs a from-scratch farthest-first on tiny integer inputs with ties."""
    rng = np.random.default_rng(seed)
    nS, d = int(rng.integers(2, 13)), int(rng.integers(1, 4))
    pts = rng.integers(0, 4, size=(nS, d)).astype(np.float32)
    nM = int(rng.integers(1, nS + 1))
    q0 = int(rng.integers(0, nS))
    pos, pd = orc.greedy(pts, np.arange(nS), nM, q0)
    assert pos.tolist() == _greedy_brute(pts.astype(np.float64), q0, nM)
    assert np.all(np.diff(pd[1:]) <= 0)  # max-min distances never increase
    assert len(set(pos.tolist())) == nM


def test_greedy_prefix_property(orc):
    rng = np.random.default_rng(5)
    pts = rng.random((300, 6)).astype(np.float32)
    S = rng.permutation(300)[:200]
    a, _ = orc.greedy(pts, S, 20, 7)
    b, _ = orc.greedy(pts, S, 60, 7)
    assert a.tolist() == b[:20].tolist()


# ------------------------------------------------------------------ ComputeL
def test_delta_and_L_brute(orc):
    """Alg 3, readings R6, R9, against scipy on integer data."""
    rng = np.random.default_rng(1)
    data = rng.integers(0, 6, size=(300, 4)).astype(np.float32)
    med = data[[3, 50, 99, 120]]
    for metric, name in ((orc.METRIC_L2, "euclidean"), (orc.METRIC_L1, "cityblock")):
        dl = orc.delta(med, metric)
        MM = cdist(med, med, name)
        np.fill_diagonal(MM, np.inf)
        assert np.array_equal(dl, MM.min(1))
        inL, nL, X = orc.locality_X(data, med, dl, metric)
        PD = cdist(data, med, name)
        assert np.array_equal(inL, PD <= dl[None, :])
        assert np.array_equal(nL, inL.sum(0))
        for i in range(4):
            want = np.abs(data[inL[:, i]].astype(np.float64) - med[i]).mean(0)
            np.testing.assert_allclose(X[i], want, rtol=1e-13, atol=0)
        # m_i is in L_i, and so is its nearest other medoid (delta is attained)
        for i, r in enumerate([3, 50, 99, 120]):
            assert inL[r, i]
            j = int(np.argmin(MM[i]))
            assert inL[[3, 50, 99, 120][j], i]


# ------------------------------------------------------------------ FindDimensions
def test_zscore_worked_example(orc):
    g = gold("zscore_select.json")
    X = np.array(g["X"], np.float64)
    m, Z, _ = orc.find_dimensions(X, g["l"])
    for i, D in enumerate(g["D"]):
        assert np.flatnonzero(m[i]).tolist() == D
    Y = np.array(g["Y"])
    sg = np.array(g["sigma"])
    np.testing.assert_allclose(Z, (X - Y[:, None]) / sg[:, None], rtol=1e-15)


@pytest.mark.parametrize("seed", range(6))
def test_zscore_numpy_and_closed_forms(orc, seed):
    """Y = mean, sigma = numpy std(ddof=1) (reading R2); sum_j Z = 0, sum_j Z^2 = d-1."""
    rng = np.random.default_rng(seed)
    k, d = 7, int(rng.integers(3, 40))
    X = rng.random((k, d)) * 10
    _, Z, _ = orc.find_dimensions(X, 2)
    want = (X - X.mean(1, keepdims=True)) / X.std(1, ddof=1, keepdims=True)
    np.testing.assert_allclose(Z, want, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(Z.sum(1), 0, atol=1e-12)
    np.testing.assert_allclose((Z ** 2).sum(1), d - 1, rtol=1e-12)


def _select_brute(Z, l):
    """Enumerate every D with >= 2 dims per row and k*l in total; pick the
    minimum sum of Z (the greedy of Alg 4 l.15-16 is optimal by exchange)."""
    k, d = Z.shape
    cells = [(i, j) for i in range(k) for j in range(d)]
    best, bestset = np.inf, None
    for comb in itertools.combinations(range(k * d), k * l):
        rows = np.bincount([cells[c][0] for c in comb], minlength=k)
        if rows.min() < 2:
            continue
        s = sum(Z[cells[c]] for c in comb)
        if s < best - 1e-12:
            best, bestset = s, comb
    m = np.zeros((k, d), bool)
    for c in bestset:
        m[cells[c]] = True
    return m


@pytest.mark.parametrize("seed", range(20))
def test_selection_brute_force(orc, seed):
    rng = np.random.default_rng(100 + seed)
    k, d = int(rng.integers(2, 4)), int(rng.integers(2, 6))
    if k * d > 12:
        d = 12 // k
    l = int(rng.integers(2, d + 1))
    X = rng.random((k, d))
    m, Z, _ = orc.find_dimensions(X, l)
    assert m.sum() == k * l and m.sum(1).min() >= 2
    assert np.array_equal(m, _select_brute(Z, l))


def test_selection_special_cases(orc):
    X = np.random.default_rng(3).random((4, 6))
    m, _, _ = orc.find_dimensions(X, 6)  # l = d -> every dimension
    assert m.all()
    # sigma = 0 -> Z = 0: per row the keys (0, j) pick j = 0, 1; the 9 - 6 = 3
    # remaining picks follow (0, i, j) and all go to row 0 (j = 2, 3, 4)
    X0 = np.ones((3, 5))
    m, Z, _ = orc.find_dimensions(X0, 3)
    assert (Z == 0).all()
    assert m.astype(int).tolist() == [[1, 1, 1, 1, 1], [1, 1, 0, 0, 0], [1, 1, 0, 0, 0]]


# ------------------------------------------------------------------ AssignPoints
def test_assign_worked_example(orc):
    g = gold("assign_ties.json")
    med = np.array(g["medoids"], np.float32)
    for case in g["cases"]:
        lab, _ = orc.assign(np.array(case["points"], np.float32), med, np.array(case["dims"]))
        assert lab.tolist() == case["labels"]


@pytest.mark.parametrize("seed", range(5))
def test_assign_brute_and_kmedoids_special_case(orc, seed):
    rng = np.random.default_rng(seed)
    n, d, k = 400, 6, 5
    data = rng.integers(0, 5, size=(n, d)).astype(np.float32)
    med = data[rng.choice(n, k, replace=False)]
    mask = rng.random((k, d)) < 0.5
    mask[:, :2] = True
    lab, _ = orc.assign(data, med, mask)
    seg = np.stack([np.abs(data - med[i])[:, mask[i]].sum(1) / mask[i].sum() for i in range(k)], 1)
    assert np.array_equal(lab, np.argmin(seg, 1))  # argmin returns the first minimum
    # l = d: plain L1 nearest medoid (k-medoids assignment) via scipy
    lab2, _ = orc.assign(data, med, np.ones((k, d), bool))
    assert np.array_equal(lab2, np.argmin(cdist(data, med, "cityblock"), 1))


# ------------------------------------------------------------------ EvaluateCluster
def test_cost_worked_example(orc):
    g = gold("cost_eval.json")
    c, sizes = orc.evaluate(np.array(g["data"], np.float32), g["labels"], 2, np.array(g["dims"]))
    assert c == g["cost"] and sizes.tolist() == g["sizes"]
    assert orc.evaluate_eq9(np.array(g["data"], np.float32), g["labels"], 2,
                            np.array(g["dims"])) == g["cost"]


@pytest.mark.parametrize("seed", range(5))
def test_cost_eq2_equals_eq9_and_invariants(orc, seed):
    rng = np.random.default_rng(seed)
    n, d, k = 500, 8, 4
    data = rng.random((n, d)).astype(np.float32)
    lab = rng.integers(0, k, n).astype(np.int32)
    mask = rng.random((k, d)) < 0.6
    mask[:, :2] = True
    c, sizes = orc.evaluate(data, lab, k, mask)
    np.testing.assert_allclose(c, orc.evaluate_eq9(data, lab, k, mask), rtol=1e-13)
    assert sizes.tolist() == np.bincount(lab, minlength=k).tolist()
    # numpy restatement of eq 1-2 with numpy's own mean
    want = 0.0
    for i in range(k):
        x = data[lab == i].astype(np.float64)[:, mask[i]]
        want += len(x) * np.abs(x - x.mean(0)).mean(0).mean()
    np.testing.assert_allclose(c, want / n, rtol=1e-12)
    # invariant under relabelling the clusters
    perm = rng.permutation(k)
    c2, _ = orc.evaluate(data, perm[lab].astype(np.int32), k, mask[np.argsort(perm)])
    np.testing.assert_allclose(c2, c, rtol=1e-13)
    # cost = 0 iff every cluster is constant on its dimensions
    const = np.repeat(rng.random((k, d)), 3, axis=0).astype(np.float32)
    lab3 = np.repeat(np.arange(k), 3).astype(np.int32)
    assert orc.evaluate(const, lab3, k, mask)[0] == 0.0


def test_cost_empty_cluster(orc):
    data = np.random.default_rng(0).random((10, 3)).astype(np.float32)
    lab = np.zeros(10, np.int32)
    m = np.ones((2, 3), bool)
    c, sizes = orc.evaluate(data, lab, 2, m)
    assert sizes.tolist() == [10, 0] and np.isfinite(c)


# ------------------------------------------------------------------ bad medoids
def test_bad_medoids_golden(orc):
    for case in gold("bad_medoids.json")["cases"]:
        got = orc.bad_medoids(case["sizes"], case["n"], case["minDev"])
        assert got.tolist() == case["bad"], case["note"]


# ------------------------------------------------------------------ refinement
def test_refinement_pieces(orc):
    rng = np.random.default_rng(2)
    data = rng.integers(0, 5, size=(200, 5)).astype(np.float32)
    med = data[[0, 1, 2]]
    lab = rng.integers(0, 3, 200).astype(np.int32)
    X = orc.cluster_X(data, lab, med)
    for i in range(3):
        np.testing.assert_allclose(
            X[i], np.abs(data[lab == i].astype(np.float64) - med[i]).mean(0), rtol=1e-13)
    mask = np.ones((3, 5), bool)
    mask[:, 4] = False
    out, Dl = orc.remove_outliers(data, med, mask, lab)
    seg = np.stack([np.abs(data - med[i])[:, mask[i]].sum(1) / 4 for i in range(3)], 1)
    MM = np.stack([np.abs(med - med[i])[:, mask[i]].sum(1) / 4 for i in range(3)], 0)
    np.fill_diagonal(MM, np.inf)
    assert np.array_equal(Dl, MM.min(1))
    outl = (seg > Dl[None, :]).all(1)
    assert np.array_equal(out == -1, outl)
    assert np.array_equal(out[~outl], lab[~outl])


# ------------------------------------------------------------------ whole run
def _check_run_invariants(orc, data, r, k, l, itrPat, n):
    t = r.trace
    d = data.shape[1]
    assert r.dims.sum() == k * l and r.dims.sum(1).min() >= 2
    assert r.labels.min() >= -1 and r.labels.max() < k
    assert len(set(r.medoids.tolist())) == k
    for it in range(len(t.cost)):
        assert t.dims[it].sum() == k * l and t.dims[it].sum(1).min() >= 2
        assert t.sizes[it].sum() == n
    # costBest is the minimum over iterations and improvements are strict
    best = np.inf
    for it, c in enumerate(t.cost):
        assert t.improved[it] == (c < best)
        best = min(best, c)
    assert r.cost == best
    # stop rule (Alg 1 l.5): exactly itrPat non-improving iterations at the end
    assert r.iterations >= itrPat + 1
    assert not t.improved[-itrPat:].any() and t.improved[-itrPat - 1]
    # replacement (Alg 1 l.14): MCur(t+1) = MBest(t) except at bad slots, new
    # medoids come from M \ MBest
    mbest = None
    for it in range(len(t.cost) - 1):
        if t.improved[it]:
            mbest = t.mcur[it]
        nxt = t.mcur[it + 1]
        same = nxt == mbest
        assert np.all(same | t.bad[it])
        for i in np.flatnonzero(~same):
            assert nxt[i] not in mbest
        assert len(set(nxt.tolist())) == k
    return d


def _replay_loop_control(orc, r, n, k, l, minDev, seed):
    """Replay Alg 1 l.4 and l.10-14 from the trace's cost
    and cluster sizes alone, with the spec's draws (stream IT, reading R2):
    the initial MCur (partial Fisher-Yates over [0, #M)), improved = cost <
    costBest (strict, R14), MBest / sizesBest = MCur / sizes of the last
    improved iteration, MBad from the sizes of CBest -- the best clustering,
    Alg 1 l.13 and P:91, reading R11 (not the current iteration's
    sizes, as Table 1's 'MBad subset of MCur' could be read) -- with
    thr = n/k*minDev (bad_medoids is pinned by its golden cases), and the
    replacement of Alg 1 l.14 from M \\ MBest in ascending bad-slot order
    (R12).  Checks every recorded MCur, improved and MBad against it."""
    t = r.trace
    st = orc.stream_it(seed, k, l)
    pool = list(range(r.nM))
    for i in range(k):                       # O5: MCur
        v, st = orc.uniform(st, r.nM - i)
        j = i + v
        pool[i], pool[j] = pool[j], pool[i]
    mcur = np.array(pool[:k])
    best = np.inf
    mbest = sizes_best = None
    for it in range(len(t.cost)):
        assert np.array_equal(t.mcur[it], mcur), f"MCur at iteration {it}"
        improved = t.cost[it] < best
        assert bool(t.improved[it]) == improved, f"improved at iteration {it}"
        if improved:
            best = t.cost[it]
            mbest = mcur.copy()
            sizes_best = t.sizes[it].copy()
        bad = orc.bad_medoids(sizes_best, n, minDev)
        assert np.array_equal(t.bad[it], bad), f"MBad at iteration {it} (from sizesBest)"
        pool = [q for q in range(r.nM) if q not in set(mbest.tolist())]
        mcur = mbest.copy()
        for i in np.flatnonzero(bad):
            if not pool:
                break
            v, st = orc.uniform(st, len(pool))
            mcur[i] = pool.pop(v)
    return mbest


def _init_M(orc, data, r, k, A, B, seed, metric):
    """Point ids of M from the pinned pieces (O2-O4): stream SM, the sample
    S (Alg 1 l.2), the greedy start q0 and Greedy (Alg 2)."""
    n = data.shape[0]
    nS = min(A * k, n)
    st = orc.stream_sm(seed, k)
    S, st = orc.sample(n, nS, st)
    q0, st = orc.uniform(st, nS)
    pos, _ = orc.greedy(data, S, min(B * k, nS), q0, metric)
    return S[pos]


def _check_refinement(orc, data, r, k, l, A, B, seed, metric, mbest):
    """Alg 1 l.15-19 composed from the pinned pieces: the
    output medoids are MBest (R16) as point ids; CBest = the assignment of the
    last improved iteration (its MCur and D); refinement X over CBest
    with MBest ('computing the dimensions using the clusters CBest'),
    FindDimensions, the final assignment and RemoveOutliers (R17)."""
    t = r.trace
    last = int(np.flatnonzero(t.improved)[-1])
    Mid = _init_M(orc, data, r, k, A, B, seed, metric)
    assert np.array_equal(r.medoids, Mid[mbest]), "medoids = MBest"
    med = data[r.medoids]
    cbest, _ = orc.assign(data, med, t.dims[last])
    assert np.array_equal(np.bincount(cbest, minlength=k), t.sizes[last])
    X = orc.cluster_X(data, cbest, med)
    dstar, _, _ = orc.find_dimensions(X, l)
    assert np.array_equal(r.dims, dstar), "refined dimensions from CBest / MBest"
    lab, _ = orc.assign(data, med, dstar)
    lab, _ = orc.remove_outliers(data, med, dstar, lab)
    assert np.array_equal(r.labels, lab), "final labels"


@pytest.mark.parametrize("seed", range(1, 9))
def test_run_invariants_C1(orc, seed):
    data, cfg = synth.config_data("C1", seed=seed)
    r = orc.proclus(data, cfg["k"], cfg["l"], seed=seed, trace=True)
    _check_run_invariants(orc, data, r, cfg["k"], cfg["l"], 5, cfg["n"])


@pytest.mark.parametrize("metric", [0, 1])
@pytest.mark.parametrize("seed", range(1, 7))
def test_loop_control_and_refinement_composed(orc, seed, metric):
    """The whole run's loop decisions and refinement, recomputed from the
    pinned pieces (MBad from CBest's sizes, refinement over CBest / MBest).
    minDev = 1.0 makes MBad non-trivial (several bad slots per iteration)."""
    data, cfg = synth.config_data("C1", seed=seed)
    k, l = cfg["k"], cfg["l"]
    for minDev in (0.7, 1.0):
        r = orc.proclus(data, k, l, minDev=minDev, seed=seed, metric=metric, trace=True)
        mbest = _replay_loop_control(orc, r, cfg["n"], k, l, minDev, seed)
        _check_refinement(orc, data, r, k, l, 100, 10, seed, metric, mbest)


def test_loop_control_on_generator_shapes(orc):
    """Same pins at other shapes (d > 16, k > 8, a small #M pool)."""
    for (n, d, k, l, A, B, s) in ((3000, 20, 9, 4, 30, 4, 1), (2500, 9, 4, 3, 5, 2, 2)):
        data = synth.generate(n, d, max(2, k // 2), max(2, d // 4), seed=s)
        r = orc.proclus(data, k, l, A, B, minDev=0.9, seed=s, trace=True)
        mbest = _replay_loop_control(orc, r, n, k, l, 0.9, s)
        _check_refinement(orc, data, r, k, l, A, B, s, 0, mbest)


@pytest.mark.parametrize("metric", [0, 1])
@pytest.mark.parametrize("seed", range(1, 6))
def test_fast_equals_plain(orc, seed, metric):
    """Theorems 3.1 / 3.2 and P:390: FAST-PROCLUS (Dist cache,
    Delta L bands, incremental H) reaches the same clustering as PROCLUS."""
    data = synth.generate(3000, 12, 6, 4, seed=seed)
    a = orc.proclus(data, 6, 4, seed=seed, metric=metric, trace=True)
    b = orc.proclus(data, 6, 4, seed=seed, metric=metric, fast=True, trace=True)
    assert np.array_equal(a.labels, b.labels) and np.array_equal(a.dims, b.dims)
    assert np.array_equal(a.medoids, b.medoids) and a.iterations == b.iterations
    assert np.array_equal(a.trace.nL, b.trace.nL)
    assert np.array_equal(a.trace.mcur, b.trace.mcur)
    np.testing.assert_allclose(a.trace.X, b.trace.X, rtol=1e-12, atol=1e-15)
    assert a.cost == b.cost


def test_planted_subspaces_recovered(orc):
    """Sanity, not parity: with well-separated planted clusters the selected
    dimensions of most clusters are the planted ones."""
    rng = np.random.default_rng(11)
    n, d, k, s = 4000, 10, 4, 3
    data = rng.random((n, d))
    truth = []
    for c in range(k):
        dims = np.sort(rng.permutation(d)[:s])
        truth.append(set(dims.tolist()))
        idx = np.arange(c * n // k, (c + 1) * n // k)
        data[np.ix_(idx, dims)] = rng.random(s) + 0.005 * rng.standard_normal((len(idx), s))
    r = orc.proclus(data.astype(np.float32), k, s, seed=3)
    hits = 0
    for i in range(k):
        got = set(np.flatnonzero(r.dims[i]).tolist())
        hits += any(got == t for t in truth)
    assert hits >= k - 1


def test_validation(orc):
    data = np.random.default_rng(0).random((100, 5)).astype(np.float32)
    assert orc.validate(data, 5, 3) == 0
    for kw in (dict(k=1, l=3), dict(k=5, l=1), dict(k=5, l=6), dict(k=5, l=3, A=0),
               dict(k=5, l=3, B=0), dict(k=5, l=3, minDev=0.0), dict(k=5, l=3, itrPat=0),
               dict(k=5, l=3, metric=2), dict(k=150, l=3, A=1, B=1)):
        assert orc.validate(data, **kw) == -1, kw
    bad = data.copy()
    bad[3, 2] = np.nan
    assert orc.validate(bad, 5, 3) == -1
    assert orc.validate(data[:, :1], 2, 2) == -1  # d >= 2
    with pytest.raises(ValueError):
        orc.proclus(data, 1, 3)


def test_clamping_nM(orc):
    """B*k > A*k is clamped (#M = min(B k, #S)), not an error."""
    data = synth.generate(500, 6, 3, 2, seed=4)
    r = orc.proclus(data, 3, 2, A=4, B=10, seed=1)
    assert r.nS == 12 and r.nM == 12


def test_determinism_and_seed_dependence(orc):
    data, cfg = synth.config_data("C1", seed=2)
    a = orc.proclus(data, 5, 3, seed=5)
    b = orc.proclus(data, 5, 3, seed=5)
    c = orc.proclus(data, 5, 3, seed=6)
    assert np.array_equal(a.labels, b.labels) and a.cost == b.cost
    assert not (np.array_equal(a.medoids, c.medoids) and a.cost == c.cost)


def test_multi_levels(orc):
    """level 1 == independent runs; level 2 shares S, M of k_max."""
    data = synth.generate(2000, 8, 4, 3, seed=9)
    ks, ls = [3, 4], [2, 3]
    m1 = orc.proclus_multi(data, ks, ls, seed=4, reuse_level=1)
    for a, k in enumerate(ks):
        for b, l in enumerate(ls):
            r = orc.proclus(data, k, l, seed=4)
            got = m1[a * 2 + b]
            assert np.array_equal(got.labels, r.labels) and got.cost == r.cost
    m2 = orc.proclus_multi(data, ks, ls, seed=4, reuse_level=2)
    assert all(r.nM == 40 and r.nS == 400 for r in m2)
    for r, (k, l) in zip(m2, itertools.product(ks, ls)):
        assert r.dims.sum() == k * l


def test_multi_level3_warm_start(orc):
    """P:213 level 3 [R21]: the first setting is level 2's; a repeated (k, l)
    starts from a permutation of the previous MBest, so its costBest cannot
    exceed the previous one (slot order changes only the rounding of eq 2).
    Level 2 repeats the first run exactly (same stream IT); level 3 must not
    (its start differs) for some seed."""
    data = synth.generate(3000, 8, 4, 3, seed=21)
    differs = 0
    for seed in range(1, 9):
        m2 = orc.proclus_multi(data, [4, 4], [3], seed=seed, reuse_level=2)
        m3 = orc.proclus_multi(data, [4, 4], [3], seed=seed, reuse_level=3)
        assert np.array_equal(m3[0].labels, m2[0].labels) and m3[0].cost == m2[0].cost
        assert m3[1].cost <= m3[0].cost * (1 + 1e-12)
        assert np.array_equal(m2[1].labels, m2[0].labels) and m2[1].cost == m2[0].cost
        differs += m3[1].iterations != m2[1].iterations or not np.array_equal(
            m3[1].medoids, m2[1].medoids)
        for r in m3:
            assert r.dims.sum() == 4 * 3 and (r.dims.sum(axis=1) >= 2).all()
            assert len(set(r.medoids.tolist())) == 4
    assert differs > 0


def test_multi_level3_grid_shapes(orc):
    """Level 3 over a grid where k grows and shrinks (top-up from M minus MBest
    and subsets of MBest): invariants of every setting."""
    data = synth.generate(2500, 9, 5, 3, seed=22)
    ks, ls = [3, 5, 2], [2, 4]
    m3 = orc.proclus_multi(data, ks, ls, seed=3, reuse_level=3)
    for r, (k, l) in zip(m3, itertools.product(ks, ls)):
        assert r.dims.sum() == k * l and (r.dims.sum(axis=1) >= 2).all()
        assert len(set(r.medoids.tolist())) == k
        assert ((r.labels >= -1) & (r.labels < k)).all()
