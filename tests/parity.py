"""Parity helpers: compare a GPU run with an oracle run on the same seeded
inputs and RNG streams (north_star contract: labels, medoids and dimension
sets bit-exact; cost within 1e-5 relative; divergence allowed only at a
decision the oracle reports as a near tie)."""
from __future__ import annotations

import numpy as np

NEAR_TIE = 1e-9      # relative Z-selection / cost-comparison gap (SURVEY 8(c) iii)
COST_RTOL = 1e-5     # north_star tolerance for fp64 sums in a different order


def first_divergence(gt, ot):
    """First iteration where the GPU trace and the oracle trace differ, with
    the oracle's margin there, or None."""
    n = min(len(gt.cost), len(ot.cost))
    for it in range(n):
        if not np.array_equal(gt.mcur[it], ot.mcur[it]):
            return it, "mcur", None
        if not np.array_equal(gt.nL[it], ot.nL[it]):
            return it, "nL", None
        if not np.array_equal(gt.dims[it], ot.dims[it]):
            return it, "dims", float(ot.zgap[it])
        if not np.array_equal(gt.sizes[it], ot.sizes[it]):
            return it, "sizes", None
        if bool(gt.improved[it]) != bool(ot.improved[it]):
            return it, "improved", float(ot.costgap[it])
    if len(gt.cost) != len(ot.cost):
        return n, "length", None
    return None


def assert_parity(g, o, gt=None, ot=None, what=""):
    """g/o: results (labels, medoids, dims, cost, iterations); gt/ot traces."""
    if gt is not None and ot is not None:
        div = first_divergence(gt, ot)
        if div is not None:
            it, field, margin = div
            if margin is not None and margin < NEAR_TIE:
                return f"near-tie divergence at iteration {it} ({field}, gap {margin:.3g})"
            raise AssertionError(f"{what}: trace diverges at iteration {it} in {field} "
                                 f"(oracle margin {margin})")
        np.testing.assert_allclose(gt.cost, ot.cost, rtol=COST_RTOL, atol=0)
        np.testing.assert_allclose(gt.X, ot.X, rtol=1e-9, atol=1e-12)
        np.testing.assert_array_equal(gt.bad, ot.bad)
    assert g.iterations == o.iterations, f"{what}: iterations {g.iterations} vs {o.iterations}"
    np.testing.assert_array_equal(g.medoids, o.medoids, err_msg=f"{what}: medoids")
    np.testing.assert_array_equal(g.dims, o.dims, err_msg=f"{what}: dims")
    lab_g = np.asarray(g.labels)
    bad = np.flatnonzero(lab_g != o.labels)
    assert bad.size == 0, f"{what}: {bad.size} labels differ, first at {bad[:5]}"
    np.testing.assert_allclose(g.cost, o.cost, rtol=COST_RTOL, atol=0)
    return None
