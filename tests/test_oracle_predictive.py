"""Pins of the oracle's Predictive-RP variant: the paper's COMPUTE-POTENTIALS (Algorithm 1,
PAPER.md P:110-166) with forecast access patterns (kNN), uniform partitioning,
k-means clustering, MERGE-LISTS and adaptive refinement of the
intervals that miss the tolerance (lines 18-24).  Reading R-26 of DESIGN.md.

* kNN forecast: closed forms on a constant field and on a single spike.
* RP-CLUSTERING: the same Lloyd iterations as scikit-learn's KMeans from the same centres.
* MERGE-LISTS: the breakpoints are exactly the distinct rationals t/n (fractions.Fraction)
  of the members' grids, placed on S_j.
* The whole variant: "always achieves the required error tolerance" on the static
  Gaussian closed form; with one cluster per point and a forecast of one interval per
  subregion it is the canonical single-root tree (n_root = 1) bit for bit.
"""
import math
from fractions import Fraction

import numpy as np
import scipy.special as sp

import oracle

SQ = math.sqrt(math.pi / 2)


def test_knn_pattern_closed_forms():
    nx, ny, kmax = 7, 6, 3
    prev = np.full((nx * ny, kmax), 5, dtype=np.uint16)
    for p in range(nx * ny):
        for knn in (1, 5, 9, 25):
            assert oracle.knn_pattern(prev, nx, ny, p, 1, knn) == 5
    prev[:] = 0
    prev[3 * nx + 3, 2] = 9  # spike at (3, 3)
    assert oracle.knn_pattern(prev, nx, ny, 3 * nx + 3, 2, 1) == 9
    assert oracle.knn_pattern(prev, nx, ny, 3 * nx + 4, 2, 9) == 1      # (9 + 4) // 9
    assert oracle.knn_pattern(prev, nx, ny, 4 * nx + 4, 2, 5) == 0      # not a cross neighbour
    assert oracle.knn_pattern(prev, nx, ny, 2 * nx + 3, 2, 5) == 2      # (9 + 2) // 5
    prev[0, 0] = 9  # corner: 4 nodes in the 3x3 block
    assert oracle.knn_pattern(prev, nx, ny, 0, 0, 9) == 2                # (9 + 2) // 4
    assert oracle.knn_pattern(prev, nx, ny, 0, 0, 25) == 1               # (9 + 4) // 9


def test_kmeans_matches_scikit_learn_lloyd():
    from sklearn.cluster import KMeans
    rng = np.random.default_rng(5)
    npts, kmax, m = 300, 12, 7
    base = rng.integers(0, 60, size=(m, kmax))
    pat = (base[rng.integers(0, m, size=npts)] + rng.integers(0, 9, size=(npts, kmax))).astype(np.uint16)
    assign, it = oracle.kmeans(pat, m, max_iters=50)
    init = pat[[c * npts // m for c in range(m)]].astype(np.float64)
    km = KMeans(n_clusters=m, init=init, n_init=1, algorithm="lloyd", max_iter=50, tol=0.0)
    km.fit(pat.astype(np.float64))
    np.testing.assert_array_equal(assign, km.labels_)
    assert 1 < it < 50


def test_merge_lists_are_the_distinct_rationals():
    P = oracle.Problem(nx=4, ny=4, hx=1.0, hy=1.0, c=1.0, dt=0.7, tau=1e-6, kappa_max=3, k=5,
                       n_pre=0)
    rng = np.random.default_rng(2)
    npts, m = 16, 3
    pat = rng.integers(0, 13, size=(npts, 3)).astype(np.uint16)
    pat[0, 1] = 0
    assign = rng.integers(0, m, size=npts).astype(np.int32)
    off, bp = P.merge_partitions(pat, assign, m)
    cdt = 0.7
    for c in range(m):
        for j in range(3):
            got = bp[off[c * 3 + j]:off[c * 3 + j + 1]]
            ns = {int(pat[p, j]) for p in range(npts) if assign[p] == c and pat[p, j] > 0}
            want = sorted({Fraction(t, n) for n in ns for t in range(n + 1)})
            assert len(got) == len(want)
            if not want:
                continue
            a, b = j * cdt, (j + 1) * cdt
            assert np.all(np.diff(got) > 0)
            np.testing.assert_allclose(got, [a + (b - a) * float(f) for f in want], rtol=0,
                                       atol=1e-15)
            assert got[0] == a and got[-1] == b


def _gauss(kap=12, cdt=1.6, k=20, n_root=2):
    return oracle.Problem(nx=8, ny=8, hx=1.0, hy=1.0, c=1.0, dt=cdt, tau=1e-6 * SQ,
                          kappa_max=kap, k=k, n_pre=0, source=oracle.SRC_GAUSS, x0=0.0, y0=0.0,
                          width=1.0, q=1.0, bx=0.3, by=-0.2, n_root=n_root)


def test_predictive_meets_tolerance_on_the_gaussian_closed_form():
    """the forecast partition is only an initial condition; the result still meets
    the tolerance (here: the static Gaussian sheet, phi = sqrt(pi/2) i0e(s^2/4))."""
    P = _gauss()
    pts = np.arange(64)
    _, leaves = P.potentials_items(pts)
    res, clusters, leaves2, it = P.potentials_predictive(leaves, pts, knn=9)
    assert clusters.max() < 8 and it >= 1
    for p in pts:
        s = math.hypot(p % 8, p // 8)
        exact = SQ * sp.i0e(s * s / 4)
        assert abs(res["phi"][p] - exact) < 1e-6 * SQ
        assert abs(res["ax"][p] - 0.3 * res["phi"][p]) < 1e-15
    # the forecast partition changes the work, not the tolerance: some points do differ
    # from the canonical tree in their segment counts
    canon = P.potentials(pts)
    assert (res["nseg"] != canon["nseg"]).any()


def test_predictive_singleton_clusters_one_interval_is_the_single_root_tree():
    """One cluster per point and a forecast of one interval per subregion: every item's roots
    are its support [A, B] cut by S_j's ends, i.e. [A, B] itself -- the canonical tree with
    n_root = 1, bit for bit."""
    P = _gauss(n_root=1)
    pts = np.arange(64)
    prev = np.ones((64, 12), dtype=np.uint16)
    res, clusters, _, _ = P.potentials_predictive(prev, pts, knn=1, m=64)
    canon = P.potentials(pts)
    for key in ("phi", "ax", "ay", "err", "nseg", "nleaf", "evals"):
        np.testing.assert_array_equal(res[key], canon[key])


# ---------------------------------------------------------------- adaptive partitioning
def test_adaptive_partition_refines_the_earlier_partition_golden():
    """P:104 / R-26b: each piece of the earlier partition of S_j is cut into round(n/d) equal
    pieces (half up, at least 1), a_j and b_j close the list, a member without an earlier
    partition partitions S_j uniformly, and the cluster's lists are merged (sorted, distinct).
    Dyadic values, so every breakpoint is exact; expected lists written out by hand."""
    P = oracle.Problem(nx=2, ny=1, hx=1.0, hy=1.0, c=1.0, dt=1.0, tau=1e-6, kappa_max=1, k=5,
                       n_pre=0)
    x = [0.25, 0.5, 0.625, 0.75]                      # d = 3 pieces inside S_0 = [0, 1]
    prev_parts = np.array(x)
    prev_off = np.array([0, 0], dtype=np.int64)
    prev_len = np.array([4, 0], dtype=np.int32)       # point 1: no earlier partition
    assign = np.array([0, 0], dtype=np.int32)
    cases = {
        # n = 6, d = 3 -> 2 pieces each; point 1, n = 2 -> uniform halves of [0, 1]
        (6, 2): [0.0, 0.25, 0.375, 0.5, 0.5625, 0.625, 0.6875, 0.75, 1.0],
        # n = 4 -> round(4/3) = 1: the earlier partition itself, plus a_j, b_j
        (4, 1): [0.0, 0.25, 0.5, 0.625, 0.75, 1.0],
        # n = 5 -> round(5/3) = 2 (half up from 1.67)
        (5, 1): [0.0, 0.25, 0.375, 0.5, 0.5625, 0.625, 0.6875, 0.75, 1.0],
        # n = 1 -> round(1/3) = 0 -> at least 1
        (1, 4): [0.0, 0.25, 0.5, 0.625, 0.75, 1.0],
        # n = 9 -> 3 pieces each (thirds of 0.25 / 0.125 / 0.125)
        (9, 0): [0.0, 0.25, 0.25 + 0.25 / 3, 0.25 + 0.25 * 2 / 3, 0.5, 0.5 + 0.125 / 3,
                 0.5 + 0.125 * 2 / 3, 0.625, 0.625 + 0.125 / 3, 0.625 + 0.125 * 2 / 3, 0.75, 1.0],
    }
    for (n0, n1), want in cases.items():
        pat = np.array([[n0], [n1]], dtype=np.uint16)
        off, bp = P.merge_partitions_adaptive(pat, assign, 1, prev_off, prev_len, prev_parts)
        if n1 == 4:  # point 1 uniform in quarters on top
            want = sorted(set(want) | {0.0, 0.25, 0.5, 0.75, 1.0})
        np.testing.assert_allclose(bp[off[0]:off[1]], want, rtol=0, atol=1e-16)
        assert bp[off[0]] == 0.0 and bp[off[1] - 1] == 1.0


def test_adaptive_partition_with_unchanged_forecast_reproduces_the_canonical_leaves():
    """A static history, a one-point mesh (one cluster, one member) and the forecast equal to
    the earlier counts (k = 1): the merged list of every S_j is the earlier accepted partition
    plus a_j, b_j, so every root is an earlier leaf and is accepted at once -- the result is
    the canonical tree's, one segment per leaf (whatever k-means does on a larger mesh, where
    identical patterns share a cluster and their partitions merge, as the golden case
    above pins)."""
    for x0, y0 in ((0.0, 0.0), (1.3, -0.4), (3.1, 2.2), (-5.0, 0.5)):
        P = oracle.Problem(nx=1, ny=1, hx=1.0, hy=1.0, c=1.0, dt=1.6, tau=1e-6 * SQ,
                           kappa_max=12, k=20, n_pre=0, source=oracle.SRC_GAUSS, x0=x0, y0=y0,
                           width=1.0, q=1.0, bx=0.3, by=-0.2)
        canon, leaves, off, plen, parts = P.potentials_parts([0])
        for j in range(12):  # each partition tiles the item's support [A, B] in order
            L = parts[off[j]:off[j] + plen[j]]
            if len(L):
                A, B = P.clip(0.0, 0.0, j)
                # the last right end is the one the tree computed: A + (B - A) * 1
                assert L[0] == A and L[-1] == A + (B - A) and np.all(np.diff(L) > 0)
        res, _, _, _ = P.potentials_predictive_adaptive(leaves, off, plen, parts, [0], knn=1, m=1)
        assert res["ties"][0] + res["noise_ties"][0] == 0
        assert res["nseg"][0] == res["nleaf"][0] == canon["nleaf"][0]
        for key in ("phi", "ax", "ay"):
            assert abs(res[key][0] - canon[key][0]) <= 1e-14 * abs(canon["phi"][0])
