"""Pins of the oracle's elementary rules against mathematics, not against itself.

* GK15 / G7 (outer rule of PAPER.md Eq. 2): exactness on
  monomials (K15 to degree 23, G7 to degree 13) and G7 == numpy's Gauss-Legendre.
* TSC weights (R-6, the 27-point stencil of P:45): partition of unity, first and
  second moments, C^1 continuity across the nearest-node switch.
* Lagrange-3 in time (R-2): reproduces quadratics.
* The whole gk15() segment path: a uniform disk seen from its centre with a
  quadratic-in-time amplitude makes inner(r') an exact quadratic in r', so K15 and G7
  must both equal the closed-form integral and err must vanish.
"""
import math

import numpy as np
import pytest

import oracle


def test_gk15_monomials():
    x, wk, wg = oracle.gk15_constants()
    nodes = np.concatenate([-x[:7], [0.0], x[6::-1]])
    wkf = np.concatenate([wk[:7], [wk[7]], wk[6::-1]])
    for deg in range(0, 24):
        exact = 0.0 if deg % 2 else 2.0 / (deg + 1)
        assert abs(np.dot(wkf, nodes ** deg) - exact) < 2e-15, deg
    # degree 24 is NOT integrated exactly (catches a weight table that is secretly higher order)
    assert abs(np.dot(wkf, nodes ** 24) - 2.0 / 25) > 1e-12
    gn = np.array([-x[1], -x[3], -x[5], 0.0, x[5], x[3], x[1]])
    gw = np.array([wg[0], wg[1], wg[2], wg[3], wg[2], wg[1], wg[0]])
    for deg in range(0, 14):
        exact = 0.0 if deg % 2 else 2.0 / (deg + 1)
        assert abs(np.dot(gw, gn ** deg) - exact) < 2e-15, deg


def test_g7_matches_numpy_legendre():
    x, wk, wg = oracle.gk15_constants()
    ln, lw = np.polynomial.legendre.leggauss(7)
    np.testing.assert_allclose(np.sort(ln), np.sort([-x[1], -x[3], -x[5], 0.0, x[5], x[3], x[1]]),
                               atol=1e-15)
    np.testing.assert_allclose(np.sort(lw), np.sort([wg[0], wg[1], wg[2], wg[3], wg[2], wg[1], wg[0]]),
                               atol=1e-15)


@pytest.mark.parametrize("d", [-0.5, -0.37, -0.1, 0.0, 0.2, 0.49999, 0.5])
def test_tsc_moments(d):
    w = oracle.tsc_weights(d)
    off = np.array([-1.0, 0.0, 1.0])
    assert abs(w.sum() - 1.0) < 1e-15
    assert abs(np.dot(w, off) - d) < 1e-15           # reproduces linear functions
    assert abs(np.dot(w, (off - d) ** 2) - 0.25) < 1e-15  # quadratic B-spline variance 1/4
    assert (w >= 0).all()


def test_tsc_c1_across_switch():
    # The interpolant of an arbitrary node sequence has the same value and slope on
    # both sides of t = n + 1/2, where the nearest node switches from n to n+1
    # (left: node n, delta = +1/2; right: node n+1, delta = -1/2).
    g = np.array([0.3, -1.2, 2.5, 0.7, 1.9, -0.4])
    eps = 1e-6
    wl, wr = oracle.tsc_weights(0.5), oracle.tsc_weights(-0.5)
    dl = (oracle.tsc_weights(0.5) - oracle.tsc_weights(0.5 - eps)) / eps
    dr = (oracle.tsc_weights(-0.5 + eps) - oracle.tsc_weights(-0.5)) / eps
    for n in (1, 2, 3):
        left = sum(wl[a] * g[n + a - 1] for a in range(3))
        right = sum(wr[a] * g[n + a] for a in range(3))
        assert abs(left - right) < 1e-15
        sl = sum(dl[a] * g[n + a - 1] for a in range(3))
        sr = sum(dr[a] * g[n + a] for a in range(3))
        assert abs(sl - sr) < 1e-5
        assert abs(sl - (g[n + 1] - g[n])) < 1e-5


def test_lagrange3_reproduces_quadratics():
    rng = np.random.default_rng(3)
    for _ in range(20):
        a, b, c = rng.standard_normal(3)
        p = lambda t: a + b * t + c * t * t
        for t in (0.0, 0.13, 0.5, 0.77, 1.0):
            w = oracle.lagrange3_weights(t)
            assert abs(w[0] * p(-1) + w[1] * p(0) + w[2] * p(1) - p(t)) < 1e-14
    # node values (t = 0 -> level k-j-1, t = 1 -> level k-j)
    np.testing.assert_array_equal(oracle.lagrange3_weights(1.0), [0.0, 0.0, 1.0])
    np.testing.assert_array_equal(oracle.lagrange3_weights(0.0), [0.0, 1.0, 0.0])


@pytest.mark.parametrize("rule", [0, 1])
def test_gk15_segment_on_exact_quadratic(rule):
    # disk of radius a=10 centred on p: inner(r') = 2*pi*sigma_s*amp(t_k - r'/c) for r' < a.
    # amp is quadratic in time -> Lagrange-3 exact -> inner is an exact quadratic in r'.
    kap, dt, k = 4, 1.0, 9
    H = kap + 2
    al, be, ga = 1.5, -0.3, 0.07
    amp = np.zeros(H)
    for l in range(k - H + 1, k + 1):
        t = l * dt
        amp[l % H] = al + be * t + ga * t * t
    P = oracle.Problem(nx=8, ny=8, hx=1.0, hy=1.0, c=1.0, dt=dt, tau=1e-9, kappa_max=kap, k=k,
                       n_pre=0, source=oracle.SRC_DISK, x0=0.0, y0=0.0, width=10.0, q=2.0, amp=amp,
                       rule=rule)
    for j, (a, b) in [(0, (0.1, 0.9)), (2, (2.0, 3.0)), (3, (3.25, 3.5))]:
        K, G, err = P.gk15(0.0, 0.0, j, a, b)
        tk = k * dt
        F = lambda r: (al * r + be * (tk * r - r * r / 2) + ga * (tk * tk * r - tk * r * r + r ** 3 / 3))
        exact = 2 * math.pi * 2.0 * (F(b) - F(a))
        assert abs(K[0] - exact) < 1e-13 * abs(exact)
        assert abs(G[0] - exact) < 1e-13 * abs(exact)
        assert err < 1e-13 * abs(exact)


def test_simpson_boole_weights():
    """Rule 1 (the paper's Simpson, with the standard Richardson value = Boole's rule,
    R-22): Boole h/90 (7,32,12,32,7) is exact to degree 5 and not 6, Simpson h/12 (1,4,2,4,1)
    to degree 3 and not 4, on [0, 1] with nodes 0, 1/4, 1/2, 3/4, 1."""
    x = np.array([0.0, 0.25, 0.5, 0.75, 1.0])
    wb = np.array([7, 32, 12, 32, 7]) / 90.0
    ws = np.array([1, 4, 2, 4, 1]) / 12.0
    for d in range(6):
        assert abs(np.dot(wb, x ** d) - 1.0 / (d + 1)) < 1e-15
    assert abs(np.dot(wb, x ** 6) - 1.0 / 7) > 1e-6
    for d in range(4):
        assert abs(np.dot(ws, x ** d) - 1.0 / (d + 1)) < 1e-15
    assert abs(np.dot(ws, x ** 4) - 1.0 / 5) > 1e-5
    # the oracle's rule-1 segment on a constant inner integral (disk seen from its centre)
    P = oracle.Problem(nx=8, ny=8, hx=1.0, hy=1.0, c=1.0, dt=1.0, tau=1e-9, kappa_max=3, k=9,
                       n_pre=0, source=oracle.SRC_DISK, x0=0.0, y0=0.0, width=10.0, q=1.5, rule=1)
    K, G, err = P.gk15(0.0, 0.0, 1, 1.2, 1.9)
    assert abs(K[0] - 2 * math.pi * 1.5 * 0.7) < 1e-13 and err < 1e-13
