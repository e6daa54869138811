"""Pins of the Lagrange-3 spatial variant (reading R-25 of DESIGN.md).

PAPER.md P:45 approximates the integrand "using 27 neighboring points from the data grids of
moments D_{i-1}, D_i, D_{i+1}".  The product reading (R-6) takes TSC weights in space; the
variant reads the 27 points as one tri-quadratic Lagrange stencil: the quadratic Lagrange
weights the time interpolation already uses (R-2), applied in x and y about the nearest
node.  These tests pin the oracle's variant to closed forms that the TSC reading fails.
"""
import math

import numpy as np

import oracle


def _quadratic_ring(nx, ny, hx, hy, H, coeffs):
    """Node samples of p(u, v) = a + b u + c v + d u^2 + e u v + f v^2 on every level; the two
    current components carry 2p and -p."""
    a, b, c, d, e, f = coeffs
    u = np.arange(nx) * hx
    v = np.arange(ny) * hy
    U, V = np.meshgrid(u, v)  # [ny, nx]
    p = a + b * U + c * V + d * U * U + e * U * V + f * V * V
    ring = np.zeros((H, ny, nx, 4))
    ring[..., 0] = p
    ring[..., 1] = 2.0 * p
    ring[..., 2] = -p
    return ring


def _problem(interp, coeffs=(0.7, 0.3, -0.2, 0.05, -0.03, 0.02)):
    nx, ny, hx, hy = 40, 36, 0.5, 0.55
    kmax = 3
    ring = _quadratic_ring(nx, ny, hx, hy, kmax + 2, coeffs)
    return oracle.Problem(nx=nx, ny=ny, hx=hx, hy=hy, c=1.0, dt=1.0, tau=1e-6,
                          kappa_max=kmax, k=3, n_pre=0, ring=ring, interp=interp), coeffs


def _p(coeffs, u, v):
    a, b, c, d, e, f = coeffs
    return a + b * u + c * v + d * u * u + e * u * v + f * v * v


def test_lagrange3_reproduces_quadratics_pointwise():
    """Biquadratic-exact: at any interior point the Lagrange-3 integrand equals p(u, v) (for
    every time weight, the levels being equal); the TSC integrand does not (it smooths p by
    (d h_x^2 + f h_y^2) / 4)."""
    rng = np.random.default_rng(25)
    P_l, co = _problem(1)
    P_t, _ = _problem(0)
    worst_l = worst_t = 0.0
    for _ in range(200):
        u, v = rng.uniform(2.0, 17.0), rng.uniform(2.0, 16.0)
        tau = rng.uniform(0.0, 1.0)
        want = _p(co, u, v)
        f = P_l.integrand(0, u, v, tau)
        np.testing.assert_allclose(f, [want, 2 * want, -want], rtol=0, atol=1e-13)
        worst_l = max(worst_l, abs(f[0] - want))
        worst_t = max(worst_t, abs(P_t.integrand(0, u, v, tau)[0] - want))
    d, f2 = co[3], co[5]
    smooth = (d * 0.5 ** 2 + f2 * 0.55 ** 2) / 4.0
    assert worst_l < 1e-13
    assert abs(worst_t - smooth) < 1e-9  # the TSC reading fails this pin by its smoothing


def test_lagrange3_interpolates_nodes():
    """At a grid node the variant returns the node value (Lagrange is interpolatory; TSC is not)."""
    rng = np.random.default_rng(7)
    P_l, _ = _problem(1)
    ring = P_l.ring
    for _ in range(50):
        ix, iy = rng.integers(2, 37), rng.integers(2, 33)
        f = P_l.integrand(0, ix * 0.5, iy * 0.55, 0.3)
        np.testing.assert_allclose(f, ring[0, iy, ix, :3], rtol=0, atol=1e-13)


def test_lagrange3_inner_circle_closed_form():
    """Full circle inside the grid: the periodic trapezoid on the exactly reproduced quadratic
    gives the circle mean p(c) + (d + f) r^2 / 2, times 2 pi (R-11, R-25)."""
    P_l, co = _problem(1)
    d, f2 = co[3], co[5]
    for (px, py, r) in [(10.0, 9.7, 3.3), (9.25, 10.45, 5.1), (11.0, 8.8, 0.37)]:
        out, n = P_l.inner(px, py, 0, r)
        assert n == 64
        want = 2 * math.pi * (_p(co, px, py) + (d + f2) * r * r / 2)
        np.testing.assert_allclose(out, [want, 2 * want, -want], rtol=1e-13, atol=1e-13)


def test_arc_end_nodes_take_the_outside_limit():
    """R-25b: the Lagrange-3 integrand jumps on the support boundary (just inside, the node
    row outside the grid has weight 0 but the first grid row has -1/8; just outside, every
    node is outside the grid), and every arc ends on that boundary.  The end nodes take the
    outside limit 0, so inner(r') no longer depends on which side the rounding of a crossing
    angle puts them: it is continuous in r' (a 1e-13 relative change of r' moves it by
    rounding only), which evaluating the end nodes fails by O(h g / 3)."""
    P, coeffs = _problem(1)
    hx = P.params.hx
    # the jump: just inside / outside the left edge u = -1.5 h of the support rectangle
    v = 7.3 * P.params.hy
    inside = P.integrand(0, -1.5 * hx * (1 - 1e-12), v, 0.5)
    outside = P.integrand(0, -1.5 * hx * (1 + 1e-12), v, 0.5)
    assert np.all(outside == 0.0) and abs(inside[0]) > 1e-3
    rng = np.random.default_rng(3)
    worst = 0.0
    for _ in range(150):
        ix, iy = rng.integers(0, 40), rng.integers(0, 36)
        r = rng.uniform(2.0, 25.0)
        px, py = P.mesh_point(ix, iy)
        a, _ = P.inner(px, py, 0, r)
        b, _ = P.inner(px, py, 0, r * (1 + 1e-13))
        worst = max(worst, float(np.max(np.abs(a - b))) / max(float(np.max(np.abs(a))), 1e-300))
    assert worst < 1e-9, worst
