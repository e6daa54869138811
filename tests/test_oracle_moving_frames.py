"""Pins of the oracle's moving-frame geometry (retarded time t' = k dt - r'/c, PAPER.md P:43;
grids that move from step to step; interpolation from D_{i-1..i+1}; DESIGN.md
reading R-7: the frame at t' is the quadratic Lagrange interpolant of the three level frames).

Every expected value here comes from a closed-form trajectory the test defines, evaluated at
t' and inverted with numpy's linear solver -- not from the oracle's own formulas:

* a frame translating on a quadratic trajectory O(t) = O0 + V t + a t^2 / 2 with a fixed,
  rotated orientation is reproduced EXACTLY by the quadratic interpolation (rounding only);
* a frame rotating at constant angular velocity is reproduced within the Lagrange remainder
  bound max|f'''| / 3! * |(tau+1) tau (tau-1)| dt^3 of its cos/sin (R-7: no renormalisation);
* an analytic Gaussian carried by a translating, rotated frame (SURVEY C.4 source, static in
  the frame) gives phi(p) = int (Q/sigma^2) exp(-(r-s)^2/2sigma^2) i0e(r s/sigma^2) dr with
  s(r) = |p_local(t'(r)) - x0| -- scipy quad of the theta-closed form;
* a quarter-turn frame (c, s) = (0, 1) bins particles by hand-computed indices
  (tests/golden/bins_quarter_turn.json).

A w0 <-> w2 swap in the frame interpolation, a linear instead of quadratic interpolant, or a
sign error in the rotation to frame-local coordinates fails each of the first three.
"""
import json
import math
import os

import numpy as np
import pytest
import scipy.integrate as si
import scipy.special as sp

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _ring_frames(H, k, frame_of_t, dt):
    """Frames of levels k-H+1..k in ring-slot order (slot = level mod H)."""
    out = np.zeros((H, 4))
    for level in range(k - H + 1, k + 1):
        out[level % H] = frame_of_t(level * dt)
    return out


def _local(frame, p):
    """Frame-local coordinates of lab point p: solve lab = O + u (c, s) + v (-s, c)."""
    ox, oy, c, s = frame
    A = np.array([[c, -s], [s, c]])
    return np.linalg.solve(A, np.asarray(p) - np.array([ox, oy]))


def _problem(frames, kap, dt, k, n_pre=0, **src):
    return oracle.Problem(nx=8, ny=8, hx=0.5, hy=0.5, c=1.0, dt=dt, tau=1e-10, kappa_max=kap,
                          k=k, n_pre=n_pre, frames=frames, **src)


def test_translating_frame_reproduced_exactly():
    dt, kap, k = 0.7, 6, 10
    O0, V, acc, psi = np.array([1.5, -2.0]), np.array([0.45, -0.3]), np.array([0.08, 0.05]), 0.6

    def frame_of_t(t):
        o = O0 + V * t + 0.5 * acc * t * t
        return np.array([o[0], o[1], math.cos(psi), math.sin(psi)])

    P = _problem(_ring_frames(kap + 2, k, frame_of_t, dt), kap, dt, k)
    rng = np.random.default_rng(11)
    worst = 0.0
    for _ in range(60):
        p = rng.uniform(-4, 8, size=2)
        j = int(rng.integers(0, kap))
        r = (j + rng.uniform()) * dt
        cu, cv, w = P.centre(p[0], p[1], j, r)
        tp = k * dt - r  # retarded time t' = t_k - r/c, c = 1
        exp = _local(frame_of_t(tp), p)
        worst = max(worst, abs(cu - exp[0]), abs(cv - exp[1]))
        assert abs(w.sum() - 1.0) < 1e-15
    assert worst < 1e-12, worst


def test_rotating_frame_within_lagrange_remainder():
    dt, kap, k, om = 0.5, 6, 9, 0.1  # omega dt = 0.05 rad per step
    O0, V = np.array([0.3, 0.2]), np.array([0.2, 0.1])

    def frame_of_t(t):
        o = O0 + V * t
        return np.array([o[0], o[1], math.cos(0.4 + om * t), math.sin(0.4 + om * t)])

    P = _problem(_ring_frames(kap + 2, k, frame_of_t, dt), kap, dt, k)
    rng = np.random.default_rng(12)
    for _ in range(60):
        p = rng.uniform(-3, 6, size=2)
        j = int(rng.integers(0, kap))
        tau_t = rng.uniform()
        r = (j + 1 - tau_t) * dt
        cu, cv, _ = P.centre(p[0], p[1], j, r)
        tp = k * dt - r
        f = frame_of_t(tp)
        exp = _local(f, p)
        # cos/sin interpolated, not renormalised: each is off by at most the cubic remainder
        bound = om ** 3 / 6 * abs((tau_t + 1) * tau_t * (tau_t - 1)) * dt ** 3
        d = np.asarray(p) - f[:2]
        tol = (abs(d[0]) + abs(d[1])) * bound * 1.001 + 1e-13
        assert abs(cu - exp[0]) <= tol and abs(cv - exp[1]) <= tol, (cu - exp[0], cv - exp[1], tol)
        # and the remainder is not vacuous: a sign error in the rotation is many bounds away
        assert tol < 1e-4


@pytest.mark.parametrize("pt", [(0.0, 0.0), (1.2, -0.7), (-2.0, 1.5)])
def test_gaussian_in_translating_frame_vs_quadrature(pt):
    """A Gaussian sheet static in a moving frame: the retarded integral reduces (theta done in
    closed form over the full circle) to a 1-D integral in r' that scipy evaluates directly."""
    dt, kap = 1.8, 16
    n_pre = kap + 1
    k = 0
    psi, V, O0 = 0.5, np.array([0.09, 0.04]), np.array([-3.0, 2.0])
    x0 = np.array([2.0, 1.5])  # Gaussian centre, frame-local

    def frame_of_t(t):
        o = O0 + V * t
        return np.array([o[0], o[1], math.cos(psi), math.sin(psi)])

    frames = _ring_frames(kap + 2, k, frame_of_t, dt)
    P = _problem(frames, kap, dt, k, n_pre=n_pre, source=oracle.SRC_GAUSS, x0=x0[0], y0=x0[1],
                 width=1.0, q=1.0, bx=0.3, by=-0.2)
    # lab point: the frame-local point x0 + pt at t = 0
    f0 = frame_of_t(0.0)
    u, v = x0 + np.array(pt)
    p = (f0[0] + u * f0[2] - v * f0[3], f0[1] + u * f0[3] + v * f0[2])
    res = P.point_lab(*p)

    def s_of(r):
        return float(np.linalg.norm(_local(frame_of_t(-r), p) - x0))

    def inner(r):
        s = s_of(r)
        return math.exp(-0.5 * (r - s) ** 2) * sp.i0e(r * s)  # (Q/sigma^2) e^{-(r^2+s^2)/2} I0(rs)

    R = kap * dt
    exact, est = si.quad(inner, 0.0, R, limit=400, epsabs=1e-15, epsrel=1e-13)
    assert est < 1e-12
    assert res.phi > 0.1
    assert abs(res.phi - exact) < 1e-9 * exact, (res.phi, exact)
    # rigid current: A = beta * phi
    assert abs(res.ax - 0.3 * res.phi) < 1e-15 and abs(res.ay + 0.2 * res.phi) < 1e-15
    # the frame motion matters at this tolerance: the same source in a frame at rest differs
    Ps = _problem(_ring_frames(kap + 2, k, lambda t: frame_of_t(0.0), dt), kap, dt, k,
                  n_pre=n_pre, source=oracle.SRC_GAUSS, x0=x0[0], y0=x0[1], width=1.0, q=1.0)
    assert abs(Ps.point_lab(*p).phi - exact) > 1e-4 * exact


def test_quarter_turn_bins_golden():
    with open(os.path.join(GOLD, "bins_quarter_turn.json")) as f:
        g = json.load(f)
    fr = g["frame"]
    assert fr[2] == 0.0 and fr[3] == 1.0
    for case in g["cases"]:
        b, ix, iy, dx, dy = oracle.bin_of(case["x"], case["y"], fr, g["hx"], g["hy"], g["nx"],
                                          g["ny"])
        assert b == case["bin"], case
        if b >= 0:
            assert (ix, iy) == (case["ix"], case["iy"]), case
            assert dx == case["dx"] and dy == case["dy"], case
