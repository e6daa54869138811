"""Pins of the theta limits ("limits as in [9]"; reading R-5).

The arcs of a circle inside the support rectangle (grid path) or disk (analytic
source) are checked against dense sampling of the plain inside test, and the
support clip [A, B] of a subregion against a brute-force scan over r'.
"""
import math

import numpy as np
import pytest

import oracle

TWO_PI = 2 * math.pi


def _inside_fraction_rect(cu, cv, r, U0, U1, V0, V1, n=400_000):
    th = (np.arange(n) + 0.5) * (TWO_PI / n)
    u, v = cu + r * np.cos(th), cv + r * np.sin(th)
    return ((u >= U0) & (u <= U1) & (v >= V0) & (v <= V1)).mean() * TWO_PI


def _arc_total(n, arcs):
    if n < 0:
        return TWO_PI
    return float(np.sum(arcs[:, 1] - arcs[:, 0]))


def test_arcs_rect_random_vs_sampling():
    rng = np.random.default_rng(11)
    U0, U1, V0, V1 = -1.0, 3.0, -0.5, 1.5
    for _ in range(300):
        cu, cv = rng.uniform(-4, 6), rng.uniform(-4, 5)
        r = rng.uniform(0.05, 6.0)
        n, arcs = oracle.arcs_rect(cu, cv, r, U0, U1, V0, V1)
        got = _arc_total(n, arcs)
        want = _inside_fraction_rect(cu, cv, r, U0, U1, V0, V1)
        assert abs(got - want) < 5e-5, (cu, cv, r, n, arcs)
        for t1, t2 in (arcs if n > 0 else []):
            assert t1 < t2
            mid = 0.5 * (t1 + t2)
            u, v = cu + r * math.cos(mid), cv + r * math.sin(mid)
            assert U0 <= u <= U1 and V0 <= v <= V1
            for t in (t1, t2):  # endpoints lie on the boundary
                u, v = cu + r * math.cos(t), cv + r * math.sin(t)
                dist = min(abs(u - U0), abs(u - U1), abs(v - V0), abs(v - V1))
                assert dist < 1e-12


def test_arcs_rect_special_cases():
    # fully inside -> full circle
    assert oracle.arcs_rect(1.0, 0.5, 0.2, -1, 3, -0.5, 1.5)[0] == -1
    # disjoint -> none
    assert oracle.arcs_rect(10.0, 10.0, 0.5, -1, 3, -0.5, 1.5)[0] == 0
    # circle enclosing the rectangle -> none
    assert oracle.arcs_rect(1.0, 0.5, 10.0, -1, 3, -0.5, 1.5)[0] == 0
    # circle through a corner, centred at the opposite corner of a unit square:
    # the quarter arc inside is [0, pi/2]
    n, arcs = oracle.arcs_rect(0.0, 0.0, 1.0, 0.0, 1.0, 0.0, 1.0)
    assert n == 1 and abs(arcs[0, 0]) < 1e-15 and abs(arcs[0, 1] - math.pi / 2) < 1e-15
    # centre on an edge: half circle inside a wide rectangle
    n, arcs = oracle.arcs_rect(0.0, 0.0, 1.0, -5, 5, 0.0, 5.0)
    assert n == 1 and abs(arcs[0, 1] - arcs[0, 0] - math.pi) < 1e-15
    # four arcs: circle crossing all four edges of a square centred on it
    n, arcs = oracle.arcs_rect(0.0, 0.0, 1.2, -1.0, 1.0, -1.0, 1.0)
    assert n == 4
    want = TWO_PI - 8 * math.acos(1 / 1.2)
    assert abs(_arc_total(n, arcs) - want) < 1e-14


def test_arcs_disk_vs_sampling():
    rng = np.random.default_rng(12)
    for _ in range(200):
        cu, cv = rng.uniform(-3, 3), rng.uniform(-3, 3)
        r = rng.uniform(0.05, 5.0)
        a = rng.uniform(0.3, 2.0)
        n, arcs = oracle.arcs_disk(cu, cv, r, 0.0, 0.0, a)
        got = _arc_total(n, arcs)
        th = (np.arange(200_000) + 0.5) * (TWO_PI / 200_000)
        inside = ((cu + r * np.cos(th)) ** 2 + (cv + r * np.sin(th)) ** 2 <= a * a).mean() * TWO_PI
        assert abs(got - inside) < 1e-4


def _problem_static_grid(nx=12, ny=10, kap=6, cdt=1.3):
    H = kap + 2
    return oracle.Problem(nx=nx, ny=ny, hx=0.7, hy=0.9, c=1.0, dt=cdt, tau=1e-6, kappa_max=kap,
                          k=10, n_pre=0, ring=np.zeros((H, ny, nx, 4)))


def _problem_moving(kap=6):
    # frames translating along +u at speed 0.6 c and rotating slowly
    H = kap + 2
    fr = np.zeros((H, 4))
    k = 10
    for l in range(k - H + 1, k + 1):
        psi = 0.02 * l
        fr[l % H] = [0.6 * l, 0.1 * l, math.cos(psi), math.sin(psi)]
    return oracle.Problem(nx=12, ny=10, hx=0.7, hy=0.9, c=1.0, dt=1.0, tau=1e-6, kappa_max=kap,
                          k=k, n_pre=0, ring=np.zeros((H, 10, 12, 4)), frames=fr)


@pytest.mark.parametrize("mk", [_problem_static_grid, _problem_moving])
def test_clip_vs_brute_scan(mk):
    P = mk()
    rng = np.random.default_rng(5)
    cdt = P.params.c * P.params.dt
    for _ in range(40):
        px, py = rng.uniform(-6, 14), rng.uniform(-6, 12)
        for j in range(P.kappa()):
            a, b = j * cdt, (j + 1) * cdt
            rs = np.linspace(a, b, 4001)
            sup = np.array([(lambda d: d[0] <= r * r <= d[1])(P.dists(px, py, j, r)) for r in rs])
            clip = P.clip(px, py, j)
            if not sup.any():
                # an empty scan must not hide a wide support interval
                assert clip is None or clip[1] - clip[0] < 2 * (b - a) / 4000
                continue
            assert clip is not None
            A, B = clip
            lo, hi = rs[sup.argmax()], rs[len(sup) - 1 - sup[::-1].argmax()]
            step = (b - a) / 4000
            assert A <= lo + 1e-12 and A >= lo - step - 1e-12
            assert B >= hi - 1e-12 and B <= hi + step + 1e-12


def test_static_clip_closed_form():
    # static frame: A = max(a_j, d_min), B = min(b_j, d_max)
    P = _problem_static_grid()
    U0, U1, V0, V1 = -1.5 * 0.7, 12.5 * 0.7, -1.5 * 0.9, 10.5 * 0.9
    for px, py in [(-4.0, 3.0), (12.0, 13.0), (2.0, 2.0), (-3.0, -3.0)]:
        ex = max(U0 - px, 0.0, px - U1)
        ey = max(V0 - py, 0.0, py - V1)
        dmin = math.hypot(ex, ey)
        dmax = math.hypot(max(abs(px - U0), abs(px - U1)), max(abs(py - V0), abs(py - V1)))
        for j in range(P.kappa()):
            a, b = j * 1.3, (j + 1) * 1.3
            clip = P.clip(px, py, j)
            A, B = max(a, dmin), min(b, dmax)
            if A >= B:
                assert clip is None
            else:
                assert clip is not None
                assert abs(clip[0] - A) < 1e-13 and abs(clip[1] - B) < 1e-13


def test_integrand_vanishes_at_arc_ends():
    """R-24: the end nodes of every arc lie on the support rectangle [-1.5h, (N+0.5)h]^2,
    where every node of the zero-padded 3x3 TSC stencil is outside the grid or has weight
    0, so the integrand there is 0 up to the rounding of the crossing angle.  (The GPU path
    skips these nodes; the oracle evaluates them.)"""
    rng = np.random.default_rng(24)
    nx, ny, hx, hy = 12, 9, 0.7, 0.45
    kmax = 2
    H = kmax + 2
    ring = rng.uniform(0.5, 1.5, size=(H, ny, nx, 4))
    ring[..., 3] = 0.0
    P = oracle.Problem(nx=nx, ny=ny, hx=hx, hy=hy, c=1.0, dt=1.0, tau=1e-6, kappa_max=kmax,
                       k=2, n_pre=0, ring=ring)
    U0, U1, V0, V1 = -1.5 * hx, (nx + 0.5) * hx, -1.5 * hy, (ny + 0.5) * hy
    scale = float(np.abs(ring).max())
    n_ends = 0
    for _ in range(400):
        cu, cv = rng.uniform(-3, 11), rng.uniform(-3, 7)
        r = rng.uniform(0.1, 9.0)
        n, arcs = oracle.arcs_rect(cu, cv, r, U0, U1, V0, V1)
        for t1, t2 in (arcs if n > 0 else []):
            for t in (t1, t2):
                u, v = cu + r * math.cos(t), cv + r * math.sin(t)
                f = P.integrand(0, u, v, rng.uniform(0.0, 1.0))
                assert np.all(np.abs(f) <= 1e-20 * scale), (cu, cv, r, t, f)
                n_ends += 1
    assert n_ends > 200
