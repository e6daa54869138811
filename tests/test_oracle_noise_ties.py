"""Pin of the oracle's decision-noise diagnostic (DESIGN reading R-28; R-10 acceptance
err <= tau (b - a) / R).

err = max_c |K15_c - G7_c| is the difference of two nearly equal sums, so summing the same
terms in another (equally valid) order moves it by a few ulp of |K| + |G|; a decision whose
margin |err - tol| is inside that noise is decided by rounding.  The oracle reports, per
point, the smallest margin in units of eps (|K_rho| + |G_rho|) (`min_noise`) and counts the
decisions below 4 such units (`noise_ties`).  With one root segment (max_depth = 0,
n_root = 1, kappa = 1, S_0 = [0, R]) the point's err and phi are that segment's err and
K_rho, so tau can be set to put the single decision exactly on the tie, or a known number of
noise units away from it."""
import math

import numpy as np

import oracle

EPS = np.finfo(float).eps


def _root_problem(tau):
    # static Gaussian (sigma = 1, Q = 1), one subregion [0, 1.6] = [0, R]: tol = tau exactly
    # up to the rounding of (tau * 1.6) / 1.6
    return oracle.Problem(nx=8, ny=8, hx=1.0, hy=1.0, c=1.0, dt=1.6, tau=tau, kappa_max=1, k=20,
                          n_pre=0, source=oracle.SRC_GAUSS, x0=0.0, y0=0.0, width=1.0, q=1.0,
                          max_depth=0, n_root=1)


def test_noise_margin_of_a_single_decision():
    r0 = _root_problem(1.0).point_lab(0.5, 0.3)
    assert r0.nseg == 1 and r0.nleaf == 1
    err0, phi0 = r0.err, r0.phi
    assert 0.0 < err0 < 1e-3 * phi0
    # exactly on the tie: flagged by both criteria
    r = _root_problem(err0).point_lab(0.5, 0.3)
    assert r.noise_ties == 1 and r.min_noise < 1.0 and r.ties == 1
    # 100 noise units away (|K| + |G| = 2 |K| to within err0): not flagged, and min_noise is
    # |err - tol| / (eps (|K| + |G|)) -- a wrong scale (eps |K|, ulp(err), ...) fails here
    delta = 100.0 * EPS * 2.0 * abs(phi0)
    r = _root_problem(err0 + delta).point_lab(0.5, 0.3)
    assert r.noise_ties == 0
    assert abs(r.min_noise - 100.0) < 1.0, r.min_noise
    # 2 noise units: flagged by R-28 although the relative margin 2 eps 2|K| / err0 can exceed
    # the old 1e-9 tie bar when |K| / err0 is large
    r = _root_problem(err0 + delta / 50.0).point_lab(0.5, 0.3)
    assert r.noise_ties == 1 and 1.0 < r.min_noise < 3.0 and r.ties == 0
    assert r.phi == phi0  # the diagnostic never changes the result


def test_smooth_source_has_no_noise_ties():
    """The closed-form Gaussian at the default tau: every decision far outside the noise."""
    P = oracle.Problem(nx=8, ny=8, hx=1.0, hy=1.0, c=1.0, dt=1.6, tau=1e-6 * math.sqrt(math.pi / 2),
                       kappa_max=12, k=20, n_pre=0, source=oracle.SRC_GAUSS, x0=0.0, y0=0.0,
                       width=1.0, q=1.0)
    r = P.point_lab(1.0 * math.cos(0.4), 1.0 * math.sin(0.4))
    assert r.noise_ties == 0 and r.min_noise > 4.0
