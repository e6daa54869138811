"""Invariants of the oracle's potentials that hold exactly or to rounding.

* Linearity with exact power-of-two scaling: (M, tau) -> (2M, 2tau) gives bit-identical 2x
  results and the same subdivision (Eq. 2 is linear in f; accept test err <= tau (b-a)/R).
* J = 0 => A = 0 exactly (P:32 moments; R-1).
* Steady state (P:176-177 LCLS bend, rigid pre-history): a rigid bunch on a circular orbit
  gives the same potentials at steps k and k+m (to rounding) and the same subdivision.
* Static rigid history: the result does not depend on the step index k.
"""
import math

import numpy as np
import pytest

import oracle
import workloads as W


def _grid_problem(ring, fr, cfg, k, tau, n_pre=0):
    return oracle.Problem(nx=cfg.nx, ny=cfg.ny, hx=cfg.hx, hy=cfg.hy, c=cfg.c, dt=cfg.dt, tau=tau,
                          kappa_max=cfg.kappa_max, k=k, n_pre=n_pre, ring=ring, frames=fr)


def _cfg_static(n=16, kap=8):
    return W.Config(number=0, name="t", nx=n, ny=n, n_particles=1, steps=1, kappa_max=kap,
                    geometry="static", sigma=1.0, cdt=1.6)


def test_scaling_by_two_is_exact():
    cfg = _cfg_static()
    x, y, ux, uy = W.particles(W.config(1), n=3000, seed=3)
    M, _, _ = oracle.deposit(x, y, ux + 0.1, uy, 1e-3, W.frame(cfg, 0), cfg.nx, cfg.ny, cfg.hx, cfg.hy)
    ring = np.repeat(M[None], cfg.H, axis=0)
    fr = W.ring_frames(cfg, 5)
    pts = np.arange(0, cfg.nx * cfg.ny, 17)
    r1 = _grid_problem(ring, fr, cfg, 5, 1e-7).potentials(pts)
    r2 = _grid_problem(2 * ring, fr, cfg, 5, 2e-7).potentials(pts)
    for key in ("phi", "ax", "ay", "err"):
        np.testing.assert_array_equal(r2[key], 2 * r1[key])
    np.testing.assert_array_equal(r2["nseg"], r1["nseg"])


def test_zero_current_gives_zero_vector_potential():
    cfg = _cfg_static()
    x, y, ux, uy = W.particles(W.config(1), n=3000, seed=4)
    M, _, _ = oracle.deposit(x, y, ux, uy, 1e-3, W.frame(cfg, 0), cfg.nx, cfg.ny, cfg.hx, cfg.hy)
    assert (M[..., 1:] == 0).all()
    ring = np.repeat(M[None], cfg.H, axis=0)
    r = _grid_problem(ring, W.ring_frames(cfg, 4), cfg, 4, 1e-6).potentials(np.arange(0, 256, 9))
    assert (r["ax"] == 0).all() and (r["ay"] == 0).all()
    assert (r["phi"] > 0).all()


def test_static_result_independent_of_step():
    cfg = _cfg_static()
    ring = W.node_gaussian_ring(cfg, k=0)
    ra = _grid_problem(ring, W.ring_frames(cfg, 0), cfg, 0, 1e-6, n_pre=cfg.n_pre).potentials([0, 77, 136])
    # same rigid grids in every slot, viewed at step 23 without pre-history
    rb = _grid_problem(ring, W.ring_frames(cfg, 23), cfg, 23, 1e-6).potentials([0, 77, 136])
    np.testing.assert_array_equal(ra["phi"], rb["phi"])
    np.testing.assert_array_equal(ra["nseg"], rb["nseg"])


def _bend_small():
    c = W.config(2)
    return W.Config(number=2, name="bend-small", nx=24, ny=24, n_particles=1, steps=60,
                    kappa_max=60, geometry="bend", sigma=c.sigma, cdt=c.cdt, gamma0=c.gamma0,
                    r0=c.r0, sigma_xp=c.sigma_xp, q_over_mc=c.q_over_mc)


@pytest.mark.slow
def test_bend_steady_state_stationarity():
    cfg = _bend_small()
    ring = W.node_gaussian_ring(cfg, k=0, beta=(cfg.beta0, 0.0))
    pts = [12 * 24 + 12, 12 * 24 + 20, 5 * 24 + 3]
    out = []
    for k in (0, 1, 7):
        P = _grid_problem(ring, W.ring_frames(cfg, k), cfg, k, cfg.tau, n_pre=cfg.n_pre)
        out.append(P.potentials(pts))
    for r in out[1:]:
        np.testing.assert_array_equal(r["nseg"], out[0]["nseg"])
        rel = np.abs(r["phi"] - out[0]["phi"]) / np.abs(out[0]["phi"])
        assert rel.max() < 1e-10, rel
    # sanity: the bend potential at the bunch centre is O(Q/sigma)
    scale = 1.0 / cfg.sigma * math.sqrt(math.pi / 2)
    assert 0.5 < out[0]["phi"][0] / scale < 10


# ---------------------------------------------------------------- rigid pre-history (R-23)
def test_rigid_level_static_frames_is_exact_copy():
    cfg = _cfg_static()
    rng = np.random.default_rng(5)
    M = rng.standard_normal((cfg.ny, cfg.nx, 4))
    out = oracle.rigid_level(M, W.frame(cfg, 0), W.frame(cfg, -3))
    np.testing.assert_array_equal(out, M)


def test_rigid_level_quarter_turn_is_exact():
    # psi_0 = 0, psi_l = pi/2 given exactly as (cos, sin) = (0, 1): (jx, jy) -> (-jy, jx)
    M = np.random.default_rng(6).standard_normal((5, 6, 4))
    out = oracle.rigid_level(M, [0, 0, 1.0, 0.0], [0, 0, 0.0, 1.0])
    np.testing.assert_array_equal(out[..., 0], M[..., 0])
    np.testing.assert_array_equal(out[..., 1], -M[..., 2])
    np.testing.assert_array_equal(out[..., 2], M[..., 1])


def test_rigid_ring_carries_the_tangent_current_of_each_level():
    """A bunch moving along the step-0 tangent becomes, at every pre-history level, a bunch
    moving along THAT level's tangent (circular orbit; the closed form of the rotation), with
    the same charge density and the same local (J.t, J.n) components."""
    cfg = _bend_small()
    fr = W.ring_frames(cfg, 0)
    g = W.node_gaussian_ring(cfg, k=0)[0, :, :, 0]
    b = cfg.beta0
    M0 = np.zeros((cfg.ny, cfg.nx, 4))
    M0[..., 0] = g
    M0[..., 1] = g * b * fr[0, 2]
    M0[..., 2] = g * b * fr[0, 3]
    ring = oracle.rigid_ring(M0, fr)
    for l in range(-cfg.n_pre, 0):
        _, _, c, s = W.frame(cfg, l)
        R = ring[l % cfg.H]
        np.testing.assert_array_equal(R[..., 0], g)
        np.testing.assert_allclose(R[..., 1], g * b * c, rtol=0, atol=1e-15 * g.max())
        np.testing.assert_allclose(R[..., 2], g * b * s, rtol=0, atol=1e-15 * g.max())
    # the oldest level (l = -61, psi = -0.12 rad) is rotated, not copied
    assert np.abs(ring[1, ..., 2]).max() > 0.1 * b * g.max()


def test_oracle_thread_count_overrides_the_environment():
    """bench.py's oracle legs run on all host cores even under torchrun, which exports
    OMP_NUM_THREADS=1 before torch loads libgomp; the result does not depend on the count."""
    cfg = _bend_small()
    import bench
    pts = np.arange(0, cfg.nx * cfg.ny, 97, dtype=np.int32)
    P = bench._oracle_rigid_state(cfg)
    assert oracle.set_threads(1) == 1
    r1 = P.potentials(pts)
    assert oracle.set_threads(2) == 2
    r2 = P.potentials(pts)
    assert oracle.set_threads(bench._cores()) == bench._cores()
    assert len(r1) == len(pts) and r1.tobytes() == r2.tobytes()
