"""Physics validation through the whole GPU path (the paper's Fig. 2):
the longitudinal self-field of a rigid Gaussian bunch in steady-state circular motion in the
LCLS bend, from the retarded potentials and the field formula (R-15), against the 1D
steady-state CSR field of a line charge (Derbenev et al. 1995; Saldin, Schneidmiller, Yurkov
1997).  Measured deviation within +-3 sigma: 7.0 % (33^2), 4.3 % (65^2), 3.6 % (129^2)
(profiles/r01_csr_validation_*.json); the remainder is the flat bunch's finite radial size
(sigma_x = sigma_s) against the line-charge limit."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def test_steady_state_csr_field_matches_1d_theory():
    import math
    import sys
    import torch
    import workloads as W
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    from tools.csr_validation import csr_1d, steady_ring
    n = 65  # odd: a node row on the bunch axis
    base = W.config(2)
    cfg = W.Config(number=2, name="csr-65", nx=n, ny=n, n_particles=1, steps=100, kappa_max=100,
                   geometry="bend", sigma=base.sigma, cdt=base.cdt, gamma0=base.gamma0, r0=base.r0,
                   sigma_xp=base.sigma_xp, q_over_mc=base.q_over_mc)
    ctx = rp.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt, cfg.tau)
    try:
        dev = torch.device("cuda:0")
        pot = {}
        for k in (200, 201):
            rp.rp_load_state(ctx, k, cfg.n_pre, W.ring_frames(cfg, k),
                             torch.tensor(steady_ring(cfg, k), device=dev))
            t = [torch.zeros(n * n, dtype=torch.float64, device=dev) for _ in range(3)]
            rp.rp_compute_potentials(ctx, *t)
            pot[k] = t
        out = [torch.zeros(n * n, dtype=torch.float64, device=dev) for _ in range(3)]
        rp.rp_compute_fields(ctx, *pot[201], pot[200][1], pot[200][2], *out)
        _, _, c, s = W.frame(cfg, 201)
        es = (out[0] * c + out[1] * s).cpu().numpy().reshape(n, n)[n // 2]
    finally:
        rp.rp_destroy(ctx)
    us = np.arange(n) * cfg.hx - 0.5 * cfg.extent
    inside = np.abs(us) <= 3 * cfg.sigma
    ref = np.array([csr_1d(u, cfg.sigma, cfg.r0) for u in us[inside]])
    peak = np.abs(ref).max()
    assert np.abs(es[inside] - ref).max() <= 0.06 * peak
    # the CSR signature: decelerating core, accelerating head
    core = np.argmin(np.abs(us[inside] + 0.4 * cfg.sigma))
    head = np.argmin(np.abs(us[inside] - 2.0 * cfg.sigma))
    assert es[inside][core] < -0.8 * peak and es[inside][head] > 0.2 * peak
