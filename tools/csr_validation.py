"""Physics validation in the LCLS bend (the paper's Fig. 2): the
longitudinal self-field of a rigid Gaussian bunch in steady-state circular motion, computed
through the whole GPU path (retarded potentials -> fields), against the 1D steady-state CSR
field of a line charge (Derbenev et al. 1995; Saldin, Schneidmiller, Yurkov 1997):

    E_s(s) = -2 Q / (3^(1/3) R^(2/3)) * int_0^inf x^(-1/3) lambda'(s - x) dx      (Gaussian units)

The history is noise-free (node samples of the Gaussian, current along each level's tangent),
so the comparison tests the integrator and the field formula rather than particle noise.

    python tools/csr_validation.py [n] [--out file.json]
"""
import json
import math
import os
import sys

import numpy as np
import scipy.integrate as si
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import workloads as W  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200 import rp  # noqa: E402


def steady_ring(cfg, k):
    """Ring at step k: every level is the same comoving Gaussian, current along the level's
    tangent (lab components)."""
    H = cfg.H
    u = np.arange(cfg.nx) * cfg.hx
    v = np.arange(cfg.ny) * cfg.hy
    U, V = np.meshgrid(u, v)
    half = 0.5 * cfg.extent
    g = np.exp(-((U - half) ** 2 + (V - half) ** 2) / (2 * cfg.sigma ** 2)) / (2 * math.pi * cfg.sigma ** 2)
    ring = np.zeros((H, cfg.ny, cfg.nx, 4))
    for l in range(k - H + 1, k + 1):
        _, _, c, s = W.frame(cfg, l)
        ring[l % H, :, :, 0] = g
        ring[l % H, :, :, 1] = g * cfg.beta0 * c
        ring[l % H, :, :, 2] = g * cfg.beta0 * s
    return ring


def csr_1d(s, sigma, R):
    lam_p = lambda x: -x / sigma ** 2 * math.exp(-x * x / (2 * sigma ** 2)) / (math.sqrt(2 * math.pi) * sigma)
    f = lambda x: x ** (-1.0 / 3.0) * lam_p(s - x)
    val, _ = si.quad(f, 0, s + 12 * sigma, limit=400, points=[max(s, 1e-30)] if s > 0 else None)
    if s + 12 * sigma < 0:
        val = 0.0
    return -2.0 / (3 ** (1 / 3) * R ** (2 / 3)) * val


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 64
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
    base = W.config(2)
    cfg = W.Config(number=2, name=f"csr-{n}", nx=n, ny=n, n_particles=1, steps=100, kappa_max=100,
                   geometry="bend", sigma=base.sigma, cdt=base.cdt, gamma0=base.gamma0, r0=base.r0,
                   sigma_xp=base.sigma_xp, q_over_mc=base.q_over_mc)
    ctx = rp.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt, cfg.tau)
    npts = n * n
    dev = torch.device("cuda:0")
    res = {}
    for k in (200, 201):
        ring = torch.tensor(steady_ring(cfg, k), device=dev)
        rp.rp_load_state(ctx, k, cfg.n_pre, W.ring_frames(cfg, k), ring)
        phi, ax, ay = (torch.zeros(npts, dtype=torch.float64, device=dev) for _ in range(3))
        rp.rp_compute_potentials(ctx, phi, ax, ay)
        res[k] = (phi, ax, ay)
    phi, ax, ay = res[201]
    _, axp, ayp = res[200]
    ex, ey, bz = (torch.zeros(npts, dtype=torch.float64, device=dev) for _ in range(3))
    rp.rp_compute_fields(ctx, phi, ax, ay, axp, ayp, ex, ey, bz)
    torch.cuda.synchronize()
    _, _, c, s = W.frame(cfg, 201)
    es = (ex * c + ey * s).cpu().numpy().reshape(n, n)
    row = es[n // 2]  # the node row through the bunch centre (v = 5 sigma)
    us = np.arange(n) * cfg.hx - 0.5 * cfg.extent
    ref = np.array([csr_1d(u, cfg.sigma, cfg.r0) for u in us])
    inside = np.abs(us) <= 3 * cfg.sigma
    peak = np.abs(ref[inside]).max()
    err = np.abs(row[inside] - ref[inside]).max() / peak
    rec = {"mesh": n, "sigma": cfg.sigma, "R0": cfg.r0, "peak_csr_field": peak,
           "max_rel_deviation_within_3sigma": err,
           "s_over_sigma": (us[inside] / cfg.sigma).tolist(), "computed": row[inside].tolist(),
           "csr_1d": ref[inside].tolist()}
    print(json.dumps({k: v for k, v in rec.items() if not isinstance(v, list)}))
    for a, b, cc in zip(rec["s_over_sigma"][::4], rec["computed"][::4], rec["csr_1d"][::4]):
        print(f"  s/sigma {a:+6.2f}  computed {b:+.5e}  1D CSR {cc:+.5e}")
    if out:
        json.dump(rec, open(out, "w"), indent=1)
    rp.rp_destroy(ctx)


if __name__ == "__main__":
    main()
