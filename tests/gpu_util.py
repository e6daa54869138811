"""Helpers shared by the -m gpu tests: build a librp context and an oracle problem from
the same seeded workload, and compare them element by element."""
from __future__ import annotations

import numpy as np

import oracle
import workloads as W

REL = 1e-11  # parity bar for FP64 potentials / fields (north_star)


def torch_dev():
    import torch
    assert torch.cuda.is_available(), "GPU test on a box without CUDA"
    return torch.device("cuda:0")


def make_ctx(cfg: W.Config, **over):
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    kw = dict(n_theta=cfg.n_theta, max_depth=cfg.max_depth, n_root=cfg.n_root, rule=cfg.rule,
              interp=cfg.interp)
    kw.update(over)
    return rp.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt,
                        over.get("tau", cfg.tau), kw["n_theta"], kw["max_depth"], kw["n_root"], 0,
                        kw["rule"], kw["interp"])


def oracle_problem(cfg: W.Config, ring, frames, k, n_pre, **over):
    kw = dict(nx=cfg.nx, ny=cfg.ny, hx=cfg.hx, hy=cfg.hy, c=cfg.c, dt=cfg.dt, tau=cfg.tau,
              kappa_max=cfg.kappa_max, k=k, n_pre=n_pre, ring=ring, frames=frames,
              n_theta=cfg.n_theta, max_depth=cfg.max_depth, n_root=cfg.n_root, rule=cfg.rule,
              interp=cfg.interp)
    kw.update(over)
    return oracle.Problem(**kw)


def gpu_potentials(ctx, npts):
    import torch
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    dev = torch_dev()
    out = {k: torch.zeros(npts, dtype=torch.float64, device=dev) for k in ("phi", "ax", "ay", "err")}
    nseg = torch.zeros(npts, dtype=torch.int32, device=dev)
    info = rp.rp_compute_potentials(ctx, out["phi"], out["ax"], out["ay"], out["err"], nseg, info=True)
    nleaf = torch.zeros(npts, dtype=torch.int32, device=dev)
    capped = torch.zeros(npts, dtype=torch.int32, device=dev)
    rp.rp_debug_point_counts(ctx, nleaf, capped)
    torch.cuda.synchronize()
    res = {k: v.cpu().numpy() for k, v in out.items()}
    res["nseg"] = nseg.cpu().numpy()
    res["nleaf"] = nleaf.cpu().numpy()
    res["capped"] = capped.cpu().numpy()
    return res, info


def compare_potentials(gpu: dict, orc, pts, rel=REL, tau=None):
    """Element-by-element: |delta| <= rel * max(|phi|, |ax|, |ay|)_oracle per
    point for phi, A_x, A_y and the error estimate eps (the 7-tuple's p.eps, Alg. 1
    line 23 P:148), equal nseg, and -- when the GPU result carries them -- equal per-point
    nleaf and capped.

    Points with a decision the oracle flags as rounding-determined -- relative margin
    |err - tol| / tol < 1e-9 (`ties`) or within 4 ulp of |K_rho| + |G_rho| (`noise_ties`,
    reading R-28) -- may legitimately take the other branch there: with `tau` given their
    counts are not compared and their values must agree within 4 tau per such decision (a
    flipped accept/split moves the point's sum by at most ~2 tol <= 2 tau); without `tau` they
    are only reported.  Returns (fail mask, worst relative deviation, number of such points)."""
    pts = np.asarray(pts)
    scale = np.maximum.reduce([np.abs(orc["phi"]), np.abs(orc["ax"]), np.abs(orc["ay"])])
    scale = np.where(scale > 0, scale, 1e-300)
    nflag = orc["ties"] + (orc["noise_ties"] if "noise_ties" in orc.dtype.names else 0)
    tie = nflag > 0
    bad = []
    soft = []
    keys = ("phi", "ax", "ay", "err") if "err" in gpu else ("phi", "ax", "ay")
    for key in keys:
        d = np.abs(gpu[key][pts] - orc[key])
        bad.append(d > rel * scale)
        if tau is not None:
            soft.append(d > 4.0 * tau * nflag)
    nseg_bad = gpu["nseg"][pts] != orc["nseg"]
    for key in ("nleaf", "capped"):
        if key in gpu:
            nseg_bad = nseg_bad | (gpu[key][pts] != orc[key])
    fail = (np.logical_or.reduce(bad) | nseg_bad) & ~tie
    if tau is not None:
        fail = fail | (np.logical_or.reduce(soft) & tie)
    worst = 0.0
    for key in keys:
        worst = max(worst, float(np.max(np.abs(gpu[key][pts] - orc[key]) / scale)) if len(pts) else 0.0)
    return fail, worst, int(tie.sum())


def load_state(ctx, cfg, k, n_pre, ring, frames):
    import torch
    from paper_conf_icpp_arumugamrztgi17_b200 import rp
    rt = torch.tensor(np.ascontiguousarray(ring), dtype=torch.float64, device=torch_dev())
    rp.rp_load_state(ctx, k, n_pre, frames, rt)
