"""True error of the canonical tree over a whole mesh ("ensures that integral estimate
always achieves the required error tolerance").

    python tools/true_error_scan.py [config] [steps]

A simulation of the config runs `steps` steps through librp; after each step's potentials its
state (ring, frames) is loaded into a second context built with tau / 100 and D_max = 45 (the
reference of tests/capped_analysis.py, here on the GPU for every mesh point; the GPU matches
the oracle to 1e-11 on both settings), and the canonical result is compared with it per
point.  Prints one JSON line per step: the largest |phi - phi_ref| / tau and |A - A_ref| / tau,
how many points exceed tau and tau / 2, the worst point, and its own estimate eps / tau.
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200 import rp  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation  # noqa: E402

cfgn = int(sys.argv[1]) if len(sys.argv) > 1 else 2
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
cfg = W.config(cfgn)
if len(sys.argv) > 3:  # canonical roots (R-12b): 1, 2 or 4 equal pieces of the support
    cfg.n_root = int(sys.argv[3])
sim = Simulation(cfg)
npts = cfg.nx * cfg.ny
ref = rp.rp_create(cfg.nx, cfg.ny, cfg.hx, cfg.hy, cfg.kappa_max, cfg.c, cfg.dt, cfg.tau / 100,
                   cfg.n_theta, 45, cfg.n_root, 0)
f64 = dict(dtype=torch.float64, device="cuda")
out = [torch.zeros(npts, **f64) for _ in range(4)]
nseg = torch.zeros(npts, dtype=torch.int32, device="cuda")
ring = torch.zeros(cfg.H * npts * 4, **f64)
rp.rp_profile_enable(sim.ctx, True)
last_ms = 0.0
for s in range(steps):
    own = sim.step(info=True)
    torch.cuda.synchronize()
    prof = rp.rp_profile_read(sim.ctx)
    own_ms, last_ms = prof.integrate_ms - last_ms, prof.integrate_ms
    k, frames = rp.rp_save_state(sim.ctx, ring, cfg.H)
    rp.rp_load_state(ref, k, cfg.n_pre, frames, ring)
    info = rp.rp_compute_potentials(ref, *out, nseg, info=True)
    torch.cuda.synchronize()
    dphi = (sim.phi - out[0]).abs().cpu().numpy() / cfg.tau
    dA = torch.maximum((sim.Ahist[0, 0] - out[1]).abs(), (sim.Ahist[0, 1] - out[2]).abs())
    dA = dA.cpu().numpy() / cfg.tau
    worst = int(np.argmax(dphi))
    print(json.dumps({"config": cfg.name, "step": k, "max_dphi_over_tau": float(dphi.max()),
                      "max_dA_over_tau": float(dA.max()),
                      "points_over_tau": int((np.maximum(dphi, dA) > 1).sum()),
                      "points_over_half_tau": int((np.maximum(dphi, dA) > 0.5).sum()),
                      "p99_dphi_over_tau": float(np.quantile(dphi, 0.99)),
                      "median_dphi_over_tau": float(np.median(dphi)),
                      "worst_point": worst,
                      "worst_eps_over_tau": float(sim.err[worst].item() / cfg.tau),
                      "ref_capped": int(info.capped), "ref_segments": int(info.segments),
                      "n_root": cfg.n_root, "segments": int(own.segments), "evals": int(own.evals),
                      "integrate_ms": own_ms}),
          flush=True)
rp.rp_destroy(ref)
sim.close()
