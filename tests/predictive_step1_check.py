"""Where the Predictive-RP variant and the canonical tree differ most.

    python tests/predictive_step1_check.py [config] [m] [part]

Test infrastructure (it runs the CPU oracle on the GPU's state): two simulations of a config
side by side, the second with Predictive-RP (rp_set_predictive, m clusters, line 4 by
uniform (part 0) or adaptive (part 1) partitioning); after step 1 (the first forecast step,
both starting from the same state) it takes the points with the largest |phi_pred -
phi_canon|, copies the ring out (rp_save_state) and evaluates there with the oracle: the
canonical tree (tau), a reference refined to tau / 100 with D_max = 45, and the per-item
breakdown of the difference.  Prints one JSON line.
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import workloads as W  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200 import rp  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200.sim import Simulation  # noqa: E402

cfgn = int(sys.argv[1]) if len(sys.argv) > 1 else 2
m = int(sys.argv[2]) if len(sys.argv) > 2 else 0
part = int(sys.argv[3]) if len(sys.argv) > 3 else 0
cfg = W.config(cfgn)
a, b = Simulation(cfg), Simulation(cfg)
rp.rp_set_predictive(b.ctx, True, 9, m, 20)
rp.rp_set_predictive_partition(b.ctx, part)
for _ in range(2):
    a.step()
    b.step()
torch.cuda.synchronize()
d = (a.phi - b.phi).abs().cpu().numpy()
top = np.argsort(-d)[:5]
ring = torch.zeros(cfg.H * cfg.ny * cfg.nx * 4, dtype=torch.float64, device="cuda")
k, frames = rp.rp_save_state(a.ctx, ring, cfg.H)
ring = ring.cpu().numpy().reshape(cfg.H, cfg.ny, cfg.nx, 4)
kw = dict(nx=cfg.nx, ny=cfg.ny, hx=cfg.hx, hy=cfg.hy, c=cfg.c, dt=cfg.dt, tau=cfg.tau,
          kappa_max=cfg.kappa_max, k=k, n_pre=cfg.n_pre, ring=ring, frames=frames,
          n_theta=cfg.n_theta, max_depth=cfg.max_depth, n_root=cfg.n_root)
P = oracle.Problem(**kw)
kw2 = dict(kw, tau=cfg.tau / 100, max_depth=45)
Pref = oracle.Problem(**kw2)
orc, _ = P.potentials_items(top)
ref, _ = Pref.potentials_items(top)
phi_a, phi_b = a.phi.cpu().numpy(), b.phi.cpu().numpy()
rows = []
for i, p in enumerate(top):
    rows.append(dict(point=int(p), dphi_over_tau=float(d[p] / cfg.tau),
                     canon_gpu_minus_ref=float((phi_a[p] - ref["phi"][i]) / cfg.tau),
                     pred_gpu_minus_ref=float((phi_b[p] - ref["phi"][i]) / cfg.tau),
                     canon_oracle_minus_ref=float((orc["phi"][i] - ref["phi"][i]) / cfg.tau),
                     canon_capped=int(orc["capped"][i]), ref_capped=int(ref["capped"][i]),
                     canon_eps_over_tau=float(orc["err"][i] / cfg.tau)))
print(json.dumps({"config": cfg.name, "m": m, "part": part, "step": k, "tau": cfg.tau,
                  "points": rows}), flush=True)
a.close()
b.close()
