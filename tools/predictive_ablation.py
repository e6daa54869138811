"""Ablation: the paper's Predictive-RP partitioning (Algorithm 1, R-26) against the canonical
dyadic tree on one B200, same workload, same steps.

Two simulations of a config run side by side.  Step 0 has no observed pattern (both run the
canonical tree, identical results and states); from step 1 the second one forecasts,
clusters and merges.  Step 1 starts from the same state in both, so its max |phi_pred -
phi_canon| / tau measures the forecast dependence of the result; later steps
drift apart by that much.  Per step: integrator time (CUDA events), host time of the
forecast/cluster/merge pipeline, integrand evaluations and segments.  usage: python tools/predictive_ablation.py [config] [steps] [knn] [m] [part]
(part: 0 uniform partitioning; 1 adaptive partitioning, P:104 / R-26b)
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
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 4
knn = int(sys.argv[3]) if len(sys.argv) > 3 else 9
m = int(sys.argv[4]) if len(sys.argv) > 4 else 0
part = int(sys.argv[5]) if len(sys.argv) > 5 else 0
cfg = W.config(cfgn)
a, b = Simulation(cfg), Simulation(cfg)
rp.rp_set_predictive(b.ctx, True, knn, m, 20)
rp.rp_set_predictive_partition(b.ctx, part)
for s in (a, b):
    rp.rp_profile_enable(s.ctx, True)
rows = []
last = [0.0, 0.0]
for k in range(steps):
    ia = a.step(info=True)
    ib = b.step(info=True)
    torch.cuda.synchronize()
    pa, pb = rp.rp_profile_read(a.ctx), rp.rp_profile_read(b.ctx)
    pinfo = rp.rp_predictive_info_read(b.ctx)
    d = float((a.phi - b.phi).abs().max()) / cfg.tau
    rows.append(dict(step=k, canon_ms=pa.integrate_ms - last[0], pred_ms=pb.integrate_ms - last[1],
                     pred_host_ms=pinfo.host_ms if pinfo.active else 0.0,
                     active=pinfo.active, partition=pinfo.partition if pinfo.active else None,
                     clusters=pinfo.clusters, passes=pinfo.kmeans_passes,
                     breakpoints=pinfo.breakpoints, canon_evals=ia.evals, pred_evals=ib.evals,
                     canon_segments=ia.segments, pred_segments=ib.segments,
                     max_dphi_over_tau=d))
    last = [pa.integrate_ms, pb.integrate_ms]
    print(json.dumps(rows[-1]), flush=True)
act = [r for r in rows if r["active"]]
if act:
    print(json.dumps({"summary": True, "config": cfg.name, "knn": knn, "m": m, "part": part,
                      "canon_ms": float(np.mean([r["canon_ms"] for r in act])),
                      "pred_ms": float(np.mean([r["pred_ms"] for r in act])),
                      "pred_host_ms": float(np.mean([r["pred_host_ms"] for r in act])),
                      "evals_ratio": float(np.mean([r["pred_evals"] / r["canon_evals"] for r in act])),
                      "first_step_max_dphi_over_tau": act[0]["max_dphi_over_tau"]}))
a.close()
b.close()
