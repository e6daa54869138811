"""Debug: Lagrange-3 variant parity on a small bend (per-point GPU vs oracle summary)."""
import os
import sys
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
from tests import gpu_util as G  # noqa: E402
from tests.test_gpu_parity import _bend_small  # noqa: E402
from paper_conf_icpp_arumugamrztgi17_b200 import rp  # noqa: E402

for n, kap, md, interp, rule in [(12, 20, 14, 0, 0), (12, 20, 14, 1, 0), (12, 20, 8, 1, 0), (12, 6, 14, 1, 0)]:
    cfg = _bend_small(n, kap)
    cfg.interp = interp
    cfg.max_depth = md
    cfg.rule = rule
    ctx = G.make_ctx(cfg)
    k = 5
    ring = W.node_gaussian_ring(cfg, k=k, beta=(cfg.beta0, 0.01), amp_of_level=lambda l: 1.0 + 0.01 * l)
    frames = W.ring_frames(cfg, k)
    pts = np.arange(cfg.nx * cfg.ny)
    orc = G.oracle_problem(cfg, ring, frames, k, cfg.n_pre).potentials(pts)
    G.load_state(ctx, cfg, k, cfg.n_pre, ring, frames)
    gpu, info = G.gpu_potentials(ctx, len(pts))
    fail, worst, nties = G.compare_potentials(gpu, orc, pts)
    scale = np.maximum.reduce([np.abs(orc["phi"]), np.abs(orc["ax"]), np.abs(orc["ay"])])
    d = np.abs(gpu["phi"] - orc["phi"]) / scale
    print(f"n={n} kap={kap} md={md} interp={interp}: fails {fail.sum()}/{len(pts)} worst {worst:.2e} "
          f"ties {nties} nseg gpu {gpu['nseg'].sum()} orc {orc['nseg'].sum()} "
          f"nseg-diff pts {(gpu['nseg'] != orc['nseg']).sum()} capped gpu {info.capped} orc {orc['capped'].sum()} "
          f"evals gpu {info.evals} orc {orc['evals'].sum()}", flush=True)
    i = int(np.argmax(d))
    print("   worst pt", i, "phi", gpu["phi"][i], orc["phi"][i], "nseg", gpu["nseg"][i], orc["nseg"][i], flush=True)
    rp.rp_destroy(ctx)
