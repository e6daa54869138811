"""Capped leaves of the canonical tree ("always achieves the required error tolerance";
DESIGN R-12: a leaf is accepted at D_max = 30 with err > tol, counted as capped).

    python tests/capped_analysis.py [config] [points] [--out file.json]

Test infrastructure (it runs the CPU oracle): on the rigid steady state of a config (the oracle's
own deposit of the seeded bunch + the rigid pre-history, as bench.py's reference arm), for a
stratified sample of mesh points it reports
  * the capped leaves, and the share of the integrand evaluations spent in segments whose subtree
    ends in a capped leaf (the chain of splits chasing it, plus the capped leaf itself);
  * at the points with the most capped leaves, the true error of the canonical result: the same
    integral refined to tau / 100 with D_max = 45 is the reference; |delta| is compared with tau
    and with the tree's own error estimate eps.
"""
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import workloads as W  # noqa: E402


def problem(cfg, ring, frames, **over):
    kw = dict(nx=cfg.nx, ny=cfg.ny, hx=cfg.hx, hy=cfg.hy, c=cfg.c, dt=cfg.dt, tau=cfg.tau,
              kappa_max=cfg.kappa_max, k=0, n_pre=cfg.n_pre, ring=ring, frames=frames,
              n_theta=cfg.n_theta, max_depth=cfg.max_depth, n_root=cfg.n_root)
    kw.update(over)
    return oracle.Problem(**kw)


def analyse(cfgno=2, npts=400, worst=5):
    cfg = W.config(cfgno)
    x, y, ux, uy = W.particles(cfg)
    M, _, _ = oracle.deposit(x, y, ux, uy, 1.0 / len(x), W.frame(cfg, 0), cfg.nx, cfg.ny,
                             cfg.hx, cfg.hy)
    frames = W.ring_frames(cfg, 0)
    ring = oracle.rigid_ring(M, frames)
    pts = W.sample_points(cfg.nx, cfg.ny, npts, seed=11)
    t0 = time.perf_counter()
    res = problem(cfg, ring, frames).potentials(pts)
    t_canon = time.perf_counter() - t0
    out = {"config": cfg.name, "tau": cfg.tau, "max_depth": cfg.max_depth, "points": int(len(pts)),
           "oracle_s": t_canon,
           "capped_leaves": int(res["capped"].sum()), "leaves": int(res["nleaf"].sum()),
           "points_with_capped": int((res["capped"] > 0).sum()),
           "evals": int(res["evals"].sum()), "chase_evals": int(res["chase_evals"].sum()),
           "segments": int(res["nseg"].sum()), "chase_segments": int(res["chase_segs"].sum())}
    out["chase_eval_share"] = out["chase_evals"] / out["evals"]
    order = np.argsort(-res["capped"])[:worst]
    ref = problem(cfg, ring, frames, tau=cfg.tau / 100, max_depth=45).potentials(pts[order])
    rows = []
    for i, r in zip(order, ref):
        c = res[i]
        d = max(abs(c["phi"] - r["phi"]), abs(c["ax"] - r["ax"]), abs(c["ay"] - r["ay"]))
        rows.append({"point": int(pts[i]), "capped": int(c["capped"]), "err_estimate": float(c["err"]),
                     "true_error": float(d), "true_error_over_tau": float(d / cfg.tau),
                     "phi": float(c["phi"]), "ref_capped": int(r["capped"])})
    out["worst_points"] = rows
    out["max_true_error_over_tau"] = max(r["true_error_over_tau"] for r in rows)
    return out


if __name__ == "__main__":
    cfgno = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 2
    n = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2].isdigit() else 400
    oracle.set_threads(os.cpu_count() or 1)
    o = analyse(cfgno, n)
    print(json.dumps({k: v for k, v in o.items() if k != "worst_points"}))
    for r in o["worst_points"]:
        print(r)
    if "--out" in sys.argv:
        json.dump(o, open(sys.argv[sys.argv.index("--out") + 1], "w"), indent=1)
