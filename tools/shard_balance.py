"""Multi-GPU projection from one GPU: the per-rank integrator time of the mesh-point shards.

With N GPUs each rank integrates its shard of mesh points (dealt longest-predicted-first in a
snake order from the previous step's segment counts) against the replicated
history; the only exchanges are two small all-gathers per step.  So the N-GPU step time is the
slowest shard's time plus the exchange.  This tool runs a config for a few steps on one GPU,
then, from the same state, computes every shard of every N in {1, 2, 4, 8} through the product
call (`rp_compute_potentials_shard`) and times each with CUDA events.  It also checks that the
scattered shards reproduce the single-call result bit for bit.

usage: python tools/shard_balance.py [config] [warm steps]
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
warm = int(sys.argv[2]) if len(sys.argv) > 2 else 3
cfg = W.config(cfgn)
sim = Simulation(cfg)
for _ in range(warm):
    sim.step()
# the next step's history: deposit it, then integrate it whole and in shards
fk = W.frame(cfg, sim.k)
rp.rp_deposit_step(sim.ctx, sim.x, sim.y, sim.ux, sim.uy, sim.q, fk)
npts = cfg.nx * cfg.ny
f64 = dict(dtype=torch.float64, device="cuda")
# shards first: their point map comes from the previous step's counts, as in a real N-GPU run
per_n, scattered = {}, {}
for world in (1, 2, 4, 8):
    cap = rp.rp_shard_capacity(sim.ctx, world)
    shards = torch.zeros((world, cap, 6), **f64)
    times, evals, units = [], [], []
    for r in range(world):
        rp.rp_profile_enable(sim.ctx, True)
        n, inf = rp.rp_compute_potentials_shard(sim.ctx, r, world, shards[r], info=True)
        pr = rp.rp_profile_read(sim.ctx)
        times.append(pr.integrate_ms)
        units.append(round(pr.units_ms, 3))
        evals.append(inf.evals)
    res = {k: torch.zeros(npts, **f64) for k in ("phi", "ax", "ay", "err")}
    ns = torch.zeros(npts, dtype=torch.int32, device="cuda")
    rp.rp_shard_scatter(sim.ctx, shards, world, res["phi"], res["ax"], res["ay"], res["err"], ns)
    scattered[world] = (res, ns)
    per_n[world] = {"shard_ms": [round(t, 3) for t in times], "units_ms": units,
                    "max_ms": max(times),
                    "evals_imbalance": max(evals) / (sum(evals) / world)}
full = {k: torch.zeros(npts, **f64) for k in ("phi", "ax", "ay", "err")}
nseg = torch.zeros(npts, dtype=torch.int32, device="cuda")
rp.rp_profile_enable(sim.ctx, True)
info = rp.rp_compute_potentials(sim.ctx, full["phi"], full["ax"], full["ay"], full["err"], nseg,
                                info=True)
t_full = rp.rp_profile_read(sim.ctx).integrate_ms
torch.cuda.synchronize()
for world, (res, ns) in scattered.items():
    per_n[world]["bit_identical_to_single_call"] = (
        all(torch.equal(res[k], full[k]) for k in res) and torch.equal(ns, nseg))
out = {"config": cfg.name, "step": sim.k, "evals": info.evals, "single_call_ms": t_full,
       "per_n": per_n}
base = out["per_n"][1]["max_ms"]
for world, d in out["per_n"].items():
    d["projected_speedup"] = base / d["max_ms"]
    d["projected_efficiency"] = base / (world * d["max_ms"])
print(json.dumps(out), flush=True)
sim.close()
